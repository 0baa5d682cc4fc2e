set -x
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q -k "long or c5 or striped or m256" > gpurun_out/pytest_gpu.log 2>&1
B="python bench.py --no-cpu-baseline --no-e2e --no-filter --steps 5"
timeout 300 $B --config 4 > gpurun_out/x_c4_def.json 2>/dev/null
BPBC_MAX_BLOCKS_PER_SM=4 timeout 300 $B --config 4 > gpurun_out/x_c4_b4.json 2>/dev/null
BPBC_MAX_BLOCKS_PER_SM=3 timeout 300 $B --config 2 > gpurun_out/x_c2_b3.json 2>/dev/null
timeout 300 $B --config 2 > gpurun_out/x_c2_def.json 2>/dev/null
timeout 300 $B --config 5 > gpurun_out/x_c5_r4.json 2>/dev/null
BPBC_STRIPE_R=2 timeout 300 $B --config 5 > gpurun_out/x_c5_r2.json 2>/dev/null
timeout 300 $B --config 1 > gpurun_out/x_c1.json 2>/dev/null
echo done
