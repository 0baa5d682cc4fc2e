set -x
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench.json 2> gpurun_out/bench.err
B="python bench.py --no-cpu-baseline --no-e2e --no-filter --steps 5"
for c in 3 4 5 6; do timeout 300 $B --config $c > gpurun_out/bench_c$c.json 2>/dev/null; done
BPBC_NO_MULTIWARP=1 timeout 300 $B --config 5 > gpurun_out/x_c5_nomw.json 2>/dev/null
BPBC_NO_MULTIWARP=1 timeout 300 $B --config 6 > gpurun_out/x_c6_nomw.json 2>/dev/null
echo done
