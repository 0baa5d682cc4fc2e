# bench line with parity from the cpu_baseline leg; C5 sweep (35 points)
set -x
mkdir -p gpurun_out
timeout 600 python bench.py > gpurun_out/r33_bench.json 2> gpurun_out/r33_bench.err
timeout 2400 python tools/c5_sweep.py --out gpurun_out/r33_c5_sweep.json > gpurun_out/r33_c5_sweep.log 2>&1
echo done
