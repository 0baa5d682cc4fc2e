set -x
mkdir -p gpurun_out
ls build 2>&1 | head -3 > gpurun_out/pushed_build.txt
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1
timeout 300 compute-sanitizer --tool racecheck python -m pytest tests/test_gpu_parity.py -q -k "few_long" > gpurun_out/san_skew.log 2>&1
B="python bench.py --no-cpu-baseline --no-e2e --no-filter --steps 5"
timeout 300 $B --config 6 > gpurun_out/bench_c6.json 2>/dev/null
BPBC_NO_SKEW=1 timeout 300 $B --config 6 > gpurun_out/x_c6_noskew.json 2>/dev/null
timeout 300 $B --config 6 --n 16384 > gpurun_out/x_c6_n16k.json 2>/dev/null
BPBC_NO_SKEW=1 timeout 300 $B --config 6 --n 16384 > gpurun_out/x_c6_n16k_noskew.json 2>/dev/null
echo done
