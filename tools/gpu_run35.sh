# (R, L) = (4, 8) for m <= 32 on the fused kernel: GPU suite, C5 m=32 row, C1
set -x
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r35_pytest_gpu.log 2>&1
timeout 600 python tools/c5_sweep.py --m 32,64 --s 6,7,8 --out gpurun_out/r35_c5.json > gpurun_out/r35_c5.log 2>&1
timeout 300 python bench.py --no-e2e --no-filter --config 1 > gpurun_out/r35_c1.json 2>/dev/null
echo done
