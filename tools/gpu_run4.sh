set -x
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1
./tools/lop3_peak > gpurun_out/lop3_peak.json 2>&1 || (nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/lop3_peak tools/lop3_peak.cu && /tmp/lop3_peak > gpurun_out/lop3_peak.json 2>&1)
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
echo done
