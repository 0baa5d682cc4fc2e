set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r22_smi.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r22_smoke.log 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/r22_pytest_gpu.log 2>&1
timeout 600 python bench.py > gpurun_out/r22_bench.json 2> gpurun_out/r22_bench.err
echo done
