# full GPU suite incl. the short-target fused tests; smoke
set -x
mkdir -p gpurun_out
timeout 300 python -c 'import __graft_entry__ as g; g.smoke()' > gpurun_out/r36_smoke.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r36_pytest_gpu.log 2>&1
echo done
