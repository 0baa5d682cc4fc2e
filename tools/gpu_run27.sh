# ssub without the materialised first borrow (90 LOP3 per word-cell at C2)
set -x
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/r27_pytest_gpu.log 2>&1
B="python bench.py --no-cpu-baseline --no-e2e --no-filter --steps 10"
for c in 2 3 4 5 6; do timeout 300 $B --config $c > gpurun_out/r27_c$c.json 2>/dev/null; done
echo done
