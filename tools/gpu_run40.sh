# multi-warp W = 3 for 257..384 rows: GPU suite, sanitizers, m = 300 / 384 bench
set -x
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r40_pytest_gpu.log 2>&1
timeout 900 compute-sanitizer --tool memcheck python tests/sanitize_run.py > gpurun_out/r40_memcheck.log 2>&1
timeout 900 compute-sanitizer --tool racecheck python tests/sanitize_run.py > gpurun_out/r40_racecheck.log 2>&1
timeout 900 compute-sanitizer --tool synccheck python tests/sanitize_run.py > gpurun_out/r40_synccheck.log 2>&1
B="python bench.py --no-cpu-baseline --no-e2e --no-filter --steps 5"
timeout 300 $B --config 5 --m 384 --n 384 --pairs 2097152 > gpurun_out/r40_m384.json 2>/dev/null
timeout 300 $B --config 5 --m 300 --n 300 --pairs 2097152 --score-bits 10 > gpurun_out/r40_m300.json 2>/dev/null
timeout 300 $B --config 5 > gpurun_out/r40_c5.json 2>/dev/null
echo done
