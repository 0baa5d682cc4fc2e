# multi-warp W = 3 (four groups per 12-warp block, dynamic shared memory): GPU suite, sanitizers, m = 300 / 384
set -x
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r42_pytest_gpu.log 2>&1
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool python tests/sanitize_run.py > gpurun_out/r42_$tool.log 2>&1
done
B="python bench.py --no-cpu-baseline --no-e2e --no-filter --steps 5"
timeout 300 $B --config 5 --m 384 --n 384 --pairs 2097152 > gpurun_out/r42_m384.json 2>/dev/null
timeout 300 $B --config 5 --m 320 --n 320 --pairs 2097152 --score-bits 10 > gpurun_out/r42_m320.json 2>/dev/null
timeout 300 $B --config 5 > gpurun_out/r42_c5.json 2>/dev/null
echo done
