# exact runtime circuit on every kernel family: GPU suite, sanitizers, A/B on m = 300 / 512
set -x
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r53_pytest_gpu.log 2>&1
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool python tests/sanitize_run.py > gpurun_out/r53_$tool.log 2>&1
done
for k in 0 1; do
  BPBC_NO_EXACT_RUN=$k timeout 300 python tools/wide_plane_bench.py --pairs 1048576 --m 384 --n 384 --consts=1,-1,-1 --s 16 >> gpurun_out/r53_ab_$k.log 2>&1
  BPBC_NO_EXACT_RUN=$k timeout 300 python tools/wide_plane_bench.py --pairs 524288 --m 512 --n 512 --consts=3,-2,-2 --s 16 >> gpurun_out/r53_ab_$k.log 2>&1
  BPBC_NO_EXACT_RUN=$k timeout 300 python tools/wide_plane_bench.py --pairs 65536 --m 1000 --n 1000 --consts=1,-1,-1 --s 16 >> gpurun_out/r53_ab_$k.log 2>&1
done
timeout 300 python bench.py --no-cpu-baseline --no-e2e --no-filter --steps 10 > gpurun_out/r53_c2.json 2>/dev/null
echo done
