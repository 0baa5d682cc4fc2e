# exact circuit with runtime constants: GPU suite, memcheck, A/B vs the saturating runtime circuit
set -x
mkdir -p gpurun_out
BPBC_NO_EXACT_RUN=0 timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r51_pytest_gpu.log 2>&1
timeout 900 compute-sanitizer --tool memcheck python tests/sanitize_run.py > gpurun_out/r51_memcheck.log 2>&1
for k in 0 1; do
  for c in "1,-1,-1" "3,-2,-2" "1,-3,-5" "5,-4,-4"; do
    BPBC_NO_EXACT_RUN=$k timeout 300 python tools/wide_plane_bench.py --pairs 1048576 --m 128 --n 128 --consts=$c --s 16 >> gpurun_out/r51_ab_$k.log 2>&1
  done
  BPBC_NO_EXACT_RUN=$k timeout 300 python tools/wide_plane_bench.py --pairs 1048576 --m 64 --n 1024 --consts=1,-1,-1 --s 16 >> gpurun_out/r51_ab_$k.log 2>&1
  BPBC_NO_EXACT_RUN=$k timeout 300 python tools/wide_plane_bench.py --pairs 1048576 --m 256 --n 256 --consts=1,-1,-1 --s 16 >> gpurun_out/r51_ab_$k.log 2>&1
done
echo done
