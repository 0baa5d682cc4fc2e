# multi-warp blocks of whole SMSP sets (W = 2: two groups per block): GPU suite + sanitizers on the new
# build; wide-plane W = 2 and C5 point (W = 4) new vs old
set -x
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r41_pytest_gpu.log 2>&1
timeout 900 compute-sanitizer --tool racecheck python tests/sanitize_run.py > gpurun_out/r41_racecheck.log 2>&1
timeout 900 compute-sanitizer --tool synccheck python tests/sanitize_run.py > gpurun_out/r41_synccheck.log 2>&1
for t in new old; do
  L=exp_libs/$t.so; [ $t = new ] && L=paper_conf_ipps_nishimurabin17_b200/libbpbc_sw.so
  for rep in 1 2; do
  BPBC_SW_LIB=$L timeout 300 python tools/wide_plane_bench.py > gpurun_out/r41_${t}_wide_$rep.log 2>&1
  BPBC_SW_LIB=$L timeout 300 python tools/wide_plane_bench.py --m 160 --n 160 --pairs 1048576 --consts 9,-3,-2 --s 14 > gpurun_out/r41_${t}_wide160_$rep.log 2>&1
  done
  BPBC_SW_LIB=$L timeout 300 python bench.py --no-cpu-baseline --no-e2e --no-filter --steps 5 --config 5 > gpurun_out/r41_${t}_c5.json 2>/dev/null
done
echo done
