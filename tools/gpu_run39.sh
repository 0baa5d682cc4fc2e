# A/B: multi-warp (R, W) = (8, 2) at 6 / 5 blocks per SM vs (4, 4) for 257..512 rows
set -x
mkdir -p gpurun_out
for t in mw8 mw8b5 main; do
  L=exp_libs/$t.so; [ $t = main ] && L=paper_conf_ipps_nishimurabin17_b200/libbpbc_sw.so
  BPBC_SW_LIB=$L timeout 900 python tools/c5_sweep.py --m 512 --s 9,10,11 --out gpurun_out/r39_$t.json > gpurun_out/r39_$t.log 2>&1
  BPBC_SW_LIB=$L timeout 300 python bench.py --no-cpu-baseline --no-e2e --no-filter --steps 5 --config 5 --m 384 --n 384 --pairs 2097152 > gpurun_out/r39_${t}_m384.json 2>/dev/null
done
echo done
