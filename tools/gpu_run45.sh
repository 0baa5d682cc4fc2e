# A/B: multi-warp W = 4 at 12 warps/SM + block model preferring more warps within 1 % (mw12), model only (tol), main
set -x
mkdir -p gpurun_out
for t in mw12 tol main; do
  L=exp_libs/$t.so; [ $t = main ] && L=paper_conf_ipps_nishimurabin17_b200/libbpbc_sw.so
  BPBC_SW_LIB=$L timeout 900 python tools/c5_sweep.py --m 64,512 --s 8,9,11 --out gpurun_out/r45_$t.json > gpurun_out/r45_$t.log 2>&1
  BPBC_SW_LIB=$L timeout 300 python bench.py --no-cpu-baseline --no-e2e --no-filter --steps 5 --config 5 --m 448 --n 448 --pairs 2097152 > gpurun_out/r45_${t}_m448.json 2>/dev/null
  BPBC_SW_LIB=$L timeout 300 python bench.py --no-cpu-baseline --no-e2e --no-filter --steps 10 --config 2 > gpurun_out/r45_${t}_c2.json 2>/dev/null
done
echo done
