# A/B: per-phase chunk position without 64-bit division (ydiv) vs main
set -x
mkdir -p gpurun_out
B="python bench.py --no-cpu-baseline --no-e2e --no-filter --steps 10"
for rep in 1 2; do
for t in ydiv main; do
  L=exp_libs/$t.so; [ $t = main ] && L=paper_conf_ipps_nishimurabin17_b200/libbpbc_sw.so
  for c in 2 3 4; do BPBC_SW_LIB=$L timeout 300 $B --config $c > gpurun_out/r50_${t}_c${c}_$rep.json 2>/dev/null; done
  BPBC_SW_LIB=$L timeout 300 $B --config 5 --m 32 --n 32 --score-bits 7 > gpurun_out/r50_${t}_m32_$rep.json 2>/dev/null
  BPBC_SW_LIB=$L timeout 300 $B --config 5 --m 64 --n 64 --score-bits 8 > gpurun_out/r50_${t}_m64_$rep.json 2>/dev/null
done
done
echo done
