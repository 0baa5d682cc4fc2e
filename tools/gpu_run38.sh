# A/B: (R, L) = (8, 16) for 64 < m <= 128 (branch / predicated switch) vs (4, 32)
set -x
mkdir -p gpurun_out
B="python bench.py --no-cpu-baseline --no-e2e --no-filter --steps 10"
for t in r816 r816p main; do
  L=exp_libs/$t.so; [ $t = main ] && L=paper_conf_ipps_nishimurabin17_b200/libbpbc_sw.so
  BPBC_SW_LIB=$L timeout 300 $B --config 2 > gpurun_out/r38_${t}_c2.json 2>/dev/null
  BPBC_SW_LIB=$L timeout 300 $B --config 6 > gpurun_out/r38_${t}_c6.json 2>/dev/null
  BPBC_SW_LIB=$L timeout 300 $B --config 2 --n 256 --pairs 524288 > gpurun_out/r38_${t}_n256.json 2>/dev/null
done
echo done
