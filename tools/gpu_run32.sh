# A/B: per-warp early exit (ee, 4 blocks/SM), + 5 blocks/SM at 96 registers (ee5), vs pred
set -x
mkdir -p gpurun_out
B="python bench.py --no-cpu-baseline --no-e2e --no-filter --steps 10"
for rep in 1 2; do
for t in ee ee5 pred; do
  for c in 2 4 6; do
    L=exp_libs/$t.so; [ $t = pred ] && L=paper_conf_ipps_nishimurabin17_b200/libbpbc_sw.so
    BPBC_SW_LIB=$L timeout 300 $B --config $c > gpurun_out/r32_${t}_c${c}_$rep.json 2>gpurun_out/r32_${t}_c${c}.err
  done
done
done
echo done
