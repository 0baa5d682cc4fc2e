# A/B: target chunks staged by cp.async one phase ahead (stage) vs direct loads (pred)
set -x
mkdir -p gpurun_out
B="python bench.py --no-cpu-baseline --no-e2e --no-filter --steps 10"
for rep in 1 2; do
for t in stage pred; do
  for c in 2 3 4 6; do
    BPBC_SW_LIB=exp_libs/$t.so timeout 300 $B --config $c > gpurun_out/r31_${t}_c${c}_$rep.json 2>gpurun_out/r31_${t}_c${c}.err
  done
done
done
echo done
