# switch-phase cost: m = 128 at n = 128..2048, same cell count as C2
set -x
mkdir -p gpurun_out
B="python bench.py --no-cpu-baseline --no-e2e --no-filter --steps 10"
for n in 128 256 512 1024 2048; do
  P=$(( 1048576 * 128 / n ))
  timeout 300 $B --config 2 --n $n --pairs $P > gpurun_out/r37_n$n.json 2>/dev/null
done
echo done
