# R=8 single loop (I-cache); switch-cost probe: C2 shape with n=1024 (same cells)
set -x
mkdir -p gpurun_out
B="python bench.py --no-cpu-baseline --no-e2e --no-filter --steps 10"
for c in 3 2; do timeout 300 $B --config $c > gpurun_out/r24_c$c.json 2>/dev/null; done
timeout 300 $B --config 2 --n 1024 --pairs 131072 > gpurun_out/r24_c2_n1024.json 2>/dev/null
timeout 300 $B --config 2 --n 512 --pairs 262144 > gpurun_out/r24_c2_n512.json 2>/dev/null
timeout 300 $B --config 2 --n 256 --pairs 524288 > gpurun_out/r24_c2_n256.json 2>/dev/null
echo done
