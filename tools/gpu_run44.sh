# ncu full: multi-warp W = 4 (C5 point, m = 512) and W = 3 (m = 384)
set -x
mkdir -p gpurun_out
B="python bench.py --no-cpu-baseline --no-e2e --no-filter --steps 1 --warmup 3"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"sw_sweep_mw" -c 1 -o gpurun_out/r44_mw4 $B --config 5 --pairs 524288 > gpurun_out/r44_mw4.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"sw_sweep_mw" -c 1 -o gpurun_out/r44_mw3 $B --config 5 --m 384 --n 384 --pairs 524288 > gpurun_out/r44_mw3.log 2>&1
echo done
