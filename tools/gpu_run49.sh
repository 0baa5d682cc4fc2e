# ncu full of the m = n = 32 sweep (C5 row, s = 7)
set -x
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"sw_sweep" -c 1 -o gpurun_out/r49_m32 python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-filter --config 5 --m 32 --n 32 --score-bits 7 > gpurun_out/r49_m32.log 2>&1
echo done
