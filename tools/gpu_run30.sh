# predicated group switch as the default (R <= 4): full GPU suite, C2/C3 bench, ncu full of C2
set -x
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r30_pytest_gpu.log 2>&1
B="python bench.py --no-cpu-baseline --no-e2e --no-filter --steps 10"
for c in 2 3; do timeout 300 $B --config $c > gpurun_out/r30_c$c.json 2>/dev/null; done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"sw_sweep" -c 1 -o gpurun_out/r30_full python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-filter > gpurun_out/r30_ncu_full.log 2>&1
echo done
