set -x
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1
B="python bench.py --no-cpu-baseline --no-e2e --no-filter --steps 10"
for c in 2 3 4 5 6; do timeout 300 $B --config $c > gpurun_out/bench_c$c.json 2>/dev/null; done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"sw_sweep" -c 1 -o gpurun_out/r17_full python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-filter > gpurun_out/ncu_full.log 2>&1
echo done
