set -x
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench.json 2> gpurun_out/bench.err
for c in 3 4 6; do timeout 600 python bench.py --config $c --no-cpu-baseline --no-e2e --steps 5 > gpurun_out/bench_c$c.json 2> gpurun_out/bench_c$c.err; done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"sw_sweep" -c 1 -o gpurun_out/r7_full python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_full.log 2>&1
echo done
