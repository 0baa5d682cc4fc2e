set -x
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1
timeout 300 python tools/sanitize_run.py > gpurun_out/sanitize_plain.log 2>&1
timeout 1500 compute-sanitizer --tool racecheck python tools/sanitize_run.py > gpurun_out/sanitize_racecheck.log 2>&1
timeout 1500 compute-sanitizer --tool memcheck python tools/sanitize_run.py > gpurun_out/sanitize_memcheck.log 2>&1
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench.json 2> gpurun_out/bench.err
B="python bench.py --no-cpu-baseline --no-e2e --no-filter --steps 5"
for c in 1 3 4 6; do timeout 300 $B --config $c > gpurun_out/bench_c$c.json 2>/dev/null; done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"sw_sweep" -c 1 -o gpurun_out/r16_full python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-filter > gpurun_out/ncu_full.log 2>&1
echo done
