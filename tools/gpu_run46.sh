# final refresh: GPU suite, smoke, bench C1-C6 (+ full default line), launch list, ncu full (C2), C5 sweep
set -x
mkdir -p gpurun_out
timeout 300 python -c 'import __graft_entry__ as g; g.smoke()' > gpurun_out/r46_smoke.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r46_pytest_gpu.log 2>&1
timeout 600 python bench.py > gpurun_out/r46_bench.json 2> gpurun_out/r46_bench.err
B="python bench.py --no-cpu-baseline --no-e2e --no-filter --steps 10"
for c in 1 3 4 5 6; do timeout 300 $B --config $c > gpurun_out/r46_c$c.json 2>/dev/null; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r46_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --no-filter > gpurun_out/r46_b_ncu.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"sw_sweep|extract" -c 2 -o gpurun_out/r46_full python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-filter > gpurun_out/r46_ncu_full.log 2>&1
timeout 2400 python tools/c5_sweep.py --out gpurun_out/r46_c5_sweep.json > gpurun_out/r46_c5_sweep.log 2>&1
echo done
