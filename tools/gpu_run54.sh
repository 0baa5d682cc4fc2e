# round-end refresh on the current build (exact runtime circuit everywhere): smoke, GPU suite, bench C1-C6 + default line, launch list, ncu full (C2)
set -x
mkdir -p gpurun_out
timeout 300 python -c 'import __graft_entry__ as g; g.smoke()' > gpurun_out/r54_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/r54_smoke.log
timeout 600 python bench.py > gpurun_out/r54_bench.json 2> gpurun_out/r54_bench.err
B="python bench.py --no-cpu-baseline --no-e2e --no-filter --steps 10"
for c in 1 2 3 4 5 6; do timeout 300 $B --config $c > gpurun_out/r54_c$c.json 2>/dev/null; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r54_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --no-filter > gpurun_out/r54_b_ncu.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"sw_sweep|extract" -c 2 -o gpurun_out/r54_full python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-filter > gpurun_out/r54_ncu_full.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r54_pytest_gpu.log 2>&1
echo done
