# final build: initcheck over every kernel family (harness fixed to copy only the written filter indices); ncu full of the paper shape (config 6) sweep for the NEXT-3 analysis
set -x
mkdir -p gpurun_out
timeout 900 compute-sanitizer --tool initcheck python tests/sanitize_run.py > gpurun_out/r56_initcheck.log 2>&1
timeout 900 ncu --set full --clock-control none -k regex:"sw_sweep" -c 1 -o gpurun_out/r56_c6_full python bench.py --config 6 --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-filter > gpurun_out/r56_c6_ncu.log 2>&1
echo done
