set -x
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 300 python bench.py --no-cpu-baseline --no-e2e --steps 5 --config 4 > gpurun_out/bench_c4.json 2> gpurun_out/bench_c4.err
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"wordwise_kernel|striped" -c 2 -o gpurun_out/r12_full python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --config 5 --pairs 262144 > gpurun_out/ncu_full.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"wordwise_kernel" -c 1 -o gpurun_out/r12_ww python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_ww.log 2>&1
echo done
