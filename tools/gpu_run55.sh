# final build: both bench arms at N=2 (two ranks sharing the one GPU), reference arm at N=1, sanitizers
set -x
mkdir -p gpurun_out
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29517 bench.py --gpus 2 --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/r55_n2.json 2> gpurun_out/r55_n2.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/r55_ref.json 2> gpurun_out/r55_ref.err
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29518 bench.py --impl reference --gpus 2 --steps 3 --warmup 3 > gpurun_out/r55_ref_n2.json 2> gpurun_out/r55_ref_n2.err
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool python tests/sanitize_run.py > gpurun_out/r55_$tool.log 2>&1
done
echo done
