# N = 2 code path on one GPU (shared, gloo) for both arms after the bench.py changes
set -x
mkdir -p gpurun_out
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29561 bench.py --gpus 2 --steps 3 --warmup 3 > gpurun_out/r47_n2.json 2> gpurun_out/r47_n2.err
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29562 bench.py --impl reference --gpus 2 --steps 2 --warmup 1 > gpurun_out/r47_ref_n2.json 2> gpurun_out/r47_ref_n2.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/r47_ref_n1.json 2> gpurun_out/r47_ref_n1.err
echo done
