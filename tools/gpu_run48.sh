# resident blocks per SM at C2: 4 (default) vs 3 vs 2 (BPBC_MAX_BLOCKS_PER_SM)
set -x
mkdir -p gpurun_out
B="python bench.py --no-cpu-baseline --no-e2e --no-filter --steps 10"
for b in 4 3 2; do BPBC_MAX_BLOCKS_PER_SM=$b timeout 300 $B --config 2 > gpurun_out/r48_b$b.json 2>/dev/null; done
echo done
