set -x
mkdir -p gpurun_out
B="python bench.py --no-cpu-baseline --no-e2e --no-filter --steps 10"
timeout 300 $B > gpurun_out/x_c2_lb4.json 2>/dev/null
BPBC_SW_LIB=$PWD/tools/exp/libbpbc_sw_lb5.so timeout 300 $B > gpurun_out/x_c2_lb5.json 2>gpurun_out/x_c2_lb5.err
timeout 300 $B > gpurun_out/x_c2_lb4b.json 2>/dev/null
echo done
