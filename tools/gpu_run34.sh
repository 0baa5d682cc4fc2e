# fused kernel for n % 32 == 0 (m = n = 32): full GPU suite on that build + C5 m=32/64 points, both builds
set -x
mkdir -p gpurun_out
BPBC_SW_LIB=exp_libs/f32.so timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r34_pytest_gpu.log 2>&1
for t in f32 main; do
  L=exp_libs/$t.so; [ $t = main ] && L=paper_conf_ipps_nishimurabin17_b200/libbpbc_sw.so
  BPBC_SW_LIB=$L timeout 600 python tools/c5_sweep.py --m 32,64 --s 6,7,8 --out gpurun_out/r34_c5_$t.json > gpurun_out/r34_c5_$t.log 2>&1
done
echo done
