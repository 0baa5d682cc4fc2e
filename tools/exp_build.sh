#!/bin/bash
# A/B experiment build: libbpbc_sw.so with extra nvcc flags into build/exp_<tag>/
# (widths 8-11, running-max mode only) as exp_libs/<tag>.so (travels with gpurun; load it
# with BPBC_SW_LIB=exp_libs/<tag>.so).
# usage: tools/exp_build.sh <tag> "<extra nvcc flags>"
set -e
tag=$1; extra=$2
root=$(cd "$(dirname "$0")/.." && pwd)
b=$root/build/exp_$tag
mkdir -p $b $root/exp_libs
# widths 8-11 (running max) rebuilt with the flags; everything else from the main build
objs=""
for w in 4 5 6 7 8 9 10 11 12 13 14 15 16; do
  case $w in 8|9|10|11) objs="$objs $b/sweep_s${w}_m0.o";; *) objs="$objs $root/build/csrc/sweep_s${w}_m0.o";; esac
  objs="$objs $root/build/csrc/sweep_s${w}_m1.o"
done
rm -f $root/exp_libs/$tag.so
make -s -C $root/paper_conf_ipps_nishimurabin17_b200/csrc -j16 BUILD=$b OUT=$root/exp_libs/$tag.so \
  WIDTHS="8 9 10 11" "SWEEP_OBJS=$objs" \
  "NVFLAGS=-gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -I$root/include -Xptxas -v $extra"
python -c "import ctypes; ctypes.CDLL('$root/exp_libs/$tag.so')"
echo built $root/exp_libs/$tag.so
