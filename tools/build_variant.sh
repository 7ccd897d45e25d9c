#!/bin/bash
# usage: tools/build_variant.sh <name> <dir-with-override-files>
# Builds tools/exp_libs/lib<name>.so from csrc/ with the files in <dir> substituted.
set -e
name=$1; ov=$2
d=/tmp/var_$name/a/b; rm -rf /tmp/var_$name; mkdir -p $d /tmp/var_$name/include; cp include/gs.h /tmp/var_$name/include/
cp paper_conf_sosp_gonglmc0lwl23_b200/csrc/*.cu paper_conf_sosp_gonglmc0lwl23_b200/csrc/*.cuh paper_conf_sosp_gonglmc0lwl23_b200/csrc/*.h $d/
cp $ov/* $d/
objs=""
for f in capi nodewise_wave shadow layerwise layerwise_bm walk pack pinsage ops pass_att; do
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -fmad=false -std=c++17 -Xcompiler -fPIC -I include -c $d/$f.cu -o $d/$f.o &
  objs="$objs $d/$f.o"
done
wait
mkdir -p tools/exp_libs
nvcc -shared -gencode arch=compute_100a,code=sm_100a -o tools/exp_libs/lib$name.so $objs -lcublas -Xlinker -rpath=/usr/local/cuda/lib64
echo built tools/exp_libs/lib$name.so
