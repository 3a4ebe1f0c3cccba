#!/bin/bash
# Build an experimental libgsap variant with extra nvcc flags: tools/build_variant.sh NAME FLAGS...
# (loaded with GSAP_LIB=exp/libgsap_NAME.so; the product library is paper_conf_icpp_changzh24_b200/libgsap.so)
set -e
name=$1; shift
out=exp/$name; mkdir -p $out
for f in api rebuild move merge mdl comm; do
  /usr/local/cuda/bin/nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -lineinfo -Xcompiler -fPIC "$@" \
    -c -o $out/$f.o ${SRC:-paper_conf_icpp_changzh24_b200/csrc}/$f.cu &
done
wait
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -shared -cudart static -ldl -o exp/libgsap_$name.so $out/*.o
rm -rf $out
