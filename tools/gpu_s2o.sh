#!/bin/bash
# bucket sort v3 parts A/B (fused RLE, packed slot/rank), then the dense capacity floor
mkdir -p gpurun_out
o=gpurun_out/s2o.txt; : > $o
for lib in paper_conf_icpp_changzh24_b200/libgsap.so exp/libgsap_rle0.so exp/libgsap_pack0.so exp/libgsap_v2.so; do
  echo "== $lib" >> $o
  GSAP_LIB=$lib timeout 600 python tools/bench_kernels.py --config 2m --rounds 4 6 --batches 8 >> $o 2>&1
  GSAP_LIB=$lib timeout 300 python tools/bench_kernels.py --config 20k --rounds 1 3 --batches 16 >> $o 2>&1
done
bash tools/gpu_s2n.sh >> $o 2>&1
cat $o
