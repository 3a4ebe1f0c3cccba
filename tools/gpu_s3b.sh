#!/bin/bash
# mid-vertex groups of 128 threads (two per CTA) instead of 64: parity with the variant + A/B
mkdir -p gpurun_out
o=gpurun_out/s3b.txt; : > $o
GSAP_LIB=exp/libgsap_mid128.so timeout 900 python -m pytest tests -m gpu -q -x -k "hubs or big_vertices or lockstep or weighted or launch_shape or 200k" > gpurun_out/pytest_s3b.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_s3b.log
tail -2 gpurun_out/pytest_s3b.log >> $o
for i in 1 2; do
echo "== mid 64" >> $o; timeout 180 python tools/partition_ab.py --config 20k --runs 8 >> $o 2>&1
echo "== mid 128" >> $o; GSAP_LIB=exp/libgsap_mid128.so timeout 180 python tools/partition_ab.py --config 20k --runs 8 >> $o 2>&1
done
timeout 300 python tools/bench_kernels.py --config 20k --rounds 3 5 --batches 16 >> $o 2>&1
GSAP_LIB=exp/libgsap_mid128.so timeout 300 python tools/bench_kernels.py --config 20k --rounds 3 5 --batches 16 >> $o 2>&1
timeout 600 python tools/bench_kernels.py --config 2m --rounds 6 --batches 8 >> $o 2>&1
GSAP_LIB=exp/libgsap_mid128.so timeout 600 python tools/bench_kernels.py --config 2m --rounds 6 --batches 8 >> $o 2>&1
cat $o
