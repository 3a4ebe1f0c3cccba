#!/bin/bash
# sorted MOVE passes with 256 splitters per line and a 4-wide bucket scan (HALF_K = 8) vs 128 / 8-wide
mkdir -p gpurun_out
o=gpurun_out/s3h.txt; : > $o
GSAP_LIB=exp/libgsap_halfk8.so timeout 900 python -m pytest tests -m gpu -q -x -k "sorted or 200k" > gpurun_out/pytest_s3h.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_s3h.log
tail -2 gpurun_out/pytest_s3h.log >> $o
for i in 1 2; do
echo "== K=4 (default)" >> $o; timeout 600 python tools/bench_kernels.py --config 2m --rounds 4 6 --batches 8 >> $o 2>&1
echo "== K=8" >> $o; GSAP_LIB=exp/libgsap_halfk8.so timeout 600 python tools/bench_kernels.py --config 2m --rounds 4 6 --batches 8 >> $o 2>&1
done
cat $o
