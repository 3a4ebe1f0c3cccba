#!/bin/bash
# sorted MOVE passes: bucket scan width from the lines' largest bucket (2 / 4 / 8) vs always 8
mkdir -p gpurun_out
o=gpurun_out/s3j.txt; : > $o
GSAP_LIB=exp/libgsap_adapt.so timeout 900 python -m pytest tests -m gpu -q -x -k "sorted or 200k or lockstep" > gpurun_out/pytest_s3j.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_s3j.log
tail -2 gpurun_out/pytest_s3j.log >> $o
for i in 1 2; do
echo "== always 8" >> $o; timeout 600 python tools/bench_kernels.py --config 2m --rounds 4 6 --batches 8 >> $o 2>&1
echo "== adaptive" >> $o; GSAP_LIB=exp/libgsap_adapt.so timeout 600 python tools/bench_kernels.py --config 2m --rounds 4 6 --batches 8 >> $o 2>&1
done
cat $o
