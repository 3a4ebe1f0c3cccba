#!/bin/bash
# row-wise MDL data term (stored entries only): full suite + A/B
mkdir -p gpurun_out
o=gpurun_out/s3c.txt; : > $o
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_s3c.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_s3c.log
tail -2 gpurun_out/pytest_s3c.log >> $o
for i in 1 2; do
echo "== rows" >> $o; timeout 180 python tools/partition_ab.py --config 20k --runs 8 >> $o 2>&1
echo "== chunks (previous commit)" >> $o; GSAP_LIB=exp/libgsap_prev.so timeout 180 python tools/partition_ab.py --config 20k --runs 8 >> $o 2>&1
done
timeout 400 python tools/partition_ab.py --config 200k --runs 3 --warmup 1 >> $o 2>&1
GSAP_LIB=exp/libgsap_prev.so timeout 400 python tools/partition_ab.py --config 200k --runs 3 --warmup 1 >> $o 2>&1
timeout 600 python tools/e2e_timing.py 2m 2>&1 | head -2 >> $o
cat $o
