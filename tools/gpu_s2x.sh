#!/bin/bash
# the iteration's dS sum deferred to the MDL kernel (no last-CTA pass per apply): full suite + A/B
mkdir -p gpurun_out
o=gpurun_out/s2x.txt; : > $o
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_s2x.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_s2x.log
tail -2 gpurun_out/pytest_s2x.log >> $o
for i in 1 2 3; do timeout 180 python tools/partition_ab.py --config 20k --runs 8 >> $o 2>&1; done
GSAP_LIB=exp/libgsap_base.so timeout 180 python tools/partition_ab.py --config 20k --runs 8 >> $o 2>&1
GSAP_LIB=exp/libgsap_base.so timeout 180 python tools/partition_ab.py --config 20k --runs 8 >> $o 2>&1
timeout 400 python tools/partition_ab.py --config 200k --runs 3 --warmup 1 >> $o 2>&1
cat $o
