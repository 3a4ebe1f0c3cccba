#!/bin/bash
# the sparse-regime cache update deferred into the persistent rebuild's first phase: full suite + A/B
mkdir -p gpurun_out
o=gpurun_out/s3d.txt; : > $o
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_s3d.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_s3d.log
tail -2 gpurun_out/pytest_s3d.log >> $o
for i in 1 2; do
echo "== deferred" >> $o; timeout 180 python tools/partition_ab.py --config 20k --runs 8 >> $o 2>&1
echo "== separate" >> $o; GSAP_NB_NODEFER=1 timeout 180 python tools/partition_ab.py --config 20k --runs 8 >> $o 2>&1
done
timeout 400 python tools/partition_ab.py --config 200k --runs 3 --warmup 1 >> $o 2>&1
GSAP_NB_NODEFER=1 timeout 400 python tools/partition_ab.py --config 200k --runs 3 --warmup 1 >> $o 2>&1
cat $o
