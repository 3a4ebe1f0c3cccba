#!/bin/bash
# dense-regime capacity floor: 2^24 (default) vs 2^25 / 2^26 at 20K and 200K
mkdir -p gpurun_out
o=gpurun_out/s2n.txt; : > $o
for fl in 24 25 26; do
  echo "== floor 2^$fl" >> $o
  GSAP_DENSE_FLOOR_LOG2=$fl timeout 180 python tools/partition_ab.py --config 20k --runs 8 >> $o 2>&1
  GSAP_DENSE_FLOOR_LOG2=$fl timeout 300 python tools/bench_kernels.py --config 20k --rounds 1 2 3 --batches 16 >> $o 2>&1
  GSAP_DENSE_FLOOR_LOG2=$fl timeout 400 python tools/partition_ab.py --config 200k --runs 3 --warmup 1 >> $o 2>&1
done
GSAP_DENSE_FLOOR_LOG2=26 timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "rebuild_20k or incremental or lockstep" > gpurun_out/pytest_s2n.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_s2n.log
tail -2 gpurun_out/pytest_s2n.log >> $o
cat $o
