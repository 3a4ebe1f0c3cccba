#!/bin/bash
# cache update beside the dense rebuild (side stream): full GPU suite, partition A/B
mkdir -p gpurun_out
o=gpurun_out/s2p.txt; : > $o
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_s2p.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_s2p.log
tail -2 gpurun_out/pytest_s2p.log >> $o
for i in 1 2; do
echo "== side" >> $o; timeout 180 python tools/partition_ab.py --config 20k --runs 8 >> $o 2>&1
echo "== in order" >> $o; GSAP_NB_INORDER=1 timeout 180 python tools/partition_ab.py --config 20k --runs 8 >> $o 2>&1
done
timeout 400 python tools/partition_ab.py --config 200k --runs 3 --warmup 1 >> $o 2>&1
GSAP_NB_INORDER=1 timeout 400 python tools/partition_ab.py --config 200k --runs 3 --warmup 1 >> $o 2>&1
cat $o
for em in 8 4; do
  echo "== dense E multiplier $em" >> $o
  GSAP_DENSE_EMULT=$em timeout 400 python tools/partition_ab.py --config 200k --runs 3 --warmup 1 >> $o 2>&1
  GSAP_DENSE_EMULT=$em timeout 600 python tools/e2e_timing.py 2m 2>&1 | head -2 >> $o
  GSAP_DENSE_EMULT=$em timeout 300 python tools/partition_ab.py --config 1k --runs 20 >> $o 2>&1
done
cat $o
