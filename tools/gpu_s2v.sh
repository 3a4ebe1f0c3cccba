#!/bin/bash
# PDL with the implicit trigger (dependents launch as the primary's CTAs exit): A/B
mkdir -p gpurun_out
o=gpurun_out/s2v.txt; : > $o
timeout 600 python -m pytest tests -m gpu -q -x -k "lockstep or incremental or end_to_end" > gpurun_out/pytest_s2v.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_s2v.log
tail -2 gpurun_out/pytest_s2v.log >> $o
for i in 1 2; do
echo "== pdl (exit trigger)" >> $o; timeout 180 python tools/partition_ab.py --config 20k --runs 8 >> $o 2>&1
echo "== no pdl" >> $o; GSAP_NO_PDL=1 timeout 180 python tools/partition_ab.py --config 20k --runs 8 >> $o 2>&1
done
cat $o
