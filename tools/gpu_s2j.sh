#!/bin/bash
# group role at high launch priority: A/B on 20K partitions and 2M batches
mkdir -p gpurun_out
o=gpurun_out/s2j.txt; : > $o
timeout 600 python -m pytest tests -m gpu -q -x -k "lockstep or hubs or big_vertices" > gpurun_out/pytest_s2j.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_s2j.log
tail -2 gpurun_out/pytest_s2j.log >> $o
for i in 1 2; do
echo "== prio" >> $o; timeout 180 python tools/partition_ab.py --config 20k --runs 8 >> $o 2>&1
echo "== no prio" >> $o; GSAP_NO_PRIO=1 timeout 180 python tools/partition_ab.py --config 20k --runs 8 >> $o 2>&1
done
timeout 300 python tools/bench_kernels.py --config 20k --rounds 3 5 --batches 16 >> $o 2>&1
GSAP_NO_PRIO=1 timeout 300 python tools/bench_kernels.py --config 20k --rounds 3 5 --batches 16 >> $o 2>&1
timeout 600 python tools/bench_kernels.py --config 2m --rounds 6 --batches 8 >> $o 2>&1
GSAP_NO_PRIO=1 timeout 600 python tools/bench_kernels.py --config 2m --rounds 6 --batches 8 >> $o 2>&1
cat $o
