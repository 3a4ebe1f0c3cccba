#!/bin/bash
# insertion pass with the running maximum + shuffled head test: parity + A/B at 2M / 20K
mkdir -p gpurun_out
o=gpurun_out/s2t.txt; : > $o
timeout 1200 python -m pytest tests -m gpu -q -x -k "rebuild or sparse_mk or 200k or lockstep or incremental or dense" > gpurun_out/pytest_s2t.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_s2t.log
tail -2 gpurun_out/pytest_s2t.log >> $o
timeout 600 python tools/bench_kernels.py --config 2m --rounds 4 6 --batches 8 >> $o 2>&1
timeout 300 python tools/bench_kernels.py --config 20k --rounds 1 3 4 5 7 --batches 16 >> $o 2>&1
for i in 1 2; do timeout 180 python tools/partition_ab.py --config 20k --runs 8 >> $o 2>&1; done
GSAP_TIMING=1 timeout 900 python tools/run_once.py --config 2m > gpurun_out/timing_2m_s2t.txt 2>&1
grep -E "^run|outer=" gpurun_out/timing_2m_s2t.txt | head -40 >> $o
cat $o
