#!/bin/bash
# graph exec update across rounds: modes 1 / 2 with and without the update, then the graph tests
mkdir -p gpurun_out
o=gpurun_out/s2h.txt; : > $o
timeout 180 python tools/partition_ab.py --config 20k --runs 8 --variant cuda_graphs=1 --variant cuda_graphs=2 >> $o 2>&1; echo "rc=$?" >> $o
GSAP_NO_EXEC_UPDATE=1 timeout 180 python tools/partition_ab.py --config 20k --runs 8 --variant cuda_graphs=1 --variant cuda_graphs=2 >> $o 2>&1
timeout 600 python -m pytest tests -m gpu -q -x -k "graph or lockstep or end_to_end or layer3 or partition" > gpurun_out/pytest_s2h.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_s2h.log
tail -2 gpurun_out/pytest_s2h.log >> $o
GSAP_TIMING=1 timeout 120 python tools/run_once.py --config 20k --runs 2 > gpurun_out/timing_s2h.txt 2>&1
cat $o
