#!/bin/bash
mkdir -p gpurun_out
o=gpurun_out/a2.txt; : > $o
GSAP_TIMING=1 timeout 300 python tools/bench_kernels.py --config 20k --rounds 1 3 5 8 --batches 16 2>&1 | grep -E "roles|R=" >> $o
GSAP_TIMING=1 timeout 300 python tools/bench_kernels.py --config 200k --rounds 2 5 --batches 8 2>&1 | grep -E "roles|R=" >> $o
GSAP_TIMING=1 timeout 600 python tools/bench_kernels.py --config 2m --rounds 6 --batches 8 2>&1 | grep -E "roles|R=" >> $o
cat $o
