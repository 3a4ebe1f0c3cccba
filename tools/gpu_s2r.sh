#!/bin/bash
# multi-kernel sparse rebuild with the row and column sides concurrent: parity + A/B at 2M
mkdir -p gpurun_out
o=gpurun_out/s2r.txt; : > $o
timeout 1200 python -m pytest tests -m gpu -q -x -k "rebuild or sparse_mk or 200k or lockstep or weighted" > gpurun_out/pytest_s2r.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_s2r.log
tail -2 gpurun_out/pytest_s2r.log >> $o
echo "== concurrent sides" >> $o
timeout 600 python tools/bench_kernels.py --config 2m --rounds 4 6 --batches 8 >> $o 2>&1
echo "== serial sides" >> $o
GSAP_SIDES_SERIAL=1 timeout 600 python tools/bench_kernels.py --config 2m --rounds 4 6 --batches 8 >> $o 2>&1
timeout 600 python tools/e2e_timing.py 2m 2>&1 | head -2 >> $o
GSAP_SIDES_SERIAL=1 timeout 600 python tools/e2e_timing.py 2m 2>&1 | head -2 >> $o
cat $o
