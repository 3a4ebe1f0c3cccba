#!/bin/bash
# vpos scatter A/B, coop bucket sort (20K), source-level ncu of the bucket line sort at 2M round 6
mkdir -p gpurun_out
o=gpurun_out/s2e.txt; : > $o
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "rebuild or sparse" > gpurun_out/pytest_s2e.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_s2e.log
tail -2 gpurun_out/pytest_s2e.log >> $o
echo "== vpos (default)" >> $o
timeout 600 python tools/bench_kernels.py --config 2m --rounds 4 6 --batches 8 >> $o 2>&1
echo "== scatter atomics" >> $o
GSAP_SCATTER_ATOMIC=1 timeout 600 python tools/bench_kernels.py --config 2m --rounds 4 6 --batches 8 >> $o 2>&1
echo "== 20k (coop bucket)" >> $o
timeout 300 python tools/bench_kernels.py --config 20k --rounds 1 2 3 --batches 16 >> $o 2>&1
timeout 300 python tools/bench_kernels.py --config 200k --rounds 2 5 --batches 8 >> $o 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"k_segsort_bucket|k_line_scatter" --profile-from-start off -c 3 -o gpurun_out/ncu_s2e_sort python tools/bench_kernels.py --config 2m --rounds 6 --batches 1 --profile-range > gpurun_out/ncu_s2e.log 2>&1
cat $o
