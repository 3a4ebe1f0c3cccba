#!/bin/bash
# bucket sort v3 (packed slot/rank, fused RLE + output) and the pairwise merge kernel: parity + A/B
mkdir -p gpurun_out
o=gpurun_out/s2m.txt; : > $o
timeout 1200 python -m pytest tests -m gpu -q -x -k "rebuild or merge or select or lockstep or end_to_end or layer3 or partition or table" > gpurun_out/pytest_s2m.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_s2m.log
tail -2 gpurun_out/pytest_s2m.log >> $o
timeout 600 python tools/bench_kernels.py --config 2m --rounds 4 6 --batches 8 >> $o 2>&1
timeout 300 python tools/bench_kernels.py --config 20k --rounds 1 3 --batches 16 >> $o 2>&1
for i in 1 2; do
echo "== pairs" >> $o; timeout 180 python tools/partition_ab.py --config 20k --runs 8 >> $o 2>&1
echo "== block warps" >> $o; GSAP_MERGE_WARP=1 timeout 180 python tools/partition_ab.py --config 20k --runs 8 >> $o 2>&1
done
timeout 400 python tools/partition_ab.py --config 200k --runs 3 --warmup 1 >> $o 2>&1
GSAP_MERGE_WARP=1 timeout 400 python tools/partition_ab.py --config 200k --runs 3 --warmup 1 >> $o 2>&1
timeout 600 python tools/e2e_timing.py 2m 2>&1 | head -2 >> $o
cat $o
