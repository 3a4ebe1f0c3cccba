#!/bin/bash
# self-loop id loads only when needed: parity subset, per-batch times, bench line, 20K partition A/B of cuda_graphs
mkdir -p gpurun_out
o=gpurun_out/s2g.txt; : > $o
timeout 1200 python -m pytest tests -m gpu -q -x -k "self_loop or weighted or hubs or lockstep or big_vertices or proposals or 200k" > gpurun_out/pytest_s2g.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_s2g.log
tail -2 gpurun_out/pytest_s2g.log >> $o
timeout 300 python tools/bench_kernels.py --config 20k --rounds 1 3 5 8 --batches 16 >> $o 2>&1
timeout 600 python tools/bench_kernels.py --config 2m --rounds 4 6 --batches 8 >> $o 2>&1
for i in 1 2; do timeout 600 python bench.py --no-2m --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads([l for l in sys.stdin if l.startswith('{')][-1]); print('bench', d['value'], d['ms_per_step'], d['e2e']['value'])" >> $o; done
timeout 600 python tools/partition_ab.py --config 20k --runs 8 --variant cuda_graphs=1 --variant cuda_graphs=2 >> $o 2>&1
GSAP_TIMING=1 timeout 300 python tools/run_once.py --config 20k > gpurun_out/timing_s2g.txt 2>&1
cat $o
