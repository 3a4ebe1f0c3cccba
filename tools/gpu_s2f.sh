#!/bin/bash
# neighbour-block cache: full GPU suite, per-batch times (20K / 200K / 2M), bench line, 2M partition
mkdir -p gpurun_out
o=gpurun_out/s2f.txt; : > $o
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_s2f.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_s2f.log
tail -2 gpurun_out/pytest_s2f.log >> $o
timeout 300 python tools/bench_kernels.py --config 20k --rounds 1 3 5 8 --batches 16 >> $o 2>&1
timeout 300 python tools/bench_kernels.py --config 200k --rounds 2 5 --batches 8 >> $o 2>&1
timeout 600 python tools/bench_kernels.py --config 2m --rounds 4 6 --batches 8 >> $o 2>&1
for i in 1 2; do timeout 600 python bench.py --no-2m --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads([l for l in sys.stdin if l.startswith('{')][-1]); print('bench', d['value'], d['ms_per_step'], d['e2e']['value'])" >> $o; done
timeout 600 python tools/e2e_timing.py 2m 2>&1 | head -2 >> $o
cat $o
