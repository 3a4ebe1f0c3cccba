#!/bin/bash
# parallel per-batch dS trees in the MDL kernel + bench e2e warm-up: full suite, A/B, bench lines
mkdir -p gpurun_out
o=gpurun_out/s2z.txt; : > $o
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_s2z.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_s2z.log
tail -2 gpurun_out/pytest_s2z.log >> $o
for i in 1 2; do timeout 180 python tools/partition_ab.py --config 20k --runs 8 >> $o 2>&1; done
for i in 1 2; do timeout 600 python bench.py --no-2m --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads([l for l in sys.stdin if l.startswith('{')][-1]); print('bench', d['value'], d['ms_per_step'], d['e2e']['value'], d['e2e']['partition_sec'])" >> $o; done
cat $o
