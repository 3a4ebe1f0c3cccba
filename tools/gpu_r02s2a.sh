#!/bin/bash
mkdir -p gpurun_out
o=gpurun_out/s2a.txt; : > $o
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_s2a.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_s2a.log
tail -2 gpurun_out/pytest_s2a.log >> $o
timeout 300 python tools/bench_kernels.py --config 20k --rounds 1 5 8 --batches 16 >> $o 2>&1
for i in 1 2; do timeout 600 python bench.py --no-2m --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads([l for l in sys.stdin if l.startswith('{')][-1]); print('bench', d['value'], d['ms_per_step'], d['e2e']['value'])" >> $o; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv --log-file gpurun_out/launches_s2a.csv python bench.py --steps 1 --warmup 1 --no-2m --no-cpu-baseline > /dev/null 2>&1
python tools/launch_metrics.py gpurun_out/launches_s2a.csv 20 > gpurun_out/launches_s2a.txt 2>&1
cat $o; head -24 gpurun_out/launches_s2a.txt
