#!/bin/bash
mkdir -p gpurun_out
o=gpurun_out/d2.txt; : > $o
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_d2.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_d2.log
tail -3 gpurun_out/pytest_d2.log >> $o
grep -E "^FAILED|Error" gpurun_out/pytest_d2.log | head -5 >> $o
timeout 300 python tools/bench_kernels.py --config 20k --rounds 4 5 6 8 12 --batches 16 >> $o 2>&1
for i in 1 2; do timeout 600 python bench.py --no-2m --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads([l for l in sys.stdin if l.startswith('{')][-1]); print('bench', d['value'], d['ms_per_step'], d['e2e']['value'], d['config']['mdl'], d['config']['B_found'])" >> $o; done
timeout 900 python tools/ablation_n2.py 200k > gpurun_out/n2_200k.txt 2>&1; tail -3 gpurun_out/n2_200k.txt >> $o
cat $o
