#!/bin/bash
mkdir -p gpurun_out
o=gpurun_out/c2.txt; : > $o
timeout 900 python -m pytest tests -m gpu -q -x -k "rebuild or incremental or dense or lockstep or export or padded or mdl" > gpurun_out/pytest_c2.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_c2.log
tail -3 gpurun_out/pytest_c2.log >> $o
grep -E "^FAILED|Error" gpurun_out/pytest_c2.log | head -5 >> $o
timeout 300 python tools/bench_kernels.py --config 20k --rounds 3 4 5 6 8 --batches 16 >> $o 2>&1
timeout 300 python tools/bench_kernels.py --config 200k --rounds 5 8 --batches 8 >> $o 2>&1
for i in 1 2; do timeout 600 python bench.py --no-2m --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads([l for l in sys.stdin if l.startswith('{')][-1]); print('bench', d['value'], d['ms_per_step'], d['e2e']['value'], d['config']['mdl'], d['config']['B_found'])" >> $o; done
cat $o
