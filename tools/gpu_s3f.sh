#!/bin/bash
# arena cache keeps the newest arena: e2e after the 2M states, plus the API tests, then the final bench line
mkdir -p gpurun_out
o=gpurun_out/s3f.txt; : > $o
timeout 900 python -m pytest tests -m gpu -q -x -k "partition or device_outputs or end_to_end or abi" > gpurun_out/pytest_s3f.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_s3f.log
tail -2 gpurun_out/pytest_s3f.log >> $o
tools/clocked.sh bench_final3 timeout 1500 python bench.py > gpurun_out/bench_final3.json 2> gpurun_out/bench_final3.err
python -c "import json; d=json.loads([l for l in open('gpurun_out/bench_final3.json') if l.startswith('{')][-1]); print('bench', d['value'], d['ms_per_step'], 'e2e', d['e2e']['value'], d['e2e']['partition_sec'], 'rb2m', [s['rebuild']['frac'] for s in d['roofline_2m']['states']])" >> $o
cat $o
