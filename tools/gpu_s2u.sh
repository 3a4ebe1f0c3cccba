#!/bin/bash
# programmatic dependent launch in the batch chain: full GPU suite + A/B
mkdir -p gpurun_out
o=gpurun_out/s2u.txt; : > $o
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_s2u.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_s2u.log
tail -2 gpurun_out/pytest_s2u.log >> $o
for i in 1 2; do
echo "== pdl" >> $o; timeout 180 python tools/partition_ab.py --config 20k --runs 8 >> $o 2>&1
echo "== no pdl" >> $o; GSAP_NO_PDL=1 timeout 180 python tools/partition_ab.py --config 20k --runs 8 >> $o 2>&1
done
timeout 400 python tools/partition_ab.py --config 200k --runs 3 --warmup 1 >> $o 2>&1
GSAP_NO_PDL=1 timeout 400 python tools/partition_ab.py --config 200k --runs 3 --warmup 1 >> $o 2>&1
for i in 1 2; do timeout 600 python bench.py --no-2m --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads([l for l in sys.stdin if l.startswith('{')][-1]); print('bench', d['value'], d['ms_per_step'], d['e2e']['value'])" >> $o; done
cat $o
