#!/bin/bash
# full GPU suite + smoke + bench line (nb cache, exec update, device-loop default)
mkdir -p gpurun_out
o=gpurun_out/s2i.txt; : > $o
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_s2i.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_s2i.log
tail -2 gpurun_out/pytest_s2i.log >> $o
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" >> $o 2>&1
for i in 1 2; do timeout 600 python bench.py --no-2m --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads([l for l in sys.stdin if l.startswith('{')][-1]); print('bench', d['value'], d['ms_per_step'], d['e2e']['value'], d['roofline']['frac'])" >> $o; done
timeout 600 python tools/e2e_timing.py 2m 2>&1 | head -2 >> $o
timeout 300 python tools/e2e_timing.py 200k 2>&1 | head -3 >> $o
cat $o
