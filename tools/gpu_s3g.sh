#!/bin/bash
# the round's final library: full GPU suite + smoke (what the driver runs at round end)
mkdir -p gpurun_out
o=gpurun_out/s3g.txt; : > $o
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_s3g.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_s3g.log
tail -2 gpurun_out/pytest_s3g.log >> $o
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" >> $o 2>&1
cat $o
