#!/bin/bash
# Round-end check of the product library: GPU tests, smoke, bench line,
# unprofiled partitions at 200K / 1M / 2M, per-batch kernel times at 2M.
set -x
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
for c in 200k 1m 2m; do timeout 900 python tools/run_once.py --config $c --runs 1 > gpurun_out/e2e_$c.log 2>&1; done
timeout 900 python tools/bench_kernels.py --config 2m --rounds 3 4 6 --batches 2 > gpurun_out/bk2m.txt 2>&1
tail -n 2 gpurun_out/pytest_gpu.log gpurun_out/smoke.log; grep -h "^run" gpurun_out/e2e_*.log; grep "R=" gpurun_out/bk2m.txt; cut -c1-200 gpurun_out/bench.json
