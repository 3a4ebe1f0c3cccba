#!/bin/bash
# Full GPU suite + smoke + a short bench + timing sanity of the current library.
mkdir -p gpurun_out
timeout 3000 python -m pytest tests -m gpu -q -rf --durations=15 > gpurun_out/pytest_full.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_full.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_full.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke_full.log
timeout 600 python tools/bench_kernels.py --config 20k --rounds 1 3 5 8 --batches 16 > gpurun_out/bk20k_full.txt 2>&1
timeout 600 python tools/bench_kernels.py --config 2m --rounds 3 6 --batches 8 > gpurun_out/bk2m_full.txt 2>&1
timeout 900 python bench.py --no-2m --no-cpu-baseline > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err
tail -25 gpurun_out/pytest_full.log; tail -2 gpurun_out/smoke_full.log; cat gpurun_out/bk20k_full.txt gpurun_out/bk2m_full.txt; cat gpurun_out/bench_full.json
