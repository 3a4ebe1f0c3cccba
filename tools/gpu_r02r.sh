#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -rA -k "full_run_lockstep or padded_blockmodel or bench_tsv" > gpurun_out/pytest_r.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_r.log
grep -E "rounds|passed|failed|Error|assert" gpurun_out/pytest_r.log | head -20
