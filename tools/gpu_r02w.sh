#!/bin/bash
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_w.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_w.log
tail -3 gpurun_out/pytest_w.log
timeout 600 python tools/bench_kernels.py --config 2m --rounds 4 6 --batches 8 > gpurun_out/bk2m_w.txt 2>&1
cat gpurun_out/bk2m_w.txt
