#!/bin/bash
# Sorted two-pass MOVE: parity of the new paths, then 2M per-batch timings both ways.
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x -k "sorted or lockstep or mcmc_phase_D or driver or end_to_end or layer3 or 1m_2m or device_outputs or evaluated or 200k_fused" > gpurun_out/pytest_b.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_b.log
for ms in 0 1; do
  timeout 900 python tools/bench_kernels.py --config 2m --rounds 1 3 4 6 --batches 8 --param move_sorted=$ms > gpurun_out/bk2m_sorted$ms.txt 2>&1
done
timeout 600 python tools/bench_kernels.py --config 200k --rounds 1 3 5 --batches 8 --param move_sorted=0 > gpurun_out/bk200k_sorted0.txt 2>&1
timeout 600 python tools/bench_kernels.py --config 200k --rounds 1 3 5 --batches 8 --param move_sorted=2 > gpurun_out/bk200k_sorted2.txt 2>&1
tail -3 gpurun_out/pytest_b.log; cat gpurun_out/bk2m_sorted*.txt gpurun_out/bk200k_sorted*.txt
