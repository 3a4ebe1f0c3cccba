#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x -k "hubs or big_vertices or lockstep or isolated or launch_shape or move_proposals or 200k_sampled or device_outputs" > gpurun_out/pytest_l.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_l.log
tail -2 gpurun_out/pytest_l.log
timeout 600 python tools/bench_kernels.py --config 20k --rounds 1 3 5 8 --batches 16 > gpurun_out/bk20k_l.txt 2>&1
timeout 600 python tools/bench_kernels.py --config 2m --rounds 3 6 --batches 8 > gpurun_out/bk2m_l.txt 2>&1
GSAP_TIMING=1 timeout 300 python tools/e2e_timing.py 20k > gpurun_out/e2e_l.txt 2>&1
cat gpurun_out/bk20k_l.txt gpurun_out/bk2m_l.txt; grep -E "e2e|create" gpurun_out/e2e_l.txt | tail -12
