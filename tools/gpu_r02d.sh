#!/bin/bash
# Staged two-pass MOVE + warp radix line sort: parity, then 2M per-kernel list and per-batch timings.
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x -k "rebuild or sorted or lockstep or hubs or 200k_fused or end_to_end" > gpurun_out/pytest_d.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_d.log
tail -3 gpurun_out/pytest_d.log
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_bytes.sum --clock-control none \
    --profile-from-start off --csv --log-file gpurun_out/l2m_r6_d.csv \
    python tools/bench_kernels.py --profile-range --config 2m --rounds 6 --batches 2 > gpurun_out/l2m_r6_d.log 2>&1
python tools/launch_metrics.py gpurun_out/l2m_r6_d.csv 30 > gpurun_out/l2m_r6_d.txt 2>&1
timeout 900 python tools/bench_kernels.py --config 2m --rounds 1 3 4 6 --batches 8 > gpurun_out/bk2m_d.txt 2>&1
cat gpurun_out/l2m_r6_d.txt gpurun_out/bk2m_d.txt
