#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x -k "sorted or 200k_fused or sim_ranks or hubs or launch_shape" > gpurun_out/pytest_q.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_q.log
tail -2 gpurun_out/pytest_q.log
timeout 600 python tools/bench_kernels.py --config 2m --rounds 3 4 6 --batches 8 > gpurun_out/bk2m_q.txt 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
    --profile-from-start off --csv --log-file gpurun_out/l2m_q.csv \
    python tools/bench_kernels.py --profile-range --config 2m --rounds 6 --batches 1 > /dev/null 2>&1
python tools/launch_metrics.py gpurun_out/l2m_q.csv 10 > gpurun_out/l2m_q.txt 2>&1
cat gpurun_out/bk2m_q.txt gpurun_out/l2m_q.txt
