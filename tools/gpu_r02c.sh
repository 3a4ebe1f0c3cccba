#!/bin/bash
# Per-kernel durations + DRAM bytes of one 2M MOVE batch + rebuild (ncu, serialised launches), both MOVE modes.
mkdir -p gpurun_out
for ms in 0 1; do
  timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_bytes.sum --clock-control none \
    --profile-from-start off --csv --log-file gpurun_out/l2m_r6_s$ms.csv \
    python tools/bench_kernels.py --profile-range --config 2m --rounds 6 --batches 2 --param move_sorted=$ms > gpurun_out/l2m_r6_s$ms.log 2>&1
  python tools/launch_metrics.py gpurun_out/l2m_r6_s$ms.csv 30 > gpurun_out/l2m_r6_s$ms.txt 2>&1
done
cat gpurun_out/l2m_r6_s*.txt
