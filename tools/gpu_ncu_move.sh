#!/bin/bash
# ncu launch list of the bench command and a full capture of the move kernels
# at the 2M round-6 state (current library).
set -x
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
  python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/bench_ncu.log 2>&1
python tools/launch_summary.py gpurun_out/launches.csv 60 > gpurun_out/launches.txt
timeout 1200 ncu --set full --import-source on --clock-control none --profile-from-start off \
  -k regex:"k_move" -c 2 -o gpurun_out/ncu_2m_r6_move -f python tools/bench_kernels.py --profile-range --config 2m --rounds 6 --batches 1 > gpurun_out/ncu_2m_r6_move.log 2>&1
python tools/ncu_summary.py gpurun_out/ncu_2m_r6_move.ncu-rep 30 > gpurun_out/ncu_2m_r6_move.txt 2>&1
rm -f gpurun_out/ncu_2m_r6_move.ncu-rep
head -60 gpurun_out/ncu_2m_r6_move.txt
