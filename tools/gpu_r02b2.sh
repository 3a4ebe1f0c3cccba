#!/bin/bash
mkdir -p gpurun_out
timeout 900 ncu --set full --import-source on --clock-control none --profile-from-start off -k regex:"k_move" -c 4 \
  -o gpurun_out/ncu20k_r5_move -f python tools/bench_kernels.py --profile-range --config 20k --rounds 5 --batches 2 > gpurun_out/ncu_b2.log 2>&1
echo rc=$?; tail -3 gpurun_out/ncu_b2.log
ls -la gpurun_out/*.ncu-rep
