#!/bin/bash
# DRAM bytes of the bench's roofline kernel (k_move at the late 20K-HH state, B ~ 30) with the final library
mkdir -p gpurun_out
tools/clocked.sh ncu20k_late timeout 900 ncu --set full --clock-control none --profile-from-start off \
  -k regex:"k_move" -c 4 -o /tmp/ncu20k_late -f python tools/bench_kernels.py --profile-range --config 20k --rounds 15 --batches 2 > gpurun_out/ncu20k_late.log 2>&1
python tools/ncu_summary.py /tmp/ncu20k_late.ncu-rep 20 > gpurun_out/ncu20k_late.txt 2>&1
grep -E "^== launch|Duration|dram__bytes" gpurun_out/ncu20k_late.txt
