#!/bin/bash
# Scale pass: end-to-end runs at 200K / 1M / 2M with per-round traces, per-kernel
# timings on 2M states, and ncu --set full captures of the hot kernels.
set -x
mkdir -p gpurun_out
for c in 200k 1m 2m; do
  timeout 1500 python tools/run_once.py --config $c --profile 1 > gpurun_out/run_$c.log 2>&1
done
timeout 900 python tools/bench_kernels.py --config 2m --rounds 1 4 10 19 --batches 8 --json gpurun_out/bk2m.json > gpurun_out/bk2m.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none --profile-from-start off \
  -k regex:"k_move|k_rebuild|k_row|k_hist|k_transpose|k_apply" -c 14 -o gpurun_out/ncu20k_late -f \
  python tools/bench_kernels.py --config 20k --rounds 19 --batches 2 --profile-range > gpurun_out/ncu20k_late.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none --profile-from-start off \
  -k regex:"k_move|k_rebuild|k_apply" -c 8 -o gpurun_out/ncu20k_early -f \
  python tools/bench_kernels.py --config 20k --rounds 1 --batches 2 --profile-range > gpurun_out/ncu20k_early.log 2>&1
timeout 1500 ncu --set full --import-source on --clock-control none --profile-from-start off \
  -k regex:"k_move|k_rebuild|k_row|k_hist|k_transpose|k_apply|k_rs|k_seg|k_line" -c 16 -o gpurun_out/ncu2m_r1 -f \
  python tools/bench_kernels.py --config 2m --rounds 1 --batches 1 --profile-range > gpurun_out/ncu2m_r1.log 2>&1
tail -25 gpurun_out/run_*.log; cat gpurun_out/bk2m.log | tail -6
