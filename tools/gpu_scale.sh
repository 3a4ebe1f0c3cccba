#!/bin/bash
# Scale pass: end-to-end runs with per-round traces, per-kernel timings on 2M
# states, and ncu --set full captures of the hot kernels (summarised on the box;
# the .ncu-rep files are deleted unless KEEP_REP=1, gpurun_out/ must stay < 64 MiB).
set -x
mkdir -p gpurun_out
for c in ${CONFIGS:-20k 200k 1m 2m}; do
  timeout 1500 python tools/run_once.py --config $c --profile 1 > gpurun_out/run_$c.log 2>&1
done
if [ "${BK:-1}" = 1 ]; then
timeout 900 python tools/bench_kernels.py --config 2m --rounds 1 4 10 19 --batches 8 --json gpurun_out/bk2m.json > gpurun_out/bk2m.log 2>&1
fi
cap() {  # name, kernel regex, count, bench_kernels args...
  local name=$1 rx=$2 n=$3; shift 3
  timeout 1500 ncu --set full --import-source on --clock-control none --profile-from-start off \
    -k regex:"$rx" -c $n -o gpurun_out/$name -f python tools/bench_kernels.py --profile-range "$@" > gpurun_out/$name.log 2>&1
  python tools/ncu_summary.py gpurun_out/$name.ncu-rep > gpurun_out/$name.txt 2>&1
  [ "${KEEP_REP:-0}" = 1 ] || rm -f gpurun_out/$name.ncu-rep
}
if [ "${NCU:-1}" = 1 ]; then
cap ncu20k_late "k_move|k_rebuild|k_row|k_hist|k_transpose|k_apply" 12 --config 20k --rounds 19 --batches 2
cap ncu20k_early "k_move|k_rebuild|k_apply" 8 --config 20k --rounds 1 --batches 2
cap ncu2m_r1 "k_move|k_rebuild|k_row|k_hist|k_transpose|k_apply|k_rs|k_seg|k_line|k_scan" 24 --config 2m --rounds 1 --batches 1
fi
du -sh gpurun_out
