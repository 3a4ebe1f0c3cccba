#!/bin/bash
# Round-2 measurement pass: bench line (clocks inside), the ncu launch list of the
# same command, ncu --set full captures of the dominant kernels (traffic), all clocked.
mkdir -p gpurun_out
tools/clocked.sh bench timeout 1500 python bench.py > gpurun_out/bench_m.json 2> gpurun_out/bench_m.err
tools/clocked.sh launches timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none -c 20000 --csv \
  --log-file gpurun_out/launches_m.csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e --no-2m > gpurun_out/bench_ncu_m.log 2>&1
python tools/launch_summary.py gpurun_out/launches_m.csv 40 > gpurun_out/launches_m.txt 2>&1
cap() {  # name, kernel regex, count, bench_kernels args...
  local name=$1 rx=$2 n=$3; shift 3
  tools/clocked.sh $name timeout 1500 ncu --set full --import-source on --clock-control none --profile-from-start off \
    -k regex:"$rx" -c $n -o gpurun_out/$name -f python tools/bench_kernels.py --profile-range "$@" > gpurun_out/$name.log 2>&1
  python tools/ncu_summary.py gpurun_out/$name.ncu-rep 30 > gpurun_out/$name.txt 2>&1
  rm -f gpurun_out/$name.ncu-rep
}
cap ncu20k_r4_move "k_move|k_rebuild|k_dense_delta|k_row|k_apply" 8 --config 20k --rounds 4 --batches 2
cap ncu20k_r1_move "k_move|k_rebuild_coop|k_apply" 6 --config 20k --rounds 1 --batches 2
cap ncu2m_r6 "k_move_half|k_move_groups|k_segsort_warp|k_line_scatter" 8 --config 2m --rounds 6 --batches 1
cap ncu2m_r4 "k_move_half|k_move_groups|k_segsort_warp|k_line_scatter" 8 --config 2m --rounds 4 --batches 1
cat gpurun_out/bench_m.json; head -30 gpurun_out/launches_m.txt
