#!/bin/bash
# Round-2 (final, second session) measurement pass of the current library: the bench line
# (clocks inside), the ncu launch list of the same command, ncu --set full captures of the
# dominant kernels (summaries kept, reports deleted), all clocked.
mkdir -p gpurun_out
tools/clocked.sh bench_w timeout 1500 python bench.py > gpurun_out/bench_w.json 2> gpurun_out/bench_w.err
tools/clocked.sh launches_w timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none -c 20000 --csv \
  --log-file gpurun_out/launches_w.csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e --no-2m > gpurun_out/bench_ncu_w.log 2>&1
python tools/launch_metrics.py gpurun_out/launches_w.csv 40 > gpurun_out/launches_w.txt 2>&1
gzip -f gpurun_out/launches_w.csv
cap() {  # name, kernel regex, count, bench_kernels args...
  local name=$1 rx=$2 n=$3; shift 3
  tools/clocked.sh $name timeout 1500 ncu --set full --import-source on --clock-control none --profile-from-start off \
    -k regex:"$rx" -c $n -o /tmp/$name -f python tools/bench_kernels.py --profile-range "$@" > gpurun_out/$name.log 2>&1
  python tools/ncu_summary.py /tmp/$name.ncu-rep 30 > gpurun_out/$name.txt 2>&1
  rm -f /tmp/$name.ncu-rep
}
cap ncu20k_r5_w "k_move|k_rebuild|k_dense|k_apply|k_nb_update" 8 --config 20k --rounds 5 --batches 2
cap ncu20k_r1_w "k_move|k_rebuild_coop|k_apply|k_nb_update" 6 --config 20k --rounds 1 --batches 2
cap ncu2m_r6_w "k_move_half|k_move_groups|k_segsort|k_line_scatter|k_nb_update|k_propose" 20 --config 2m --rounds 6 --batches 1
cap ncu2m_r4_w "k_move_half|k_move_groups|k_segsort|k_line_scatter|k_nb_update|k_propose" 20 --config 2m --rounds 4 --batches 1
du -sh gpurun_out; cat gpurun_out/bench_w.json | tail -c 2500; head -30 gpurun_out/launches_w.txt
