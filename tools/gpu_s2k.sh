#!/bin/bash
# launch list of one 20K-HH partition (device loop default), 2M round-6 rebuild/move ncu --set full
mkdir -p gpurun_out
o=gpurun_out/s2k.txt; : > $o
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_s2k.csv python tools/run_once.py --config 20k --runs 1 > /dev/null 2>&1
python tools/launch_metrics.py gpurun_out/launches_s2k.csv 40 > gpurun_out/launches_s2k.txt 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"k_segsort_bucket|k_line_scatter|k_move_half|k_move_groups|k_nb_update|k_propose" --profile-from-start off -c 12 -o gpurun_out/ncu_s2k_2m python tools/bench_kernels.py --config 2m --rounds 6 --batches 1 --profile-range > gpurun_out/ncu_s2k.log 2>&1
ncu -i gpurun_out/ncu_s2k_2m.ncu-rep --page raw --csv --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum > gpurun_out/ncu_s2k_2m_raw.csv 2>&1
head -45 gpurun_out/launches_s2k.txt
