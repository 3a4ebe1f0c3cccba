#!/bin/bash
# round-2 evidence of the current library: full bench line, its launch list, ncu --set full of the
# 20K-HH move / apply / rebuild kernels and of the 2M-LL round-4 / round-6 move and rebuild kernels
mkdir -p gpurun_out
bash tools/clocked.sh bench_s2 python bench.py > gpurun_out/bench_full_s2.json 2> gpurun_out/bench_full_s2.err
bash tools/clocked.sh launches_s2 ncu --metrics gpu__time_duration.sum --clock-control none -c 6000 --csv --log-file gpurun_out/bench_launches_s2.csv python bench.py --steps 1 --warmup 1 --no-2m --no-cpu-baseline --no-e2e > /dev/null 2>&1
python tools/launch_metrics.py gpurun_out/bench_launches_s2.csv 40 > gpurun_out/bench_launches_s2.txt 2>&1
bash tools/clocked.sh ncu20k_s2 ncu --set full --import-source on --clock-control none -k regex:"k_move|k_apply|k_nb_update|k_dense|k_rebuild" --profile-from-start off -c 10 -o gpurun_out/ncu20k_r5_s2 python tools/bench_kernels.py --config 20k --rounds 5 --batches 1 --profile-range > /dev/null 2>&1
for R in 4 6; do
bash tools/clocked.sh ncu2m_r${R}_s2 ncu --set full --clock-control none -k regex:"k_move|k_propose|k_nb_update|k_segsort|k_line|k_sort" --profile-from-start off -c 16 -o gpurun_out/ncu2m_r${R}_s2 python tools/bench_kernels.py --config 2m --rounds $R --batches 1 --profile-range > /dev/null 2>&1
done
for f in ncu20k_r5_s2 ncu2m_r4_s2 ncu2m_r6_s2; do
  ncu -i gpurun_out/$f.ncu-rep --page raw --csv --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum,launch__grid_size,launch__registers_per_thread > gpurun_out/${f}_raw.csv 2>&1
done
tail -c 3000 gpurun_out/bench_full_s2.json; head -30 gpurun_out/bench_launches_s2.txt; tail -1 gpurun_out/clocks_*.csv
