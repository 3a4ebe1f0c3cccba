#!/bin/bash
# bucket sort v2 (rank scatter + range insertion): parity, 2M per-batch times, sort kernels ncu, full 2M partition
mkdir -p gpurun_out
o=gpurun_out/s2d.txt; : > $o
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "rebuild" > gpurun_out/pytest_s2d.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_s2d.log
tail -2 gpurun_out/pytest_s2d.log >> $o
for sb in 1 0; do
  echo "== line_sort=$sb" >> $o
  timeout 600 python tools/bench_kernels.py --config 2m --rounds 4 6 --batches 8 --param line_sort=$sb >> $o 2>&1
done
timeout 600 ncu --kernel-name regex:"k_segsort|k_line_scatter|k_line_len" --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum --clock-control none --profile-from-start off -c 40 --csv --log-file gpurun_out/ncu_s2d.csv python tools/bench_kernels.py --config 2m --rounds 6 --batches 1 --profile-range > /dev/null 2>&1
python tools/launch_metrics.py gpurun_out/ncu_s2d.csv 20 > gpurun_out/ncu_s2d.txt 2>&1
timeout 600 python tools/e2e_timing.py 2m >> $o 2>&1
cat $o; cat gpurun_out/ncu_s2d.txt
