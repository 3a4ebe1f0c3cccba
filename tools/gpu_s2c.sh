#!/bin/bash
# line sorts after the bank-conflict fix: parity, per-batch times at 2M (line_sort 2 / 1 / 0), per-kernel ncu
mkdir -p gpurun_out
o=gpurun_out/s2c.txt; : > $o
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "rebuild" > gpurun_out/pytest_s2c.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_s2c.log
tail -2 gpurun_out/pytest_s2c.log >> $o
for sb in 2 1 0; do
  echo "== line_sort=$sb" >> $o
  timeout 600 python tools/bench_kernels.py --config 2m --rounds 4 6 --batches 8 --param line_sort=$sb >> $o 2>&1
done
for sb in 2 1; do
timeout 600 ncu --kernel-name regex:"k_segsort|k_line_scatter|k_pull|k_line_len" --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum --clock-control none --profile-from-start off -c 40 --csv --log-file gpurun_out/ncu_s2c_$sb.csv python tools/bench_kernels.py --config 2m --rounds 6 --batches 1 --profile-range --param line_sort=$sb > /dev/null 2>&1
python tools/launch_metrics.py gpurun_out/ncu_s2c_$sb.csv 20 > gpurun_out/ncu_s2c_$sb.txt 2>&1
done
cat $o; cat gpurun_out/ncu_s2c_*.txt
