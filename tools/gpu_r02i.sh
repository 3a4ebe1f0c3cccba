#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x -k "table_mode or incremental or sorted" > gpurun_out/pytest_i.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_i.log
tail -2 gpurun_out/pytest_i.log
for v in base halfk1 halfk2 halfminb4; do
  if [ $v = base ]; then L=paper_conf_icpp_changzh24_b200/libgsap.so; else L=exp/libgsap_$v.so; fi
  GSAP_LIB=$L timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_bytes.sum --clock-control none \
    --profile-from-start off --csv --log-file gpurun_out/l2m_r6_i_$v.csv \
    python tools/bench_kernels.py --profile-range --config 2m --rounds 3 6 --batches 2 > /dev/null 2>&1
  python tools/launch_metrics.py gpurun_out/l2m_r6_i_$v.csv 4 > gpurun_out/l2m_r6_i_$v.txt 2>&1
done
timeout 600 python tools/bench_kernels.py --config 20k --rounds 8 12 16 --batches 16 > gpurun_out/bk20k_i.txt 2>&1
for v in base halfk1 halfk2 halfminb4; do echo "== $v"; cat gpurun_out/l2m_r6_i_$v.txt; done; cat gpurun_out/bk20k_i.txt
