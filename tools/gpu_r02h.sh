#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x -k "sorted or 200k_fused or sim_ranks or incremental or lockstep or table_mode" > gpurun_out/pytest_h.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_h.log
tail -2 gpurun_out/pytest_h.log
for v in base halfminb4; do
  if [ $v = base ]; then L=paper_conf_icpp_changzh24_b200/libgsap.so; else L=exp/libgsap_$v.so; fi
  GSAP_LIB=$L timeout 600 python tools/bench_kernels.py --config 2m --rounds 3 6 --batches 8 > gpurun_out/bk2m_h_$v.txt 2>&1
done
for inc in 0 1; do
  timeout 600 python tools/bench_kernels.py --config 20k --rounds 3 5 8 12 --batches 16 --param incremental=$inc > gpurun_out/bk20k_h_inc$inc.txt 2>&1
done
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_bytes.sum --clock-control none \
    --profile-from-start off --csv --log-file gpurun_out/l2m_r6_h.csv \
    python tools/bench_kernels.py --profile-range --config 2m --rounds 6 --batches 2 > /dev/null 2>&1
python tools/launch_metrics.py gpurun_out/l2m_r6_h.csv 8 > gpurun_out/l2m_r6_h.txt 2>&1
timeout 600 python bench.py --steps 3 --warmup 3 --no-2m --no-cpu-baseline > gpurun_out/bench_h.json 2>gpurun_out/bench_h.err
timeout 900 python tools/ablation_n4.py 20k 200k > gpurun_out/ablation_n4.jsonl 2>&1
for v in base halfminb4; do echo "== $v"; cat gpurun_out/bk2m_h_$v.txt; done; cat gpurun_out/bk20k_h_inc*.txt gpurun_out/l2m_r6_h.txt gpurun_out/bench_h.json
cat gpurun_out/ablation_n4.jsonl
