#!/bin/bash
# A/B: staged vs global-search sorted passes, groups at 2 CTAs/SM; 2M and 20K per-batch timings + 2M launch lists.
mkdir -p gpurun_out
for st in 0 1; do
  GSAP_MOVE_STAGE=$st timeout 900 python tools/bench_kernels.py --config 2m --rounds 3 4 6 --batches 8 > gpurun_out/bk2m_f_st$st.txt 2>&1
  GSAP_MOVE_STAGE=$st timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_bytes.sum --clock-control none \
    --profile-from-start off --csv --log-file gpurun_out/l2m_r6_f_st$st.csv \
    python tools/bench_kernels.py --profile-range --config 2m --rounds 6 --batches 2 > /dev/null 2>&1
  python tools/launch_metrics.py gpurun_out/l2m_r6_f_st$st.csv 12 > gpurun_out/l2m_r6_f_st$st.txt 2>&1
done
timeout 600 python tools/bench_kernels.py --config 20k --rounds 1 3 5 8 --batches 16 > gpurun_out/bk20k_f.txt 2>&1
cat gpurun_out/bk2m_f_st*.txt gpurun_out/l2m_r6_f_st*.txt gpurun_out/bk20k_f.txt
