#!/bin/bash
mkdir -p gpurun_out
for v in base halfminb4 groups3; do
  if [ $v = base ]; then L=paper_conf_icpp_changzh24_b200/libgsap.so; else L=exp/libgsap_$v.so; fi
  GSAP_LIB=$L timeout 600 python tools/bench_kernels.py --config 2m --rounds 3 6 --batches 8 > gpurun_out/bk2m_g_$v.txt 2>&1
  GSAP_LIB=$L timeout 600 python tools/bench_kernels.py --config 20k --rounds 1 3 5 --batches 16 > gpurun_out/bk20k_g_$v.txt 2>&1
done
for v in base halfminb4 groups3; do echo "== $v"; cat gpurun_out/bk2m_g_$v.txt gpurun_out/bk20k_g_$v.txt; done
