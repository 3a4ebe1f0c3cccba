#!/bin/bash
mkdir -p gpurun_out
o=gpurun_out/e2.txt; : > $o
timeout 900 python -m pytest tests -m gpu -q -x -k "sorted or lockstep or 200k_fused or launch_shape" > gpurun_out/pytest_e2.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_e2.log
tail -2 gpurun_out/pytest_e2.log >> $o
for lib in exp/libgsap_base.so paper_conf_icpp_changzh24_b200/libgsap.so exp/libgsap_base.so paper_conf_icpp_changzh24_b200/libgsap.so; do
  echo "== $lib" >> $o
  GSAP_LIB=$lib GSAP_TIMING=1 timeout 600 python tools/bench_kernels.py --config 2m --rounds 3 6 --batches 8 2>&1 | grep -E "roles|R=" >> $o
done
cat $o
