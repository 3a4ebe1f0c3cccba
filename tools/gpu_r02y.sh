#!/bin/bash
mkdir -p gpurun_out
o=gpurun_out/y.txt; : > $o
timeout 900 python -m pytest tests -m gpu -q -x -k "lockstep or hubs or big_vertices or launch_shape or 200k_fused or weighted" > gpurun_out/pytest_y.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_y.log
tail -2 gpurun_out/pytest_y.log >> $o
for lib in exp/libgsap_nostream.so paper_conf_icpp_changzh24_b200/libgsap.so; do
  echo "== $lib" >> $o
  GSAP_LIB=$lib timeout 300 python tools/bench_kernels.py --config 20k --rounds 1 2 3 --batches 16 >> $o 2>&1
  GSAP_LIB=$lib timeout 300 python tools/bench_kernels.py --config 200k --rounds 2 5 --batches 8 >> $o 2>&1
  GSAP_LIB=$lib timeout 600 python tools/bench_kernels.py --config 2m --rounds 6 --batches 8 >> $o 2>&1
done
echo "== regime: default vs dense_max_B=1 (always sparse)" >> $o
timeout 300 python tools/bench_kernels.py --config 20k --rounds 4 5 6 8 --batches 16 >> $o 2>&1
timeout 300 python tools/bench_kernels.py --config 20k --rounds 4 5 6 8 --batches 16 --dense-max-B 1 >> $o 2>&1
for i in 1 2; do timeout 600 python bench.py --no-2m --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads([l for l in sys.stdin if l.startswith('{')][-1]); print('bench', d['value'], d['ms_per_step'], d['e2e']['value'])" >> $o; done
cat $o
