#!/bin/bash
mkdir -p gpurun_out
for v in base latency; do
  if [ $v = base ]; then L=paper_conf_icpp_changzh24_b200/libgsap.so; else L=exp/libgsap_$v.so; fi
  GSAP_LIB=$L timeout 600 python tools/bench_kernels.py --config 20k --rounds 1 3 5 8 --batches 16 > gpurun_out/bk20k_t_$v.txt 2>&1
  GSAP_LIB=$L timeout 600 python bench.py --no-2m --no-cpu-baseline > gpurun_out/bench_t_$v.json 2>/dev/null
  echo "== $v"; cat gpurun_out/bk20k_t_$v.txt
  python -c "import json; d=json.loads(open('gpurun_out/bench_t_$v.json').read()); print(d['value'], d['ms_per_step'], d['e2e']['value'])"
done
GSAP_LIB=exp/libgsap_latency.so timeout 900 python -m pytest tests -m gpu -q -x -k "hubs or big_vertices or launch_shape or lockstep" > gpurun_out/pytest_t.log 2>&1; tail -1 gpurun_out/pytest_t.log
