#!/bin/bash
mkdir -p gpurun_out
for rep in 1 2; do
for v in base nopool; do
  if [ $v = base ]; then L=paper_conf_icpp_changzh24_b200/libgsap.so; else L=exp/libgsap_$v.so; fi
  GSAP_LIB=$L timeout 600 python bench.py --no-2m --no-cpu-baseline > gpurun_out/bench_n_${v}_$rep.json 2>/dev/null
  python -c "import json,sys; d=json.loads(open('gpurun_out/bench_n_${v}_$rep.json').read()); print('$v', $rep, d['value'], d['ms_per_step'], d['e2e']['value'], d['e2e']['setup_sec'])"
done; done
timeout 1800 python tools/ablation_n2.py 20k 200k 2m > gpurun_out/ablation_n2.jsonl 2>&1
cat gpurun_out/ablation_n2.jsonl
