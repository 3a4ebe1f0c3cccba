#!/bin/bash
# e2e (gsap_partition: create + H2D + run + D2H + destroy) A/B: current vs the library before the deferred dS sum
mkdir -p gpurun_out
o=gpurun_out/s2y.txt; : > $o
for i in 1 2; do
echo "== current" >> $o; GSAP_TIMING=1 timeout 120 python tools/e2e_timing.py 20k >> $o 2>gpurun_out/s2y_cur_$i.err
echo "== base" >> $o; GSAP_LIB=exp/libgsap_base.so GSAP_TIMING=1 timeout 120 python tools/e2e_timing.py 20k >> $o 2>gpurun_out/s2y_base_$i.err
done
for i in 1 2; do timeout 600 python bench.py --no-2m --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads([l for l in sys.stdin if l.startswith('{')][-1]); print('bench', d['value'], d['ms_per_step'], d['e2e']['value'], d['e2e']['partition_sec'])" >> $o; done
grep -E "create|mcmc B=12000|destroy" gpurun_out/s2y_cur_2.err | head -20 >> $o
echo "-- base" >> $o
grep -E "create|mcmc B=12000|destroy" gpurun_out/s2y_base_2.err | head -20 >> $o
cat $o
