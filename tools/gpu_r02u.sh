#!/bin/bash
mkdir -p gpurun_out
tools/clocked.sh bench_u timeout 1500 python bench.py > gpurun_out/bench_u.json 2> gpurun_out/bench_u.err
GSAP_TIMING=1 timeout 300 python tools/e2e_timing.py 20k > gpurun_out/e2e_u.txt 2>&1
grep -v "^clocks" gpurun_out/bench_u.json | python -c "
import json,sys
d=json.loads(sys.stdin.read())
print('value',d['value'],'ms',d['ms_per_step'],'e2e',d['e2e']['value'],d['e2e']['partition_sec'],d['e2e']['setup_sec'])
r=d['roofline_2m']
for st in r['states']: print(st['rounds'],st['B'],'move',st['move']['ms_per_launch'],'rebuild',st['rebuild']['ms_per_launch'],st['rebuild']['frac'])
print('2m',r['partition_2m'])
print('cpu',d['cpu_baseline']['value'],d['cpu_baseline']['seconds'])
print(d['clocks'])"
grep -E "create|e2e" gpurun_out/e2e_u.txt | tail -20
