#!/bin/bash
# the final bench line of the round (full default run, clocked) + its launch list
mkdir -p gpurun_out
tools/clocked.sh bench_final2 timeout 1500 python bench.py > gpurun_out/bench_final2.json 2> gpurun_out/bench_final2.err
tools/clocked.sh launches_final2 timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none -c 20000 --csv \
  --log-file gpurun_out/launches_final2.csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e --no-2m > /dev/null 2>&1
python tools/launch_metrics.py gpurun_out/launches_final2.csv 40 > gpurun_out/launches_final2.txt 2>&1
gzip -f gpurun_out/launches_final2.csv
tail -c 1500 gpurun_out/bench_final2.json
