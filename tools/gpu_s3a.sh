#!/bin/bash
# the final bench line of the round (full default run, clocked)
mkdir -p gpurun_out
tools/clocked.sh bench_final timeout 1500 python bench.py > gpurun_out/bench_final.json 2> gpurun_out/bench_final.err
tail -c 1500 gpurun_out/bench_final.json
