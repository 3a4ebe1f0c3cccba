#!/bin/bash
mkdir -p gpurun_out
GSAP_LIB=exp/libgsap_coopprof.so timeout 300 python tools/bench_kernels.py --config 20k --rounds 1 3 --batches 8 > gpurun_out/coopprof.txt 2>&1
grep -v "^COOP" gpurun_out/coopprof.txt; grep "^COOP" gpurun_out/coopprof.txt | tail -12
timeout 1200 /usr/local/cuda/bin/compute-sanitizer --tool racecheck --racecheck-report all --print-limit 60 python tools/sanitize_run.py > gpurun_out/racecheck_all.txt 2>&1
echo "exit=$?" >> gpurun_out/racecheck_all.txt
tail -3 gpurun_out/racecheck_all.txt
grep -E "^========= +(Warning|Error)" gpurun_out/racecheck_all.txt | sort | uniq -c | head
grep -E "in .*k_|at .*\.cu" gpurun_out/racecheck_all.txt | sort | uniq -c | sort -rn | head -20
