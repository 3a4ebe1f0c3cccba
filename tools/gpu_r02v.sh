#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x -k "rebuild or padded or lockstep or 200k_fused or edge_cases or device_outputs or partition_oneshot" > gpurun_out/pytest_v.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_v.log
tail -2 gpurun_out/pytest_v.log
timeout 600 python tools/bench_kernels.py --config 2m --rounds 4 6 --batches 8 > gpurun_out/bk2m_v.txt 2>&1
GSAP_TIMING=1 timeout 300 python tools/e2e_timing.py 20k > gpurun_out/e2e_v.txt 2>&1
timeout 600 python bench.py --no-2m --no-cpu-baseline > gpurun_out/bench_v.json 2>/dev/null
cat gpurun_out/bk2m_v.txt; grep -E "e2e|arena|destroy" gpurun_out/e2e_v.txt | tail -12
python -c "import json; d=json.loads(open('gpurun_out/bench_v.json').read()); print(d['value'], d['ms_per_step'], d['e2e'])"
