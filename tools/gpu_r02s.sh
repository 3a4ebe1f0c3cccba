#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x -k "hubs or big_vertices or lockstep or launch_shape or isolated or move_proposals or 200k or weighted" > gpurun_out/pytest_s.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_s.log
tail -2 gpurun_out/pytest_s.log
timeout 600 python tools/bench_kernels.py --config 20k --rounds 1 3 5 8 --batches 16 > gpurun_out/bk20k_s.txt 2>&1
timeout 600 python tools/bench_kernels.py --config 2m --rounds 3 6 --batches 8 > gpurun_out/bk2m_s.txt 2>&1
timeout 600 python bench.py --no-2m --no-cpu-baseline > gpurun_out/bench_s.json 2>/dev/null
cat gpurun_out/bk20k_s.txt gpurun_out/bk2m_s.txt; python -c "import json; d=json.loads(open('gpurun_out/bench_s.json').read()); print(d['value'], d['ms_per_step'], d['e2e']['value'])"
