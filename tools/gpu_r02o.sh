#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x -k "incremental or lockstep or rebuild or sim_ranks or dense" > gpurun_out/pytest_o.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_o.log
tail -2 gpurun_out/pytest_o.log
for inc in 0 1; do timeout 600 python tools/bench_kernels.py --config 20k --rounds 3 5 8 --batches 16 --param incremental=$inc > gpurun_out/bk20k_o_inc$inc.txt 2>&1; done
timeout 600 python bench.py --no-2m --no-cpu-baseline > gpurun_out/bench_o.json 2>/dev/null
cat gpurun_out/bk20k_o_inc*.txt; python -c "import json; d=json.loads(open('gpurun_out/bench_o.json').read()); print(d['value'], d['ms_per_step'], d['e2e']['value'], d['e2e']['setup_sec'])"
