#!/bin/bash
# Round-end evidence pass (second): tests + smoke, bench line, launch list,
# unprofiled end-to-end partitions at 1K..2M, ncu of the 2M round-6 state.
set -x
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
  python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/bench_ncu.log 2>&1
python tools/launch_summary.py gpurun_out/launches.csv 60 > gpurun_out/launches.txt
for c in 1k 20k 200k 1m 2m; do
  timeout 1500 python tools/run_once.py --config $c --runs 2 > gpurun_out/e2e_$c.log 2>&1
done
timeout 1500 ncu --set full --import-source on --clock-control none --profile-from-start off \
  -k regex:"k_move|k_line|k_seg" -c 12 -o gpurun_out/ncu_2m_r6 -f python tools/bench_kernels.py --profile-range --config 2m --rounds 6 --batches 1 > gpurun_out/ncu_2m_r6.log 2>&1
python tools/ncu_summary.py gpurun_out/ncu_2m_r6.ncu-rep 30 > gpurun_out/ncu_2m_r6.txt 2>&1
rm -f gpurun_out/ncu_2m_r6.ncu-rep
du -sh gpurun_out
