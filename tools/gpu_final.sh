#!/bin/bash
# Round-end evidence pass: GPU tests + smoke, the bench line (+ reference arm),
# the launch list of the bench command, ncu --set full of the dominant kernel
# in the bench's states, end-to-end traces at 200K / 1M / 2M.
set -x
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 900 python bench.py --impl reference --steps 2 --warmup 0 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
  python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/bench_ncu.log 2>&1
python tools/launch_summary.py gpurun_out/launches.csv 60 > gpurun_out/launches.txt
cap() {
  local name=$1 rx=$2 n=$3; shift 3
  timeout 900 ncu --set full --import-source on --clock-control none --profile-from-start off \
    -k regex:"$rx" -c $n -o gpurun_out/$name -f python tools/bench_kernels.py --profile-range "$@" > gpurun_out/$name.log 2>&1
  python tools/ncu_summary.py gpurun_out/$name.ncu-rep 30 > gpurun_out/$name.txt 2>&1
  rm -f gpurun_out/$name.ncu-rep
}
cap ncu_move20k_late "k_move|k_rebuild_dense|k_apply" 6 --config 20k --rounds 19 --batches 2
cap ncu_move20k_early "k_move|k_rebuild_coop|k_apply" 8 --config 20k --rounds 1 --batches 2
cap ncu_2m_r4 "k_move|k_line|k_seg|k_scan" 24 --config 2m --rounds 4 --batches 1
for c in ${CONFIGS:-200k 1m 2m}; do
  timeout 1500 python tools/run_once.py --config $c --profile 1 > gpurun_out/run_$c.log 2>&1
done
du -sh gpurun_out
