#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x -k "launch_shape or hubs or big_vertices or lockstep or isolated or sim_ranks" > gpurun_out/pytest_j.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_j.log
tail -2 gpurun_out/pytest_j.log
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_bytes.sum --clock-control none \
    --profile-from-start off --csv --log-file gpurun_out/l2m_j.csv \
    python tools/bench_kernels.py --profile-range --config 2m --rounds 3 6 --batches 2 > /dev/null 2>&1
python tools/launch_metrics.py gpurun_out/l2m_j.csv 6 > gpurun_out/l2m_j.txt 2>&1
timeout 600 python tools/bench_kernels.py --config 2m --rounds 3 6 --batches 8 > gpurun_out/bk2m_j.txt 2>&1
timeout 600 python tools/bench_kernels.py --config 20k --rounds 1 3 5 --batches 16 > gpurun_out/bk20k_j.txt 2>&1
cat gpurun_out/l2m_j.txt gpurun_out/bk2m_j.txt gpurun_out/bk20k_j.txt
bash tools/gpu_r02_sanitize.sh
