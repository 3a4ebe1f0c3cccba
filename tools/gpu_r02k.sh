#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x -k "rebuild or lockstep or launch_shape or hubs" > gpurun_out/pytest_k.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_k.log
tail -2 gpurun_out/pytest_k.log
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_bytes.sum --clock-control none \
    --profile-from-start off --csv --log-file gpurun_out/l2m_k.csv \
    python tools/bench_kernels.py --profile-range --config 2m --rounds 3 6 --batches 2 > /dev/null 2>&1
python tools/launch_metrics.py gpurun_out/l2m_k.csv 8 > gpurun_out/l2m_k.txt 2>&1
timeout 600 python tools/bench_kernels.py --config 2m --rounds 3 6 --batches 8 > gpurun_out/bk2m_k.txt 2>&1
timeout 600 python tools/bench_kernels.py --config 20k --rounds 1 3 5 --batches 16 > gpurun_out/bk20k_k.txt 2>&1
timeout 600 python tools/bench_kernels.py --config 200k --rounds 1 3 5 --batches 8 > gpurun_out/bk200k_k.txt 2>&1
cat gpurun_out/l2m_k.txt gpurun_out/bk2m_k.txt gpurun_out/bk20k_k.txt gpurun_out/bk200k_k.txt
CS=/usr/local/cuda/bin/compute-sanitizer
timeout 1500 $CS --tool racecheck --racecheck-report all --print-limit 2000 python tools/sanitize_run.py > gpurun_out/sanitizer_racecheck.txt 2>&1; echo "exit=$?" >> gpurun_out/sanitizer_racecheck.txt
tail -3 gpurun_out/sanitizer_racecheck.txt
