#!/bin/bash
# sim_ranks multi-GPU data path tests; ncu --set full of the staged MOVE passes and the group kernel at 2M
# round 6; one bench.py run (new contract fields).
mkdir -p gpurun_out
nvidia-smi --query-gpu=clocks.sm,clocks.max.sm --format=csv > gpurun_out/clk_e.txt
timeout 1200 python -m pytest tests/test_gpu_multi.py -q -x > gpurun_out/pytest_e.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_e.log
tail -3 gpurun_out/pytest_e.log
timeout 900 ncu --set full --import-source on --clock-control none --profile-from-start off \
   -k regex:"k_move_half|k_move_groups" -c 3 -o gpurun_out/ncu2m_r6_half -f \
   python tools/bench_kernels.py --profile-range --config 2m --rounds 6 --batches 1 > gpurun_out/ncu2m_r6_half.log 2>&1
python tools/ncu_summary.py gpurun_out/ncu2m_r6_half.ncu-rep 40 > gpurun_out/ncu2m_r6_half.txt 2>&1
rm -f gpurun_out/ncu2m_r6_half.ncu-rep
nvidia-smi --query-gpu=clocks.sm,clocks.max.sm --format=csv >> gpurun_out/clk_e.txt
timeout 1500 python bench.py --steps 3 --warmup 3 > gpurun_out/bench_e.json 2> gpurun_out/bench_e.err
cat gpurun_out/bench_e.json; tail -5 gpurun_out/bench_e.err
