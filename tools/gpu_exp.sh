#!/bin/bash
# A/B of a kernel change: GPU parity tests of the product library, then
# per-batch kernel times of the old (exp/libgsap_old.so) and new library on the
# same SBP states, and the bench line of the new one.
set -x
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -2 gpurun_out/pytest_gpu.log
for lib in old new; do
  if [ $lib = old ]; then export GSAP_LIB=$PWD/exp/libgsap_old.so; else unset GSAP_LIB; fi
  timeout 600 python tools/bench_kernels.py --config 20k --rounds 1 2 3 --batches 8 > gpurun_out/bk20k_$lib.txt 2>&1
  timeout 900 python tools/bench_kernels.py --config 2m --rounds 3 4 6 --batches 2 > gpurun_out/bk2m_$lib.txt 2>&1
done
unset GSAP_LIB
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 1500 python tools/run_once.py --config 2m --runs 1 > gpurun_out/e2e_2m.log 2>&1
timeout 1500 python tools/run_once.py --config 1m --runs 1 > gpurun_out/e2e_1m.log 2>&1
cat gpurun_out/bk*.txt; cat gpurun_out/bench.json; tail -n 3 gpurun_out/e2e_*.log
