#!/bin/bash
# A/B of an experimental library variant: tools/gpu_ab.sh NAME
# (exp/libgsap_NAME.so vs the product library) -- parity tests of the variant,
# then per-batch kernel times of both on the same SBP states.
set -x
name=$1
mkdir -p gpurun_out
GSAP_LIB=$PWD/exp/libgsap_$name.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_scale.py -m gpu -x -q -k move > gpurun_out/pytest_$name.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_$name.log
for lib in $name prod; do
  if [ $lib = prod ]; then unset GSAP_LIB; else export GSAP_LIB=$PWD/exp/libgsap_$name.so; fi
  timeout 600 python tools/bench_kernels.py --config 20k --rounds 1 2 3 --batches 8 > gpurun_out/bk20k_$lib.txt 2>&1
  timeout 900 python tools/bench_kernels.py --config 2m --rounds 3 4 6 --batches 2 > gpurun_out/bk2m_$lib.txt 2>&1
done
tail -n 2 gpurun_out/pytest_$name.log; grep -H "R=" gpurun_out/bk*.txt
