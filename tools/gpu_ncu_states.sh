# ncu --set full captures of the hot kernels in chosen states (summaries only; .ncu-rep deleted)
set -x
mkdir -p gpurun_out
cap() {
  local name=$1 rx=$2 n=$3; shift 3
  timeout 900 ncu --set full --import-source on --clock-control none --profile-from-start off \
    -k regex:"$rx" -c $n -o gpurun_out/$name -f python tools/bench_kernels.py --profile-range "$@" > gpurun_out/$name.log 2>&1
  python tools/ncu_summary.py gpurun_out/$name.ncu-rep 40 > gpurun_out/$name.txt 2>&1
  rm -f gpurun_out/$name.ncu-rep
}
cap ncu20k_r1 "k_rebuild_coop" 2 --config 20k --rounds 1 --batches 2
cap ncu20k_r4 "k_hist|k_transpose|k_row|k_scan|k_move|k_apply" 12 --config 20k --rounds 4 --batches 2
cap ncu200k_r3 "k_rebuild_coop|k_move" 3 --config 200k --rounds 3 --batches 1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv --log-file gpurun_out/l20k_r4.csv python tools/bench_kernels.py --profile-range --config 20k --rounds 4 --batches 8 > /dev/null 2>&1
python tools/launch_summary.py gpurun_out/l20k_r4.csv 20 > gpurun_out/l20k_r4.txt
