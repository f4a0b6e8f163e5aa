# Round-2 final ncu evidence (GPU box; outputs in gpurun_out/):  bash tools/ncu_r2final.sh [tag]
TAG=${1:-r2f}
mkdir -p gpurun_out
# 1) launch lists of 3 DUET steps (cold-cache, serialised: shares only)
for c in c5 c4 c2; do
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv \
      --log-file gpurun_out/${TAG}_launches_${c}.csv python tools/launch_list.py $c 3 > gpurun_out/${TAG}_ll_${c}.log 2>&1
done
# 2) one --set full capture per dominant kernel and per kernel changed this round
full() {  # name regex skip cmd...
  local name=$1 rx=$2 skip=$3; shift 3
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:"$rx" -s $skip -c 1 \
      -o gpurun_out/${TAG}_${name} "$@" > gpurun_out/${TAG}_ncu_${name}.log 2>&1
  ncu -i gpurun_out/${TAG}_${name}.ncu-rep --page raw --csv > gpurun_out/${TAG}_${name}_raw.csv 2>/dev/null
  rm -f gpurun_out/${TAG}_${name}.ncu-rep
}
full gru1024 "rnn_persist" 1 python tools/rnn_trace_plain.py gru 4096 1024 256 16
full fc1 "gemm2_kernel" 2 python tools/gemm_micro_one.py 2048 1024 1664
full lstm "rnn_persist" 1 python tools/rnn_trace_plain.py lstm 256 512 256 64
full gru64 "rnn_persist" 1 python tools/rnn_trace_plain.py gru 64 1024 256 64
full conv64 "conv_tma" 2 python tools/gemm_micro_one.py conv 4096 8 8 64 64 3 1 1
full maxpool "maxpool3s2_rows" 2 python tools/pool_time.py 64 112 112 64
