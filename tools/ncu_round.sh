# ncu evidence for this round: bash tools/ncu_round.sh <tag>   (GPU box; outputs in gpurun_out/)
TAG=${1:-r1b}
mkdir -p gpurun_out
# 1) launch list of our kernels during bench.py c2 timed steps (cold-cache, serialised: shares only)
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
    -k regex:"gemm|gather|hash|join|conv|im2col|pool|mlp|rnn|reduce|add_act|sigmoid|logit|concat|linear" \
    --csv --log-file gpurun_out/launches_${TAG}.csv \
    python bench.py --steps 3 --warmup 3 --no-cpu-baseline --profile-samples 2 --sched model > gpurun_out/ncu_launch_${TAG}.log 2>&1
# 2) full captures: fc1 (pair GEMM 2048x1024x1664), the deep gather, the persistent LSTM (c3 tower)
full() {  # name regex skip count cmd...
  local name=$1 rx=$2 skip=$3; shift 3
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:"$rx" -s $skip -c 1 \
      -o gpurun_out/${name}_${TAG} "$@" > gpurun_out/ncu_${name}_${TAG}.log 2>&1
  ncu -i gpurun_out/${name}_${TAG}.ncu-rep --page raw --csv > gpurun_out/${name}_${TAG}_raw.csv 2>/dev/null
}
full fc1 "gemm2_kernel" 2 python tools/gemm_micro_one.py 2048 1024 1664
full gather "gather_rows16" 2 python tools/gemm_micro_one.py gather
full lstm "rnn_persist" 1 python tools/rnn_trace_plain.py lstm 256 512 256 64
full gru "rnn_persist" 1 python tools/rnn_trace_plain.py gru 64 1024 256 64
# 3) r1c additions: c5-size LSTM (several 128x256 tiles per CTA) and the MT-DNN attention
full lstmB4096 "rnn_persist" 1 python tools/rnn_trace_plain.py lstm 4096 512 256 8
