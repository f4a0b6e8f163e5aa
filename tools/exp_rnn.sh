timeout 600 python -m pytest tests -m gpu -x -q -k "lstm or gru or c3 or c4 or rnn or c5" 2>&1 | tail -3
for cn in 8 4 1; do echo "=== LSTM CN=$cn"; DUET_RNN_CN=$cn timeout 120 python tools/rnn_trace.py lstm 256 512 256 64 64 | tail -4; done
for cn in 8 1; do echo "=== GRU CN=$cn"; DUET_RNN_CN=$cn timeout 120 python tools/rnn_trace.py gru 64 1024 256 64 64 | tail -4; done
for c in c3 c4; do timeout 400 python bench.py --config $c --steps 100 --warmup 10 --no-cpu-baseline > gpurun_out/bench_$c.log 2>&1; done
