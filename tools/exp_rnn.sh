for w in 1 0; do echo "=== LSTM WRES=$w"; DUET_RNN_WRES=$w timeout 120 python tools/rnn_trace.py lstm 256 512 256 64 64 | tail -4; done
echo "=== GRU"; timeout 120 python tools/rnn_trace.py gru 64 1024 256 64 64 | tail -4
timeout 600 python -m pytest tests -m gpu -x -q -k "lstm or gru or c3 or c4 or rnn" 2>&1 | tail -3
for c in c3 c4; do timeout 300 python bench.py --config $c --steps 100 --warmup 10 --no-cpu-baseline > gpurun_out/rnn_$c.log 2>&1; done
