{
python tools/rnn_trace.py gru 64 1024 256 64
python tools/rnn_trace.py lstm 256 512 256 64
} > gpurun_out/trace1.log 2>&1
