{
python tools/rnn_trace_multi.py lstm 4096 512 256 30
python tools/rnn_trace_multi.py gru 4096 1024 256 16
} > gpurun_out/trace_multi3.log 2>&1
