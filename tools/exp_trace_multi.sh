{
python tools/rnn_trace_multi.py lstm 4096 512 256 30
python tools/rnn_trace_multi.py gru 4096 512 256 30
python tools/rnn_trace_multi.py lstm 4096 256 128 30
} > gpurun_out/trace_multi.log 2>&1
