mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "rnn_node or (full_size_sampled and c5)" > gpurun_out/b3b_tests.log 2>&1; echo rc=$? >> gpurun_out/b3b_tests.log
{
python tools/rnn_time.py lstm 4096 256 128 64
python tools/rnn_time.py lstm 4096 512 256 32
python tools/rnn_time.py gru 4096 1024 256 16
python tools/rnn_time.py gru 4096 512 256 32
} > gpurun_out/exp_b3b.log 2>&1
