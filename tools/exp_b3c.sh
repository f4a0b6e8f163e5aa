{
python tools/rnn_time.py lstm 1024 256 128 64
python tools/rnn_time.py lstm 2048 256 128 64
python tools/rnn_time.py lstm 2432 256 128 64
python tools/rnn_time.py lstm 4096 256 128 64
DUET_RNN_GRID=128 python tools/rnn_time.py lstm 4096 256 128 64
python tools/rnn_time.py lstm 8192 256 128 64
} > gpurun_out/exp_b3c.log 2>&1
