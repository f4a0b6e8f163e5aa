mkdir -p gpurun_out
{
python tools/rnn_time.py lstm 4096 256 128 64
DUET_RNN_BN=64 python tools/rnn_time.py lstm 4096 256 128 64
DUET_RNN_GRID=128 python tools/rnn_time.py lstm 4096 256 128 64
DUET_RNN_BN=64 DUET_RNN_GRID=128 python tools/rnn_time.py lstm 4096 256 128 64
python tools/rnn_time.py lstm 4096 256 128 8
python tools/rnn_time.py lstm 4096 512 256 32
DUET_RNN_BN=128 python tools/rnn_time.py lstm 4096 512 256 32
python tools/rnn_time.py gru 4096 1024 256 16
python tools/rnn_time.py gru 4096 512 256 32
} > gpurun_out/exp_b3.log 2>&1
