{
python tools/rnn_time.py lstm 4096 512 256 32
DUET_RNN_DBG=32 python tools/rnn_time.py lstm 4096 512 256 32
DUET_RNN_DBG=64 python tools/rnn_time.py lstm 4096 512 256 32
DUET_RNN_DBG=96 python tools/rnn_time.py lstm 4096 512 256 32
DUET_RNN_DBG=16 python tools/rnn_time.py lstm 4096 512 256 32
} > gpurun_out/exp_iso.log 2>&1
