mkdir -p gpurun_out
DUET_RNN_WRES_MIN=3 timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "rnn_node or (small_parity and (c3 or c4)) or (full_size_sampled and c4)" > gpurun_out/wres_tests.log 2>&1; echo rc=$? >> gpurun_out/wres_tests.log
{
python tools/rnn_time.py gru 64 1024 256 64
DUET_RNN_WRES_MIN=4 python tools/rnn_time.py gru 64 1024 256 64
DUET_RNN_WRES_MIN=3 python tools/rnn_time.py gru 64 1024 256 64
python tools/rnn_time.py lstm 256 512 256 64
DUET_RNN_WRES_MIN=4 python tools/rnn_time.py lstm 256 512 256 64
} > gpurun_out/exp_wres.log 2>&1
timeout 300 python bench.py --config c4 --steps 100 --warmup 10 --no-cpu-baseline > gpurun_out/bench_c4_w6.log 2>&1
DUET_RNN_WRES_MIN=4 timeout 300 python bench.py --config c4 --steps 100 --warmup 10 --no-cpu-baseline > gpurun_out/bench_c4_w4.log 2>&1
