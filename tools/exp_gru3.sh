mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "rnn_node or small_parity or full_size or variation" > gpurun_out/gru3_tests.log 2>&1; echo rc=$? >> gpurun_out/gru3_tests.log
{
python tools/rnn_time.py gru 64 1024 256 64
python tools/rnn_time.py gru 4096 1024 256 16
python tools/rnn_time.py gru 4096 512 256 32
python tools/rnn_time.py lstm 4096 512 256 32
} > gpurun_out/exp_gru3.log 2>&1
for c in c4 c5; do timeout 400 python bench.py --config $c --steps 100 --warmup 10 --no-cpu-baseline > gpurun_out/bench_gru3_$c.log 2>&1; done
