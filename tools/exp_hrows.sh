mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "rnn_node or small_parity or variation or full_size" > gpurun_out/hrows_tests.log 2>&1; echo rc=$? >> gpurun_out/hrows_tests.log
{
python tools/rnn_time.py gru 64 1024 256 64
python tools/rnn_time.py gru 1 1024 256 64
python tools/rnn_time.py gru 16 1024 256 64
python tools/rnn_time.py lstm 256 512 256 64
} > gpurun_out/exp_hrows.log 2>&1
timeout 600 python tools/sweeps.py --only batch,rnn --out gpurun_out/sweeps_hrows.json > gpurun_out/sweeps_hrows.log 2>&1
timeout 300 python bench.py --config c4 --steps 100 --warmup 10 --no-cpu-baseline > gpurun_out/bench_c4_hrows.log 2>&1
