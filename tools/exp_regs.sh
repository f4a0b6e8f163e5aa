mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "rnn_node or (full_size_sampled and c5) or (small_parity and c5)" > gpurun_out/regs_tests.log 2>&1; echo rc=$? >> gpurun_out/regs_tests.log
{
python tools/rnn_time.py lstm 4096 512 256 32
python tools/rnn_time.py gru 4096 512 256 32
python tools/rnn_time.py gru 4096 1024 256 16
python tools/rnn_time.py lstm 4096 256 128 64
} > gpurun_out/exp_regs.log 2>&1
timeout 300 python bench.py --config c5 --steps 30 --warmup 5 --no-cpu-baseline > gpurun_out/bench_c5_regs.log 2>&1
