mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "rnn_node or (full_size_sampled and c5) or (small_parity and (c3 or c4 or c5))" > gpurun_out/ld_tests.log 2>&1; echo rc=$? >> gpurun_out/ld_tests.log
{
python tools/rnn_time.py lstm 256 512 256 64
python tools/rnn_time.py gru 64 1024 256 64
python tools/rnn_time.py lstm 4096 256 128 64
} > gpurun_out/exp_ld.log 2>&1
for c in c3 c4; do timeout 300 python bench.py --config $c --steps 100 --warmup 10 --no-cpu-baseline > gpurun_out/bench_ld_$c.log 2>&1; done
