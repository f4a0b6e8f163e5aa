mkdir -p gpurun_out
DUET_RNN_BN=256 timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "rnn_node_seq_output or (full_size_sampled and c5)" -s > gpurun_out/rnn256_tests.log 2>&1; echo rc=$? >> gpurun_out/rnn256_tests.log
DUET_RNN_BN=256 timeout 300 python bench.py --config c5 --steps 30 --warmup 5 --no-cpu-baseline --sched model > gpurun_out/bench_c5_rnn256.log 2>&1
timeout 300 python bench.py --config c5 --steps 30 --warmup 5 --no-cpu-baseline --sched model > gpurun_out/bench_c5_rnn128.log 2>&1
