mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "attention_node or layernorm_node or c6" -s > gpurun_out/c6_tests.log 2>&1; echo rc=$? >> gpurun_out/c6_tests.log
timeout 300 python bench.py --config c6 --steps 100 --warmup 10 --no-cpu-baseline > gpurun_out/bench_c6.log 2>&1
python tools/node_times.py c6 > gpurun_out/node_times_c6.log 2>&1
