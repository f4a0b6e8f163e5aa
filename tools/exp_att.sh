mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "attention_node or c6" > gpurun_out/att_tests.log 2>&1; echo rc=$? >> gpurun_out/att_tests.log
timeout 300 python bench.py --config c6 --steps 100 --warmup 10 --no-cpu-baseline > gpurun_out/bench_c6_att.log 2>&1
python tools/node_times.py c6 > gpurun_out/node_times_c6_att.log 2>&1
