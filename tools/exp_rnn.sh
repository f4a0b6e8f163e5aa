timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
timeout 600 python tools/node_times.py c5 > gpurun_out/nodes_c5.log 2>&1
timeout 400 python bench.py --config c5 --steps 50 --warmup 5 --no-cpu-baseline > gpurun_out/bench_c5.log 2>&1
