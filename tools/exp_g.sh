timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
timeout 300 python tools/node_times.py c2 > gpurun_out/nodes_c2.log 2>&1
timeout 300 python tools/node_times.py c2 --flush > gpurun_out/nodes_c2_flush.log 2>&1
timeout 400 python bench.py --no-cpu-baseline > gpurun_out/bench_c2.log 2>&1
