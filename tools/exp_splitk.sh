mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "linear_node or c6 or small_parity or variation" > gpurun_out/splitk_tests.log 2>&1; echo rc=$? >> gpurun_out/splitk_tests.log
timeout 300 python bench.py --config c6 --steps 100 --warmup 10 --no-cpu-baseline > gpurun_out/bench_c6_splitk.log 2>&1
DUET_SPLITK=0 timeout 300 python bench.py --config c6 --steps 100 --warmup 10 --no-cpu-baseline > gpurun_out/bench_c6_nosplit.log 2>&1
python tools/node_times.py c6 > gpurun_out/node_times_c6_splitk.log 2>&1
timeout 300 python bench.py --config c4 --steps 100 --warmup 10 --no-cpu-baseline > gpurun_out/bench_c4_splitk.log 2>&1
timeout 300 python bench.py --config c1 --steps 200 --warmup 10 --no-cpu-baseline > gpurun_out/bench_c1_splitk.log 2>&1
