mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "measured or small_parity" > gpurun_out/relabel_tests.log 2>&1; echo rc=$? >> gpurun_out/relabel_tests.log
for i in 1 2; do timeout 300 python bench.py --config c2 --steps 300 --warmup 20 --no-cpu-baseline > gpurun_out/bench_rl_c2_$i.log 2>&1; done
for c in c1 c3 c4 c5 c6; do timeout 400 python bench.py --config $c --steps 100 --warmup 10 --no-cpu-baseline > gpurun_out/bench_rl_$c.log 2>&1; done
