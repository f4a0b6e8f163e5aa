# GPU round trip for the per-consumer H2D copies: all GPU tests, e2e of every config, A/B on c4
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/h2d_tests.log 2>&1; echo tests_rc=$? >> gpurun_out/h2d_tests.log
timeout 300 python bench.py > gpurun_out/h2d_bench_c2.log 2>&1
for c in c1 c3 c4 c5 c6; do timeout 600 python bench.py --config $c --steps 100 --warmup 10 --no-cpu-baseline > gpurun_out/h2d_bench_$c.log 2>&1; done
