# GPU-box round trip: full GPU tests, smoke, bench lines for every config.
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo tests_rc=$? >> gpurun_out/gpu_tests.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 300 python bench.py > gpurun_out/bench_c2.log 2>&1
for c in ${CONFIGS:-c1 c3 c4 c5}; do timeout 400 python bench.py --config $c --steps 100 --warmup 10 --no-cpu-baseline > gpurun_out/bench_$c.log 2>&1; done
