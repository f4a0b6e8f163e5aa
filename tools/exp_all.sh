mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q 2>&1 | tail -2 > gpurun_out/all_tests.log
timeout 500 python bench.py > gpurun_out/bench_c2.log 2>&1
for c in c1 c3 c4 c5; do timeout 400 python bench.py --config $c --steps 100 --warmup 10 --no-cpu-baseline > gpurun_out/bench_$c.log 2>&1; done
timeout 1200 python tools/fig13.py --configs c1,c2,c3,c4,c5 --out gpurun_out/fig13.json > gpurun_out/fig13.log 2>&1
