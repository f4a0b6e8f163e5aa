timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
timeout 120 python tools/chain_trace.py 2048 1664 1024 512 256 2>&1| head -4
python tools/gemm_micro.py 2>&1 | sed -n '7,9p'
for c in c2 c4 c5; do timeout 400 python bench.py --config $c --steps 100 --warmup 10 --no-cpu-baseline > gpurun_out/bench_$c.log 2>&1; done
DUET_MLP_CHAIN=0 timeout 400 python bench.py --config c2 --steps 100 --warmup 10 --no-cpu-baseline > gpurun_out/bench_c2_nochain.log 2>&1
