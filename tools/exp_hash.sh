mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/hash_tests.log 2>&1; echo rc=$? >> gpurun_out/hash_tests.log
for i in 1 2; do
timeout 300 python bench.py --config c2 --steps 300 --warmup 20 --no-cpu-baseline > gpurun_out/bench_hash_c2_$i.log 2>&1
DUET_HASH_FUSE=0 timeout 300 python bench.py --config c2 --steps 300 --warmup 20 --no-cpu-baseline > gpurun_out/bench_hash_c2_off_$i.log 2>&1
done
timeout 300 python bench.py --config c1 --steps 300 --warmup 20 --no-cpu-baseline > gpurun_out/bench_hash_c1.log 2>&1
DUET_HASH_FUSE=0 timeout 300 python bench.py --config c1 --steps 300 --warmup 20 --no-cpu-baseline > gpurun_out/bench_hash_c1_off.log 2>&1
