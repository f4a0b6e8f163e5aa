mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "gather_fused or small_parity or c2_full or full_size or host_buffers or measured" > gpurun_out/gf_tests.log 2>&1; echo rc=$? >> gpurun_out/gf_tests.log
timeout 300 python bench.py --config c2 --steps 300 --warmup 20 --no-cpu-baseline > gpurun_out/bench_gf_c2.log 2>&1
DUET_GATHER_FUSE=0 timeout 300 python bench.py --config c2 --steps 300 --warmup 20 --no-cpu-baseline > gpurun_out/bench_gf_c2_off.log 2>&1
timeout 300 python bench.py --config c5 --steps 50 --warmup 5 --no-cpu-baseline > gpurun_out/bench_gf_c5.log 2>&1
