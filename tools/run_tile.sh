mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "tile_n or variation or c4" -s > gpurun_out/tile_tests.log 2>&1; echo tests_rc=$? >> gpurun_out/tile_tests.log
for i in 1 2; do timeout 400 python bench.py --config c4 --steps 200 --warmup 10 --no-cpu-baseline > gpurun_out/tile_bench_c4_$i.log 2>&1; done
timeout 1500 python tools/sweeps.py --out gpurun_out/sweeps_tile.json > gpurun_out/sweeps_tile.log 2>&1; echo sweeps_rc=$? >> gpurun_out/sweeps_tile.log
