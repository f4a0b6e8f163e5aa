mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "linear_node or small_parity or c2_full" > gpurun_out/wpf_tests.log 2>&1; echo rc=$? >> gpurun_out/wpf_tests.log
for i in 1 2; do
timeout 300 python bench.py --config c2 --steps 300 --warmup 20 --no-cpu-baseline > gpurun_out/bench_wpf1_$i.log 2>&1
DUET_GEMM_WPF=0 timeout 300 python bench.py --config c2 --steps 300 --warmup 20 --no-cpu-baseline > gpurun_out/bench_wpf0_$i.log 2>&1
done
