mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "linear_node or small_parity or c2_full" > gpurun_out/fc1c_tests.log 2>&1; echo rc=$? >> gpurun_out/fc1c_tests.log
python tools/gemm_trace.py 2048 1024 1664 > gpurun_out/trace_fc1c.log 2>&1
for e in 1 0; do DUET_GEMM_EARLY_A=$e python - <<'PY' > gpurun_out/exp_fc1c_e$e.log 2>&1
import sys
sys.path.insert(0, "tools"); sys.path.insert(0, ".")
from gemm_micro import time_linear, warm
warm(1.0)
for M, N, K in [(2048, 1024, 1664), (2048, 512, 1024), (2048, 256, 512), (4096, 1024, 1664)]:
    ms, tf, err = time_linear(M, N, K)
    print(f"{M}x{N}x{K} {ms*1e3:8.2f} us {tf:7.1f} TFLOP/s err {err:.1e}")
PY
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gemm2_kernel -s 3 -c 1 -o gpurun_out/fc1c python tools/gemm_micro_one.py 2048 1024 1664 > gpurun_out/ncu_fc1c.log 2>&1
ncu -i gpurun_out/fc1c.ncu-rep --page source --csv --print-source sass > gpurun_out/fc1c_sass.csv 2>/dev/null
ncu -i gpurun_out/fc1c.ncu-rep --page raw --csv > gpurun_out/fc1c_raw.csv 2>/dev/null
