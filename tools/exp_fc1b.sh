mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "linear_node or small_parity or c2_full" > gpurun_out/fc1b_tests.log 2>&1; echo rc=$? >> gpurun_out/fc1b_tests.log
run() {  # label env...
  local label=$1; shift
  env "$@" python - <<'PY' 2>&1 | sed "s/^/$label /"
import sys, os
sys.path.insert(0, "tools"); sys.path.insert(0, ".")
from gemm_micro import time_linear, warm
warm(1.0)
for M, N, K in [(2048, 1024, 1664), (2048, 512, 1024), (2048, 256, 512), (4096, 1024, 1664)]:
    ms, tf, err = time_linear(M, N, K)
    print(f"{M}x{N}x{K} {ms*1e3:8.2f} us {tf:7.1f} TFLOP/s err {err:.1e}")
PY
}
{
run early1 DUET_GEMM_EARLY_A=1
run early0 DUET_GEMM_EARLY_A=0
run early1 DUET_GEMM_EARLY_A=1
run early0 DUET_GEMM_EARLY_A=0
} > gpurun_out/exp_fc1b.log 2>&1
python tools/gemm_trace.py 2048 1024 1664 > gpurun_out/trace_fc1b.log 2>&1
DUET_GEMM_EARLY_A=0 python tools/gemm_trace.py 2048 1024 1664 > gpurun_out/trace_fc1b_e0.log 2>&1
for c in c2; do timeout 300 python bench.py --config $c --steps 200 --warmup 10 --no-cpu-baseline > gpurun_out/bench_fc1b_$c.log 2>&1; done
DUET_GEMM_EARLY_A=0 timeout 300 python bench.py --config c2 --steps 200 --warmup 10 --no-cpu-baseline > gpurun_out/bench_fc1b_c2_e0.log 2>&1
