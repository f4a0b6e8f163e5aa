# fc1 decomposition on the GPU box: env knobs read once per process, so one process per setting.
mkdir -p gpurun_out
run() {  # label env...
  local label=$1; shift
  env "$@" python - <<'PY' 2>&1 | sed "s/^/$label /"
import sys, os
sys.path.insert(0, "tools"); sys.path.insert(0, ".")
from gemm_micro import time_linear, warm
warm(0.5)
for M, N, K in [(2048, 1024, 1664), (2048, 512, 1024), (2048, 256, 512), (4096, 1024, 1664)]:
    ms, tf, err = time_linear(M, N, K)
    print(f"{M}x{N}x{K} {ms*1e3:8.2f} us {tf:7.1f} TFLOP/s err {err:.1e}")
PY
}
{
run base DUET_GEMM_DBG=0
run noMMA DUET_GEMM_DBG=1
run noTMA DUET_GEMM_DBG=2
run noEPI DUET_GEMM_DBG=8
run noMMA_noEPI DUET_GEMM_DBG=9
run noTMA_noEPI DUET_GEMM_DBG=10
run bn64 DUET_GEMM_BN=64
run bn256 DUET_GEMM_BN=256
run mc2 DUET_GEMM_MC=2
run mc4 DUET_GEMM_MC=4
run mc4_noMMA DUET_GEMM_MC=4 DUET_GEMM_DBG=9
run nopdl DUET_NO_PDL=1
} > gpurun_out/exp_fc1.log 2>&1
python tools/gemm_trace.py 2048 1024 1664 > gpurun_out/trace_fc1.log 2>&1
DBG=8 python tools/gemm_trace.py 2048 1024 1664 > gpurun_out/trace_fc1_noepi.log 2>&1
