for d in 0 1 2 3 4; do
  echo "== DUET_GEMM_DBG=$d"
  DUET_GEMM_DBG=$d python - <<'PY'
import sys; sys.path.insert(0,'tools'); sys.path.insert(0,'.')
from gemm_micro import time_linear, warm, sm_clock
warm(1.0); print('clk', sm_clock())
for (M,N,K) in [(128,64,6400),(128,256,6400),(2048,1024,1664)]:
    ms,tf,err=time_linear(M,N,K)
    print(f"M={M} N={N} K={K} {ms*1e3:8.2f} us {tf:7.1f} TF/s err {err:.1e}", flush=True)
PY
done
