# pair GEMM with / without A multicast (4-CTA clusters); one process per setting (env read once)
for mc in 0 1; do
DUET_GEMM_MC=$mc python - <<'PY'
import sys, os; sys.path.insert(0,'tools'); sys.path.insert(0,'.')
from gemm_micro import time_linear, sm_clock
mc = os.environ['DUET_GEMM_MC']
for bn in ("128", "256"):
    os.environ['DUET_GEMM_BN'] = bn
    for (M,N,K) in [(2048,1024,1664),(2048,512,1024),(16384,2048,256),(4096,4096,4096)]:
        ms,tf,err=time_linear(M,N,K)
        print(f"mc={mc} bn={bn:>3s} M={M} N={N} K={K} {ms*1e3:8.2f} us {tf:7.1f} TF/s err {err:.1e}", flush=True)
print('clk', sm_clock())
PY
done
