python - <<'PY'
import sys, os; sys.path.insert(0,'tools'); sys.path.insert(0,'.')
from gemm_micro import time_linear, warm, sm_clock
warm(1.0); print('clk', sm_clock())
for d in (0,1,2,8,9):
    os.environ['DUET_GEMM_DBG']=str(d)
    for (M,N,K,bn) in [(2048,1024,1664,128),(2048,1024,1664,256),(4096,4096,4096,256),(256,256,6400,256)]:
        os.environ['DUET_GEMM_BN']=str(bn)
        ms,tf,err=time_linear(M,N,K)
        print(f"dbg={d} M={M} N={N} K={K} bn={bn} {ms*1e3:8.2f} us {tf:7.1f} TF/s", flush=True)
PY
