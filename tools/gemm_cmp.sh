python - <<'PY'
import sys, os; sys.path.insert(0,'tools'); sys.path.insert(0,'.')
from gemm_micro import time_linear, warm, sm_clock
warm(1.0); print('clk', sm_clock())
shapes=[(2048,1024,1664),(2048,512,1024),(2048,256,512),(4096,1024,1664),(4096,2048,512),(16384,2048,256),(300,136,320),(513,272,200),(4096,4096,4096),(8192,8192,8192)]
for (M,N,K) in shapes:
    for bn in (None, 64, 128, 256):
        if bn: os.environ['DUET_GEMM_BN']=str(bn)
        else: os.environ.pop('DUET_GEMM_BN',None)
        try:
            ms,tf,err=time_linear(M,N,K)
            print(f"M={M} N={N} K={K} bn={bn} {ms*1e3:8.2f} us {tf:7.1f} TF/s err {err:.1e}", flush=True)
        except Exception as e:
            print(f"M={M} N={N} K={K} bn={bn} ERROR {e}", flush=True)
PY
