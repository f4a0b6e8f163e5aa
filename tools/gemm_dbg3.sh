# Component costs of the pair GEMM on the c2 shapes: dbg 1 = skip MMA, 2 = skip TMA, 8 = skip
# epilogue, 9 = TMA only, 10 = MMA only (no TMA, no epilogue).
python - <<'PY'
import sys, os; sys.path.insert(0,'tools'); sys.path.insert(0,'.')
from gemm_micro import time_linear, warm, sm_clock
warm(1.0); print('clk', sm_clock())
for d in (0,1,2,8,9,10):
    os.environ['DUET_GEMM_DBG']=str(d)
    for (M,N,K) in [(2048,1024,1664),(2048,512,1024),(2048,256,512),(16384,2048,256)]:
        ms,tf,err=time_linear(M,N,K)
        print(f"dbg={d:2d} M={M} N={N} K={K} {ms*1e3:8.2f} us {tf:7.1f} TF/s", flush=True)
PY
