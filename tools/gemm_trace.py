"""Per-CTA phase timeline of one pair-GEMM launch (DUET_GEMM_DBG=32 timestamps).
  python tools/gemm_trace.py M N K [bn]"""
import ctypes
import os
import sys

os.environ["DUET_GEMM_DBG"] = str(32 | int(os.environ.get("DBG", "0")))
if len(sys.argv) > 4:
    os.environ["DUET_GEMM_BN"] = sys.argv[4]
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

from paper_conf_ipps_zhanghl21_b200 import duet

M, N, K = (int(x) for x in sys.argv[1:4])
ir = (f"param @W : bf16[{N},{K}]\nparam @b : f32[{N}]\n%x = input() : bf16[{M},{K}]\n"
      f"%y = linear(%x, @W, @b) {{act=relu}} : bf16[{M},{N}]\noutput %y\n")
g = duet.Graph(ir)
g.bind_all({"W": (torch.randn(N, K, device="cuda") * 0.05).to(torch.bfloat16), "b": torch.zeros(N, device="cuda")})
x = torch.randn(M, K, device="cuda").to(torch.bfloat16)
y = torch.empty(M, N, device="cuda", dtype=torch.bfloat16)
s = torch.cuda.Stream()
lib = ctypes.CDLL(duet.LIB_PATH)
names = ["entry", "prologue", "first TMA", "first stage in", "last commit", "acc ready", "epi done", "exit",
         "tmem loaded", "smem staged", "store issued", "store read", "cluster sync", "pdl wait", "tmem alloc",
         "bias staged"]
for rep in range(4):
    g.node_run("y", [x], y, s)
    s.synchronize()
buf = (ctypes.c_ulonglong * (16 * 4096))()
lib.duet_debug_tc2_trace(buf, 16 * 4096)
a = np.frombuffer(buf, dtype=np.uint64).reshape(4096, 16).astype(np.int64)
ctas = a[a[:, 0] > 0]
t0 = ctas[:, 0].min()
try:
    import pynvml
    pynvml.nvmlInit()
    clk = pynvml.nvmlDeviceGetClockInfo(pynvml.nvmlDeviceGetHandleByIndex(0), pynvml.NVML_CLOCK_SM)
except Exception:
    clk = -1
print(f"M={M} N={N} K={K}: {len(ctas)} CTAs; sm clock {clk} MHz; times in ns relative to the first CTA entry")
print(f"{'phase':16s} {'min':>8s} {'median':>8s} {'max':>8s}")
for i, n in enumerate(names):
    v = ctas[:, i]
    v = v[v > 0] - t0
    if len(v):
        print(f"{n:16s} {v.min():8d} {int(np.median(v)):8d} {v.max():8d}")
lead = ctas[ctas[:, 3] > 0]
d = lambda i, j: lead[:, j] - lead[:, i]
print("per-CTA (leaders) medians: prologue %d, entry->first stage %d, mainloop %d, commit->acc %d, epilogue %d" % (
    np.median(ctas[:, 1] - ctas[:, 0]), np.median(d(0, 3)), np.median(d(3, 4)), np.median(d(4, 5)), np.median(d(5, 6))))
