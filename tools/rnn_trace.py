"""Per-step phase timeline of the persistent recurrence (DUET_RNN_DBG=1 timestamps).
  python tools/rnn_trace.py lstm|gru B H E S [bn]"""
import ctypes
import os
import sys

os.environ["DUET_RNN_DBG"] = str(1 | int(os.environ.get("DBG", "0")))
if len(sys.argv) > 6:
    os.environ["DUET_RNN_BN"] = sys.argv[6]
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

from paper_conf_ipps_zhanghl21_b200 import duet

kind = sys.argv[1]
B, H, E, S = (int(x) for x in sys.argv[2:6])
G = 4 if kind == "lstm" else 3
ir = (f"param @Wih : bf16[{G * H},{E}]\nparam @Whh : bf16[{G * H},{H}]\nparam @bih : f32[{G * H}]\n"
      f"param @bhh : f32[{G * H}]\n%x = input() : bf16[{S},{B},{E}]\n"
      f"%y = {kind}(%x, @Wih, @Whh, @bih, @bhh) : bf16[{B},{H}]\noutput %y\n")
g = duet.Graph(ir)
k = 1.0 / H ** 0.5
g.bind_all({"Wih": ((torch.rand(G * H, E, device="cuda") * 2 - 1) * k).to(torch.bfloat16),
            "Whh": ((torch.rand(G * H, H, device="cuda") * 2 - 1) * k).to(torch.bfloat16),
            "bih": torch.zeros(G * H, device="cuda"), "bhh": torch.zeros(G * H, device="cuda")})
x = torch.randn(S, B, E, device="cuda").to(torch.bfloat16)
y = torch.empty(B, H, device="cuda", dtype=torch.bfloat16)
st = torch.cuda.Stream()
for _ in range(3):
    g.node_run("y", [x], y, st)
st.synchronize()
e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
e0.record(st)
g.node_run("y", [x], y, st)
e1.record(st)
st.synchronize()
lib = ctypes.CDLL(duet.LIB_PATH)
buf = (ctypes.c_ulonglong * (128 * 64 * 16))()
lib.duet_debug_rp_trace(buf, 128 * 64 * 16)
a = np.frombuffer(buf, dtype=np.uint64).reshape(128, 64, 16).astype(np.int64)
live = a[:, 1, 2] > 0
a = a[live]
t0 = a[a > 0].min()
print(f"{kind} B={B} H={H} E={E} S={S}: {live.sum()} CTAs, kernel {e0.elapsed_time(e1) * 1e3:.1f} us "
      f"({e0.elapsed_time(e1) * 1e3 / S:.2f} us/step)")
rel = np.where(a > 0, a - t0, -1)
print("step  barrier(min/med/max)   x-landed(med)  acc-ready(min/med/max)  released(min/med/max)")
for t in range(min(S, 64)):
    r = rel[:, t, :]
    def mm(c):
        v = r[:, c][r[:, c] >= 0]
        return (v.min(), int(np.median(v)), v.max()) if len(v) else (-1, -1, -1)
    b, xl, ac, rl = mm(0), mm(1), mm(2), mm(3)
    if t < 6 or t % 8 == 0 or t == S - 1:
        print(f"{t:4d}  {b[0]:7d} {b[1]:7d} {b[2]:7d}  {xl[1]:9d}  {ac[0]:7d} {ac[1]:7d} {ac[2]:7d}  {rl[0]:7d} {rl[1]:7d} {rl[2]:7d}")
st_ = [np.median(rel[:, t, 3] - rel[:, t - 1, 3]) for t in range(2, min(S - 1, 64))]
print("median per-step period (release to release):", np.median(st_))
print("median barrier->acc-ready:", np.median([np.median(rel[:, t, 2] - rel[:, t, 0]) for t in range(1, min(S, 64))]),
      " acc-ready->released:", np.median([np.median(rel[:, t, 3] - rel[:, t, 2]) for t in range(0, min(S - 1, 64))]),
      " last release -> barrier pass:", np.median([np.median(rel[:, t, 0] - rel[:, t - 1, 3].max()) for t in range(1, min(S, 64))]))

def med(c0, c1, lo=1):
    return np.median([np.median(rel[:, t, c1] - rel[:, t, c0]) for t in range(lo, min(S - 1, 64))])
print("medians: barrier->first h landed %d, h landed->last UMMA issued %d, last UMMA->acc ready %d, "
      "acc ready->released %d" % (med(0, 4), med(4, 5), med(5, 2), med(2, 3)))
print("epilogue: acc ready->TMEM read %d, ->bar.sync passed %d, ->released %d" % (med(2, 6, 0), med(6, 7, 0), med(7, 3, 0)))
print("per-warp math+stores done after acc ready (warps 2..9):", [int(med(2, 8 + w, 0)) for w in range(8)])
