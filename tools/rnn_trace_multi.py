"""Per-step phase timeline of the several-tiles-per-CTA recurrence (DUET_RNN_DBG=1 stamps).
  python tools/rnn_trace_multi.py lstm|gru B H E S   (S * tiles per CTA <= 64 units are stamped)"""
import ctypes
import os
import sys

os.environ["DUET_RNN_DBG"] = "1"
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
lib = ctypes.CDLL(duet.LIB_PATH)
buf = (ctypes.c_ulonglong * (128 * 64 * 16))()
lib.duet_debug_rp_trace(buf, 128 * 64 * 16)
a = np.frombuffer(buf, dtype=np.uint64).reshape(128, 64, 16).astype(np.int64)
names = {7: "first A load", 11: "first W load", 1: "first stage in", 4: "first h stage in", 5: "last UMMA",
         2: "acc ready", 6: "TMEM read", 3: "released"}
for mt in (1, 2, 3, 4):
    ctas = [c for c in range(128) if (a[c, :, 1] > 0).sum() == min(64, S * mt)]
    if not ctas:
        continue
    rows = {key: [[] for _ in range(mt)] for key in names}
    steps = []
    for c in ctas:
        for t in range(2, min(S, 64 // mt) - 1):
            b0 = a[c, t * mt, 0]
            b1 = a[c, (t + 1) * mt, 0] if (t + 1) * mt < 64 else 0
            if b0 <= 0:
                continue
            if b1 > 0:
                steps.append(b1 - b0)
            for i in range(mt):
                for key in names:
                    v = a[c, t * mt + i, key]
                    if v > 0:
                        rows[key][i].append(v - b0)
    print(f"{kind} B{B} H{H} E{E} S{S}: {len(ctas)} traced CTAs with {mt} tile(s); step (barrier to barrier) "
          f"median {np.median(steps) if steps else float('nan'):.0f} ns")
    for key, nm in names.items():
        print(f"  {nm:18s} " + "  ".join(f"tile{i}: {np.median(rows[key][i]) if rows[key][i] else float('nan'):8.0f}"
                                         for i in range(mt)))
