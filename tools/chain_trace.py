"""Per-item timeline of the persistent MLP chain (DUET_CHAIN_DBG=1).
  python tools/chain_trace.py M K N1 N2 ..."""
import ctypes
import os
import sys

os.environ["DUET_CHAIN_DBG"] = str(1 | int(os.environ.get("DBG", "0")))
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

from paper_conf_ipps_zhanghl21_b200 import duet

M, K = int(sys.argv[1]), int(sys.argv[2])
Ns = [int(x) for x in sys.argv[3:]]
lines, prev, binds = [f"%x = input() : bf16[{M},{K}]"], ("x", K), {}
for i, n in enumerate(Ns):
    lines = [f"param @W{i} : bf16[{n},{prev[1]}]", f"param @b{i} : f32[{n}]"] + lines
    lines.append(f"%y{i} = linear(%{prev[0]}, @W{i}, @b{i}) {{act=relu}} : bf16[{M},{n}]")
    binds[f"W{i}"] = (torch.randn(n, prev[1], device="cuda") / prev[1] ** 0.5).to(torch.bfloat16)
    binds[f"b{i}"] = torch.zeros(n, device="cuda")
    prev = (f"y{i}", n)
ir = "\n".join(lines + [f"output %{prev[0]}"]) + "\n"
g = duet.Graph(ir)
g.bind_all(binds)
part = g.partition()
prof = part.profile_from_table([0], [[1000]])
s = prof.schedule()
x = torch.randn(M, K, device="cuda").to(torch.bfloat16)
y = torch.empty(M, Ns[-1], device="cuda", dtype=torch.bfloat16)
st = torch.cuda.Stream()
slots = [(0, st)]
for _ in range(3):
    s.run(slots, [x], [y])
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
e0.record(st)
s.run(slots, [x], [y])
e1.record(st)
torch.cuda.synchronize()
ref = x.float()
for i in range(len(Ns)):
    ref = torch.relu(ref @ binds[f"W{i}"].float().T).to(torch.bfloat16).float()
err = (y.float() - ref).abs().max().item() / ref.abs().max().item()
print(f"M={M} K={K} N={Ns}: step {e0.elapsed_time(e1) * 1e3:.1f} us, rel err {err:.2e}")
lib = ctypes.CDLL(duet.LIB_PATH)
buf = (ctypes.c_ulonglong * (296 * 64))()
lib.duet_debug_chain_trace(buf, 296 * 64)
a = np.frombuffer(buf, dtype=np.uint64).reshape(296, 4, 16).astype(np.int64)
live = a[:, 0, 0] > 0
a = a[live]
t0 = a[:, 0, 0].min()
rel = np.where(a > 0, a - t0, -1)
print("cta: [entry] per item: dep-ok first-stage last-umma acc-ready tmem-read act-done staging-free written fenced released")
for c in range(0, min(len(a), 4)):
    row = [f"{rel[c, 0, 0]:6d} |"]
    for it in range(4):
        if rel[c, it, 3] < 0 and rel[c, it, 4] < 0:
            continue
        row.append(" ".join(f"{rel[c, it, k]:6d}" for k in (1, 2, 3, 4, 6, 8, 9, 10, 7, 5)) + " |")
    print(f"{c // 2:3d} " + " ".join(row))
