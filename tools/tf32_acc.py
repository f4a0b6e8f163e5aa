"""3xTF32 accumulator-split experiment: error of one fp32 linear node vs the float64 oracle for
DUET_GEMM_DBG settings (gemm_tf32.cu: dbg & 7 = big accumulators, dbg & 8 = cross terms share
them), each in a fresh process (the switch is read when the node is built).
  python tools/tf32_acc.py M N K bn dbg..."""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CHILD = r'''
import sys, numpy as np, torch
sys.path.insert(0, sys.argv[1])
from oracle import forward as OF
from paper_conf_ipps_zhanghl21_b200 import duet
from tests.helpers import rel_err, l2_rel_err
M, N, K = map(int, sys.argv[2:5])
ir = (f"param @W : f32[{N},{K}]\nparam @b : f32[{N}]\n%x = input() : f32[{M},{K}]\n"
      f"%y = linear(%x, @W, @b) {{act=relu}} : f32[{M},{N}]\noutput %y\n")
g_ = torch.Generator().manual_seed(1)
x = ((torch.rand(M, K, generator=g_, dtype=torch.float64) * 2 - 1)).float()
W = ((torch.rand(N, K, generator=g_, dtype=torch.float64) * 2 - 1) / K ** 0.5).float()
b = ((torch.rand(N, generator=g_, dtype=torch.float64) * 2 - 1) * 0.1).float()
g = duet.Graph(ir)
g.bind_all({"W": W.cuda(), "b": b.cuda()})
y = torch.empty(M, N, device="cuda")
g.node_run("y", [x.cuda()], y)
torch.cuda.synchronize()
want = OF.linear(x.double().numpy(), W.double().numpy(), b.double().numpy(), "relu")
simt = torch.relu(x.double() @ W.double().T + b.double()).float()  # fp64 rounded once: the floor
print(f"rel {rel_err(y.cpu().numpy(), want):.3e} l2 {l2_rel_err(y.cpu().numpy(), want):.3e}")
'''
M, N, K, bn = sys.argv[1:5]
for dbg in sys.argv[5:]:
    env = dict(os.environ, DUET_GEMM_DBG=dbg, DUET_GEMM_BN=bn)
    r = subprocess.run([sys.executable, "-c", CHILD, ROOT, M, N, K], env=env, capture_output=True, text=True)
    print(f"M{M} N{N} K{K} bn{bn} dbg {dbg}: {r.stdout.strip()} {r.stderr.strip()[-300:]}", flush=True)
