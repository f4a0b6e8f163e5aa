import sys, os, gc
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_zhanghl21_b200 import duet, workloads as W
from paper_conf_ipps_zhanghl21_b200.harness import Session, materialize
if len(sys.argv) > 1 and sys.argv[1] == "dirty":
    wl = W.build("c3")
    s = Session(wl, n_slots=2, profile=dict(warmup=1, samples=2, reps=2))
    ins = list(materialize(wl.inputs, "cuda").values()); outs = s.outputs()
    s.run(s.schedule(), ins, outs); torch.cuda.synchronize(); del s, ins, outs; gc.collect()
for (M, N, K) in [(802816, 64, 152), (4096, 64, 152), (2048, 256, 512)]:
    ir = (f"param @W : bf16[{N},{K}]\nparam @b : f32[{N}]\n%x = input() : bf16[{M},{K}]\n"
          f"%y = linear(%x, @W, @b) {{act=none}} : bf16[{M},{N}]\noutput %y\n")
    g = duet.Graph(ir)
    Wt = (torch.randn(N, K, device="cuda") * 0.1).bfloat16(); b = torch.zeros(N, device="cuda")
    g.bind_all({"W": Wt, "b": b})
    x = torch.randn(M, K, device="cuda").bfloat16()
    y = torch.empty(M, N, device="cuda", dtype=torch.bfloat16)
    g.node_run("y", [x], y); torch.cuda.synchronize()
    ref = x.float() @ Wt.float().T
    bad = (~torch.isfinite(y.float())).sum().item()
    err = ((y.float() - ref).abs().max() / ref.abs().max()).item()
    print(f"M={M} N={N} K={K} nonfinite={bad} err={err:.3e}", flush=True)
