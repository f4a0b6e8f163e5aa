"""Per-node kernel times of a workload (CUDA-graph timed node_run), to find hot spots."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_zhanghl21_b200 import workloads as W, duet
from paper_conf_ipps_zhanghl21_b200.harness import materialize
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from gemm_micro import warm
from oracle.ir import parse  # structure only (names/shapes) for the tool

cfg = sys.argv[1] if len(sys.argv) > 1 else "c4"
wl = W.build(cfg)
params = materialize(wl.params, "cuda")
g = duet.Graph(wl.ir)
g.bind_all(params)
ir = parse(wl.ir)
TD = {"f32": torch.float32, "bf16": torch.bfloat16, "i32": torch.int32, "i64": torch.int64}
bufs = {}
inputs = materialize(wl.inputs, "cuda")
for n in ir.nodes:
    if n.op == "input":
        bufs[n.name] = inputs[n.name]
    else:
        bufs[n.name] = torch.zeros(n.shape, dtype=TD[n.dtype], device="cuda")
warm(0.5)
s = torch.cuda.Stream()
tot = 0.0
rows = []
for n in ir.nodes:
    if n.op == "input":
        continue
    args = [bufs[ir.nodes[i].name] for i in [ir.by_name[nm] for k, nm in n.args if k == "%"]]
    try:
        g.node_run(n.name, args, bufs[n.name], s)
    except duet.DuetError as e:
        continue
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record(s)
    for _ in range(10):
        g.node_run(n.name, args, bufs[n.name], s)
    e1.record(s)
    torch.cuda.synchronize()
    us = e0.elapsed_time(e1) / 10 * 1e3
    tot += us
    rows.append((us, n.name, n.op, n.shape))
for us, name, op, shape in rows:
    print(f"{us:9.1f} us  {name:24s} {op:12s} {shape}")
print(f"total {tot:.1f} us")
