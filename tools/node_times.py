"""Per-node kernel times of a config (real intermediates; CUDA-graph replays of node_run).

  python tools/node_times.py c2 [--flush] [--dt f32]

Every node is made a graph output so one serial duet_run materialises all intermediates; then
each node is timed alone: a CUDA graph of `iters` back-to-back duet_node_run launches, replayed
`replays` times between CUDA events (optionally with an L2 flush before each replay).
"""
from __future__ import annotations

import argparse
import os
import re
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("config")
    ap.add_argument("--small", action="store_true")
    ap.add_argument("--dt", default=None, choices=[None, "bf16", "f32"])
    ap.add_argument("--iters", type=int, default=20)
    ap.add_argument("--replays", type=int, default=20)
    ap.add_argument("--flush", action="store_true", help="flush L2 before every replay (1 launch per replay)")
    args = ap.parse_args()
    import torch

    from paper_conf_ipps_zhanghl21_b200 import duet
    from paper_conf_ipps_zhanghl21_b200 import workloads as W
    from paper_conf_ipps_zhanghl21_b200.harness import materialize

    wl = W.build(args.config, small=args.small, dt=args.dt)
    decl = {}
    for line in wl.ir.splitlines():
        m = re.match(r"%(\w+) = (\w+)\((.*?)\).*: (\w+)\[([\d,]*)\]", line)
        if m:
            name, op, a, dt, shape = m.groups()
            decl[name] = (op, [x.strip()[1:] for x in a.split(",") if x.strip().startswith("%")], dt,
                          [int(v) for v in shape.split(",") if v])
    nodes = [n for n, d in decl.items() if d[0] != "input"]
    ir = "\n".join(l for l in wl.ir.splitlines() if not l.startswith("output")) + "\noutput " + \
        ", ".join("%" + n for n in nodes) + "\n"
    g = duet.Graph(ir)
    params = materialize(wl.params, "cuda")
    g.bind_all(params)
    part = g.partition()
    st = torch.cuda.Stream()
    prof = part.profile_from_table([0], [[1]] * part.n_sg)
    s = prof.schedule(mode=duet.SERIAL)
    tdt = {"f32": torch.float32, "bf16": torch.bfloat16, "i32": torch.int32, "i64": torch.int64}
    inputs = materialize(wl.inputs, "cuda")
    outs = {n: torch.empty(decl[n][3], dtype=tdt[decl[n][2]], device="cuda") for n in nodes}
    torch.cuda.synchronize()
    s.run([(0, st)], list(inputs.values()), [outs[n] for n in nodes])
    st.synchronize()
    vals = dict(inputs)
    vals.update(outs)
    flush = torch.empty(512 << 18, dtype=torch.float32, device="cuda") if args.flush else None
    total = 0.0
    print(f"{'node':24s} {'op':14s} {'us/launch':>10s}")
    for n in nodes:
        op, a, dt, shape = decl[n]
        y = torch.empty_like(outs[n])
        argv = [vals[x] for x in a]
        iters = 1 if args.flush else args.iters
        with torch.cuda.stream(st):
            gr = torch.cuda.CUDAGraph()
            for _ in range(2):
                g.node_run(n, argv, y, st)
            st.synchronize()
            with torch.cuda.graph(gr, stream=st):
                for _ in range(iters):
                    g.node_run(n, argv, y, torch.cuda.current_stream())
            times = []
            for _ in range(args.replays):
                if flush is not None:
                    flush.zero_()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(st)
                gr.replay()
                e1.record(st)
                st.synchronize()
                times.append(e0.elapsed_time(e1) * 1e3 / iters)
        us = statistics.median(times)
        total += us
        print(f"{n:24s} {op:14s} {us:10.2f}")
    print(f"{'sum':24s} {'':14s} {total:10.2f}")


if __name__ == "__main__":
    main()
