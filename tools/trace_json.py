"""Chrome trace (chrome://tracing, Perfetto) of one DUET inference: per-subgraph start / end on the
device (duet_schedule_set_trace / duet_schedule_trace), one track per stream slot, and the check that
every partition edge u -> v has start(v) >= end(u) (the executor's dependency contract, §IV-D).

    python tools/trace_json.py c5 [out.json]
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

from paper_conf_ipps_zhanghl21_b200 import duet  # noqa: E402
from paper_conf_ipps_zhanghl21_b200 import workloads as W  # noqa: E402
from paper_conf_ipps_zhanghl21_b200.harness import Session, materialize  # noqa: E402


def trace_events(wl, sess, sched, start, end):
    ex = sess.part.export()
    names = [ln.split("=")[0].strip().lstrip("%") for ln in wl.ir.splitlines() if ln.startswith("%")]
    slot_of = sched.export()["slot_of"]
    ev = []
    for s in range(ex["n_sg"]):
        nodes = [names[i] for i, g in enumerate(ex["node_to_sg"]) if g == s and i < len(names)]
        label = nodes[0] if len(nodes) == 1 else f"{nodes[0]}..{nodes[-1]}" if nodes else f"sg{s}"
        ev.append({"name": f"sg{s} {label}", "ph": "X", "pid": 0, "tid": int(slot_of[s]), "ts": start[s] / 1e3,
                   "dur": max(0.0, (end[s] - start[s]) / 1e3), "args": {"phase": ex["sg_phase"][s]}})
    return ev


def violations(sess, start, end):
    """Partition edges u -> v (subgraphs) whose consumer started before its producer ended."""
    ex = sess.part.export()
    return [(u, v, int(start[v]), int(end[u])) for (u, v) in ex["edges"] if u >= 0 and v >= 0 and start[v] < end[u]]


def main():
    cfg = sys.argv[1] if len(sys.argv) > 1 else "c5"
    out = sys.argv[2] if len(sys.argv) > 2 else f"gpurun_out/trace_{cfg}.json"
    wl = W.build(cfg)
    sess = Session(wl, n_slots=2, profile=dict(warmup=2, samples=5, reps=2))
    sched = sess.schedule(duet.GREEDY_CORRECTION, measured=True, samples=10)
    inputs = list(materialize(wl.inputs, "cuda").values())
    outs = sess.outputs()
    sched.set_trace(True)
    for _ in range(3):
        sess.run(sched, inputs, outs)
    torch.cuda.synchronize()
    start, end = sched.trace()
    os.makedirs(os.path.dirname(out) or ".", exist_ok=True)
    with open(out, "w") as f:
        json.dump({"traceEvents": trace_events(wl, sess, sched, start, end), "displayTimeUnit": "ns"}, f)
    bad = violations(sess, start, end)
    print(f"{cfg}: {len(start)} subgraphs, makespan {max(end) / 1e3:.1f} us, dependency violations {len(bad)} -> {out}")
    if bad:
        sys.exit(1)


if __name__ == "__main__":
    main()
