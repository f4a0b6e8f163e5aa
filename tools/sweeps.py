"""Model-variation sweeps (the paper's §VI-D, Figs. 14-17).

The paper varies its Wide-and-Deep model (wide + FFN + RNN + CNN, Fig. 2 — our c4,
BASELINE.json:10): stacked RNN layers 1/2/4/8 (Fig. 14), ResNet depth 18/34/50/101 (Fig. 15), FFN
depth (Fig. 16) and batch size 2..32 (Fig. 17).  For each variant: partition -> device profile ->
greedy-correction schedule (Step 3 measured on the device) -> p50 latency of DUET (2 stream slots)
and of the serial 1-stream execution of the same kernels (the paper's single-device baseline),
CUDA events on the home stream, L2 flushed before every step (bench.py's `time_steps`).

  python tools/sweeps.py --out gpurun_out/sweeps.json [--only rnn,cnn,ffn,batch] [--steps 50]
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

SWEEPS = {
    "rnn": ("Fig. 14 stacked RNN layers", [dict(rnn_layers=n) for n in (1, 2, 4, 8)]),
    "cnn": ("Fig. 15 ResNet depth", [dict(resnet=d) for d in (18, 34, 50, 101)]),
    "ffn": ("Fig. 16 FFN depth", [dict(ffn_layers=n) for n in (1, 2, 4, 8)]),
    "batch": ("Fig. 17 batch size", [dict(batch=b) for b in (1, 2, 4, 8, 16, 32, 64)]),
}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--only", default="rnn,cnn,ffn,batch")
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--slots", type=int, default=2)
    ap.add_argument("--out", default="gpurun_out/sweeps.json")
    ap.add_argument("--rnn-tiles", type=int, default=1)
    args = ap.parse_args()
    import torch

    import bench
    from paper_conf_ipps_zhanghl21_b200 import duet
    from paper_conf_ipps_zhanghl21_b200 import workloads as W
    from paper_conf_ipps_zhanghl21_b200.harness import Session, materialize, tuned_session

    flush = torch.empty(bench.L2_FLUSH_BYTES // 4, dtype=torch.float32, device="cuda")
    res = {}
    for key in args.only.split(","):
        title, variants = SWEEPS[key]
        rows = []
        for var in variants:
            t0 = time.time()
            wl = W.build("c4", **var)
            popts = dict(warmup=3, samples=30, reps=5, calibrate_comm=True)
            if args.rnn_tiles:  # gate-tile width chosen by measured latency (bench.py's default)
                sess, duet_s, tile_ns, base = tuned_session(wl, n_slots=args.slots, profile=popts, samples=20)
            else:
                sess = base = Session(wl, n_slots=args.slots, profile=popts)
                tile_ns = None
            inputs = list(materialize(wl.inputs, "cuda").values())
            outs = sess.outputs()
            torch.cuda.synchronize()
            if not args.rnn_tiles:
                duet_s = sess.schedule(duet.GREEDY_CORRECTION, measured=True, samples=20)
            serial_s = base.schedule(duet.SERIAL)
            base.home.wait_stream(torch.cuda.current_stream())
            t_ser = bench.time_steps(torch, lambda: serial_s.run(base.slots, inputs, outs), base.home, args.steps,
                                     args.warmup, flush)
            torch.cuda.synchronize()
            t_duet = bench.time_steps(torch, lambda: duet_s.run(sess.slots, inputs, outs), sess.home, args.steps,
                                      args.warmup, flush)
            prof = sess.prof.export()["t_ns"][:, 0].tolist()
            e = duet_s.export()
            p50, p50s = statistics.median(t_duet), statistics.median(t_ser)
            r = {"variant": var, "batch": wl.batch, "n_sg": sess.part.n_sg, "p50_ms": round(p50, 4),
                 "p99_ms": round(bench.percentile(t_duet, 99), 4), "serial_p50_ms": round(p50s, 4),
                 "speedup_vs_serial": round(p50s / p50, 3), "samples_per_s": round(wl.batch / p50 * 1e3, 1),
                 "slot_of": e["slot_of"], "fell_back": e["fell_back"], "model_makespan_ms": e["makespan"] / 1e6,
                 "profile_ms": [round(v / 1e6, 4) for v in prof], "launches": duet_s.launch_count(),
                 "rnn_tile_n": sess.wl.meta.get("rnn_tile_n"), "rnn_tile_measured_ns": tile_ns,
                 "wall_s": round(time.time() - t0, 1)}
            print(json.dumps({key: r}), flush=True)
            rows.append(r)
            del sess, base, inputs, outs, duet_s, serial_s
            torch.cuda.empty_cache()
        res[key] = {"title": title, "rows": rows}
    os.makedirs(os.path.dirname(os.path.abspath(args.out)), exist_ok=True)
    with open(args.out, "w") as f:
        json.dump(res, f, indent=1)


if __name__ == "__main__":
    main()
