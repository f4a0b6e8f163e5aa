"""Scheduler comparison (the paper's Fig. 13).

For each config: profile on the device, then for every scheduler report the model makespan
(C3, from the profile) and the measured p50 latency of its assignment on the B200 (CUDA events
on the home stream, inputs resident, L2 warm).  Schedulers: Random (mean over seeds),
Round-Robin, Random+Correction (mean over seeds), Greedy (Steps 1-2), Greedy+Correction (model
Step 3), Greedy+Correction measured (device Step 3), serial, and Ideal (exhaustive over the model
when D^n_sg <= 4096, its assignment measured).  Fallback is disabled so each scheduler's own
placement is what runs.

  python tools/fig13.py --configs c1,c2,c3,c4,c5 --out gpurun_out/fig13.json
"""
from __future__ import annotations

import argparse
import itertools
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="c1,c2,c3,c4,c5")
    ap.add_argument("--slots", type=int, default=2)
    ap.add_argument("--seeds", type=int, default=8)
    ap.add_argument("--reps", type=int, default=50)
    ap.add_argument("--out", default="gpurun_out/fig13.json")
    args = ap.parse_args()
    import faulthandler
    faulthandler.dump_traceback_later(int(os.environ.get("FIG13_STACK_AFTER", "0")) or 10 ** 6, repeat=True)
    import torch

    from paper_conf_ipps_zhanghl21_b200 import duet
    from paper_conf_ipps_zhanghl21_b200 import workloads as W
    from paper_conf_ipps_zhanghl21_b200.harness import Session, materialize

    res = {}
    for cfg in args.configs.split(","):
        wl = W.build(cfg)
        sess = Session(wl, n_slots=args.slots, profile=dict(warmup=5, samples=50, reps=10, calibrate_comm=True))
        inputs = list(materialize(wl.inputs, "cuda").values())
        outs = sess.outputs()
        torch.cuda.synchronize()
        home = sess.home
        n = sess.part.n_sg
        D = args.slots
        memo = {}

        def measure(a):
            a = tuple(a)
            if a in memo:
                return memo[a]
            s = sess.prof.schedule(mode=duet.FIXED, fixed=list(a))
            for _ in range(5):
                s.run(sess.slots, inputs, outs)
            ev = [torch.cuda.Event(enable_timing=True) for _ in range(args.reps + 1)]
            ev[0].record(home)
            for k in range(args.reps):
                s.run(sess.slots, inputs, outs)
                ev[k + 1].record(home)
            home.synchronize()
            ms = sorted(ev[k].elapsed_time(ev[k + 1]) for k in range(args.reps))
            memo[a] = ms[(len(ms) - 1) // 2]
            return memo[a]

        def row(scheds):
            mk = [s.export()["makespan"] / 1e6 for s in scheds]
            me = [measure(s.export()["slot_of"]) for s in scheds]
            return {"model_ms": round(statistics.mean(mk), 5), "measured_ms": round(statistics.mean(me), 5),
                    "slot_of": scheds[0].export()["slot_of"] if len(scheds) == 1 else None}

        P = sess.prof
        r = {"n_sg": n}
        import time
        t0 = time.time()

        def note(k):
            print(f"  {cfg} {k}: {json.dumps(r.get(k))} ({time.time() - t0:.1f}s, {len(memo)} measured)", flush=True)

        r["serial"] = row([P.schedule(mode=duet.SERIAL)])
        note("serial")
        r["random"] = row([P.schedule(mode=duet.RANDOM, seed=k, allow_fallback=False) for k in range(args.seeds)])
        note("random")
        r["round_robin"] = row([P.schedule(mode=duet.ROUND_ROBIN, allow_fallback=False)])
        note("round_robin")
        r["random_correction"] = row([P.schedule(mode=duet.RANDOM_CORRECTION, seed=k, allow_fallback=False)
                                      for k in range(args.seeds)])
        note("random_correction")
        r["greedy"] = row([P.schedule(mode=duet.GREEDY_ONLY, allow_fallback=False)])
        note("greedy")
        r["greedy_correction"] = row([P.schedule(mode=duet.GREEDY_CORRECTION, allow_fallback=False)])
        note("greedy_correction")
        sm = P.schedule_measured(sess.slots, mode=duet.GREEDY_CORRECTION, allow_fallback=False, samples=20)
        r["greedy_correction_measured"] = row([sm])
        r["greedy_correction_measured"]["evaluations"] = sm.evaluations
        note("greedy_correction_measured")
        if D ** n <= 4096:
            best = None
            for a in itertools.product(range(D), repeat=n):
                ms = P.schedule(mode=duet.FIXED, fixed=list(a)).export()["makespan"]
                if best is None or ms < best[0]:
                    best = (ms, list(a))
            r["ideal_model"] = row([P.schedule(mode=duet.FIXED, fixed=best[1])])
            note("ideal_model")
            if D ** n <= 256:  # exhaustive over the device too
                meas = {tuple(a): measure(a) for a in itertools.product(range(D), repeat=n)}
                a_best = min(meas, key=meas.get)
                r["ideal_measured"] = {"measured_ms": round(meas[a_best], 5), "slot_of": list(a_best)}
                note("ideal_measured")
        res[cfg] = r
        os.makedirs(os.path.dirname(args.out) or ".", exist_ok=True)
        with open(args.out, "w") as f:
            json.dump(res, f, indent=1)
        print(cfg, json.dumps(r), flush=True)
        del sess
        torch.cuda.empty_cache()
    os.makedirs(os.path.dirname(args.out) or ".", exist_ok=True)
    with open(args.out, "w") as f:
        json.dump(res, f, indent=1)


if __name__ == "__main__":
    main()
