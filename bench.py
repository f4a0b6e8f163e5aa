"""DUET on B200 — benchmark (driver contract: one JSON line on rank 0).

Headline workload: BASELINE.json configs[4] (c5, the 8-way heterogeneous ensemble, batch 4096), the
largest configuration that fits one GPU; `per_config` adds c1-c4 (configs[0..3]) and c6 (MT-DNN) measured the same
way in the same run (BASELINE.json:2 "per model").  A *step* = one inference of one batch through
the whole hot path, executed by libduet's greedy-correction schedule on CUDA-stream slots (one
CUDA-graph replay).

  value        whole-job samples/s with inputs resident in HBM (batch x K / max-rank time)
  e2e          same, through duet_run with pinned HOST buffers (H2D + D2H inside the timed step);
               also its host wall clock (duet_run + stream sync) per step
  p50/p99      per-step latency (CUDA events on the home stream, L2 flushed between steps); p99 /
               p99.9 from a separate tail pass of --tail-samples steps
  speedup      p50(serial 1-stream, same kernels) / p50(DUET)           (BASELINE.json:2)
  roofline     dominant kernel, timed live and cold (L2 flushed before every launch; CUDA events
               captured around the launch on its stream)
  cpu_baseline float64 oracle on a bounded row sample (rank 0, N = 1), all host cores and 1 thread

Multi-GPU (torchrun, one process per GPU):
  --placement shard (default for N > 1): ONE global batch per step, rows scattered from rank 0
      over NCCL, every rank runs its row block through its own schedule, outputs gathered back to
      rank 0 inside the timed step (strong scaling; multirank.ShardExecutor).
  --placement replica: every rank runs its own full batch (weak scaling, no data-path collective).
  --placement branch: ONE batch, subgraphs placed on the GPUs by greedy-correction over one slot
      per GPU with a measured NVLink comm model, cut edges over NCCL point-to-point (multigpu.py).
`--impl reference` times the oracle (the reference arm of this tier) on the host cores.
"""
from __future__ import annotations

import argparse
import json
import os
import re
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "p50 inference latency (ms) & samples/sec per model; speedup vs serial 1-stream"
L2_FLUSH_BYTES = 512 << 20  # > 126 MB L2
BASELINE_IDX = {"c1": 0, "c2": 1, "c3": 2, "c4": 3, "c5": 4}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=300)
    ap.add_argument("--warmup", type=int, default=20)
    ap.add_argument("--impl", default="duet", choices=["duet", "reference"])
    ap.add_argument("--config", default="c5", choices=["c1", "c2", "c3", "c4", "c5", "c6"],
                    help="c1-c5 = BASELINE.json configs[0..4]; c6 = MT-DNN (SURVEY.md §8(f) N4(b), not a BASELINE config)")
    ap.add_argument("--per-config", default="auto",
                    help="comma list of extra configs measured in the same run ('auto': c1-c4 and c6 beside a c5 headline "
                         "at N = 1; 'none')")
    ap.add_argument("--slots", type=int, default=2, help="CUDA-stream slots on the GPU")
    ap.add_argument("--dtype", default=None, choices=[None, "bf16", "f32"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    ap.add_argument("--ref-seconds", type=float, default=90.0,
                    help="--impl reference: timed oracle seconds over the whole --steps K --warmup W run")
    ap.add_argument("--profile-samples", type=int, default=100)
    ap.add_argument("--tail-samples", type=int, default=1000, help="separate latency pass for p99 / p99.9")
    ap.add_argument("--sched", default="measured", choices=["measured", "model"],
                    help="Step 3's `measure latency`: device measurement (default) or the C3 model")
    ap.add_argument("--rnn-tiles", type=int, default=1,
                    help="1: choose the recurrences' gate-tile width by measured latency (harness.tuned_session)")
    ap.add_argument("--placement", default="auto", choices=["auto", "shard", "replica", "branch"],
                    help="N>1: 'shard' (default) = one global batch, rows scattered / gathered over NCCL (strong); "
                         "'replica' = every rank its own batch (weak); 'branch' = subgraphs placed on GPUs (strong)")
    return ap.parse_args()


# ---------------------------------------------------------------------------------------------
def clock_sampler(device_index: int):
    """Sample SM clock and throttle reasons during the timed region (NVML)."""
    try:
        import pynvml
        pynvml.nvmlInit()
        h = pynvml.nvmlDeviceGetHandleByIndex(device_index)
    except Exception as e:  # noqa: BLE001
        return None, None, {"error": f"nvml unavailable: {e}"}
    samples, reasons = [], set()
    stop = threading.Event()
    names = {
        "hw_slowdown": 0x8, "sw_thermal_slowdown": 0x20, "hw_thermal_slowdown": 0x40,
        "sw_power_cap": 0x4, "hw_power_brake_slowdown": 0x80,
    }

    def loop():
        while not stop.is_set():
            try:
                samples.append(pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM))
                r = pynvml.nvmlDeviceGetCurrentClocksEventReasons(h)
                for k, bit in names.items():
                    if r & bit:
                        reasons.add(k)
            except Exception:  # noqa: BLE001
                pass
            time.sleep(0.02)

    t = threading.Thread(target=loop, daemon=True)
    t.start()
    max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM)

    def finish():
        stop.set()
        t.join()
        med = statistics.median(samples) if samples else None
        return {"sm_mhz": med, "sm_max_mhz": max_mhz, "reasons": sorted(reasons), "samples": len(samples)}

    return finish, max_mhz, None


def percentile(xs, q):
    s = sorted(xs)
    k = min(len(s) - 1, max(0, int(round(q / 100.0 * (len(s) - 1)))))
    return s[k]


def time_steps(torch, run_step, home, steps, warmup, flush):
    """Per-step CUDA-event latencies on the home stream; L2 flushed (untimed) before each step."""
    for _ in range(warmup):
        run_step()
    torch.cuda.synchronize()
    starts = [torch.cuda.Event(enable_timing=True) for _ in range(steps)]
    ends = [torch.cuda.Event(enable_timing=True) for _ in range(steps)]
    with torch.cuda.stream(home):
        for i in range(steps):
            flush.zero_()
            starts[i].record(home)
            run_step()
            ends[i].record(home)
    torch.cuda.synchronize()
    return [s.elapsed_time(e) for s, e in zip(starts, ends)]


def wall_steps(torch, run_step, home, steps, flush):
    """Host wall clock of duet_run + stream synchronize per step (the user-visible end-to-end
    latency including the launch path); L2 flushed and synchronised before each step, untimed."""
    out = []
    for _ in range(steps):
        flush.zero_()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        run_step()
        home.synchronize()
        out.append((time.perf_counter() - t0) * 1e3)
    return out


def node_decl(wl, name):
    """(op, %-args, dtype, shape) of node `name` in the workload's IR."""
    for ln in wl.ir.splitlines():
        m = re.match(r"^%([\w.]+) = (\w+)\((.*?)\).*: (\w+)\[([0-9,]*)\]$", ln)
        if m and m.group(1) == name:
            args = [a.strip()[1:] for a in m.group(3).split(",") if a.strip().startswith("%")]
            return m.group(2), args, m.group(4), tuple(int(x) for x in m.group(5).split(","))
    raise KeyError(name)


# recurrence gate-tile widths tried by harness.tuned_session (0 = automatic); BENCH_TILES overrides
TILE_CANDIDATES = tuple(int(x) for x in os.environ.get("BENCH_TILES", "0,128").split(","))

DOMINANT = {  # config -> node whose single launch dominates a step
    "c2": "fc1",      # 2048x1024x1664 pair GEMM
    "c3": "lstmA",    # one tower's persistent LSTM (S = 64)
    "c4": "gru",      # persistent GRU 1024 (S = 64): the longest single launch; the CNN is 20 launches
    "c5": "b4_gru",   # persistent GRU 1024 (S = 16, B = 4096): c5's longest single launch
    "c6": None,
    "c1": None,       # launch-bound at B = 1: no meaningful roofline
}


def node_work(wl, node):
    """Algorithmic FLOP of one launch of `node` (2·M·N·K; RNN = 2·S·B·G·H·(E+H))."""
    op, args, _, shape = node_decl(wl, node)
    if op == "linear":
        _, _, _, xs = node_decl(wl, args[0])
        return 2 * xs[0] * xs[1] * shape[-1]
    if op in ("lstm", "gru"):
        _, _, _, xs = node_decl(wl, args[0])   # [S, B, E]
        S, B, E = xs
        H = shape[-1]
        G = 4 if op == "lstm" else 3
        return 2 * S * B * G * H * (E + H)
    raise ValueError(op)


def time_node_cold(torch, graph, wl, node, stream, flush, samples=15):
    """Device time of one launch of `node`, L2 cold: a CUDA graph of [512 MB flush, event, the
    launch, event] on `stream`, replayed `samples` times (synchronised each time); median.  Also the
    warm back-to-back figure (20 launches in one graph) for reference."""
    op, args, dt, shape = node_decl(wl, node)
    tdt = {"bf16": torch.bfloat16, "f32": torch.float32}
    ins = []
    for a in args:
        _, _, adt, ash = node_decl(wl, a)
        ins.append((torch.randn(ash, device=stream.device) * 0.5).to(tdt[adt]))
    out = torch.empty(shape, dtype=tdt[dt], device=stream.device)
    graph.node_run(node, ins, out, stream)
    torch.cuda.synchronize()
    e0 = torch.cuda.Event(enable_timing=True, external=True)
    e1 = torch.cuda.Event(enable_timing=True, external=True)
    cg = torch.cuda.CUDAGraph()
    with torch.cuda.graph(cg, stream=stream):
        flush.zero_()
        e0.record(stream)
        graph.node_run(node, ins, out, stream)
        e1.record(stream)
    ts = []
    for i in range(samples + 2):
        cg.replay()
        torch.cuda.synchronize()
        if i >= 2:
            ts.append(e0.elapsed_time(e1))
    cold = statistics.median(ts)
    warm_g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(warm_g, stream=stream):
        for _ in range(20):
            graph.node_run(node, ins, out, stream)
    warm_g.replay()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(stream):
        a.record(stream)
        for _ in range(5):
            warm_g.replay()
        b.record(stream)
    torch.cuda.synchronize()
    return cold, a.elapsed_time(b) / 100


def load_traffic(node):
    p = os.path.join(ROOT, "profiles", "ncu_summary.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return d.get("kernels", {}).get(node, {}).get("dram_bytes")
    except Exception:  # noqa: BLE001
        return None


def load_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return d["hbm_gbs"], d["bf16_tflops"], d.get("bf16_tflops_sustained", d["bf16_tflops"]), "measured"
    except Exception:  # noqa: BLE001
        return 6650.0, 1590.0, 1590.0, "fallback"


def node_executed(wl, node):
    """FLOP the kernels actually issue for one launch of `node`: the algorithmic count with the
    recurrences' padding -- four gate blocks for GRU too (n_x and n_h kept apart), batch
    rows padded to the 128-row tiles, E padded to 64 -- (GEMMs: the algorithmic count)."""
    op, args, _, shape = node_decl(wl, node)
    if op in ("lstm", "gru"):
        _, _, _, xs = node_decl(wl, args[0])
        S, B, E = xs
        H = shape[-1]
        Bp, Ep = -(-B // 128) * 128, -(-E // 64) * 64
        return 2 * S * Bp * 4 * H * (Ep + H)
    return node_work(wl, node)


def roofline(torch, cfg, wl, sess, flush):
    node = DOMINANT.get(cfg)
    if node is None:
        return None
    hbm, burst, sustained, src = load_peaks()
    work = node_work(wl, node)
    cold_ms, warm_ms = time_node_cold(torch, sess.graph, wl, node, sess.home, flush)
    op = node_decl(wl, node)[0]
    # the kernel is timed alone (one launch per replay): the burst peak is the denominator
    # (MEASURED_PEAKS.json bf16_tflops); the sustained figure is reported beside it
    peak = burst
    achieved = work / (cold_ms / 1e3) / 1e12
    kname = {"linear": "gemm2_kernel (tcgen05 cta_group::2, TMA, TMEM)",
             "lstm": "rnn_persist_kernel (persistent LSTM: tcgen05 per step, fused gates)",
             "gru": "rnn_persist_kernel (persistent GRU: tcgen05 per step, fused gates)"}[op]
    return {"bound": "tensor", "kernel": f"{node}: {kname}", "achieved": round(achieved, 1), "peak": peak,
            "unit": "TFLOP/s", "frac": round(achieved / peak, 4), "traffic": load_traffic(f"{cfg}:{node}"),
            "peak_source": f"{src} MEASURED_PEAKS.json bf16_tflops (burst; kernel timed alone)",
            "frac_vs_sustained": round(achieved / sustained, 4),
            "algorithmic_per_launch": work, "ms_per_launch": round(cold_ms, 5), "timing": "cold (L2 flushed)",
            "warm_ms_per_launch": round(warm_ms, 5),
            "warm_frac": round(work / (warm_ms / 1e3) / 1e12 / burst, 4),
            # secondary: the rate on the FLOP the kernel issues (GRU's fourth gate block, tile padding)
            "executed_per_launch": node_executed(wl, node),
            "frac_executed": round(node_executed(wl, node) / (cold_ms / 1e3) / 1e12 / peak, 4)}


# ---------------------------------------------------------------------------------------------
def cpu_oracle_baseline(wl, params_host, inputs_host, seconds, sample_rows=128, threads=None):
    """Oracle (float64 NumPy, as it stands) on bounded row samples of the same workload."""
    import numpy as np
    import torch
    from threadpoolctl import threadpool_info, threadpool_limits

    from oracle import forward as OF

    def to_np(t):
        t = t.detach().cpu()
        return t.view(torch.int16).numpy().view(np.uint16) if t.dtype == torch.bfloat16 else t.numpy()

    # one bounded sample per call: rows drawn once, the table rows they touch generated and the
    # oracle warmed once (untimed), then timed passes over that sample until `seconds` elapse, so the
    # wall time stays ~ seconds + one warm pass (the reference arm calls this once per step)
    rng = np.random.default_rng(7)
    rows = rng.choice(wl.batch, min(sample_rows, wl.batch), replace=False)
    oin = {k: to_np(v)[rows] for k, v in inputs_host.items()}
    cache = {}

    def lazy(spec, name):
        def rows_fn(*lead):
            key = (name,) + tuple(np.asarray(a).tobytes() for a in lead)
            if key not in cache:
                idx = tuple(torch.as_tensor(np.ascontiguousarray(a), dtype=torch.int64) for a in lead)
                cache[key] = to_np(spec.rows(*idx))
            return cache[key]
        return rows_fn

    oparams = {}
    for k, spec in wl.params.items():
        oparams[k] = lazy(spec, k) if spec.numel > 10_000_000 else params_host[k]
    OF.run(wl.ir, oparams, oin)  # warm the row cache (untimed)
    done_rows, elapsed, reps = 0, 0.0, 0
    with threadpool_limits(limits=threads):
        n_threads = max([p.get("num_threads", 1) for p in threadpool_info()] or [1])
        while elapsed < seconds or reps == 0:
            t0 = time.perf_counter()
            OF.run(wl.ir, oparams, oin)
            elapsed += time.perf_counter() - t0
            done_rows += len(rows)
            reps += 1
    return {"value": done_rows / elapsed, "unit": "samples/s", "cores": n_threads, "kind": "oracle",
            "sample": f"{reps} timed passes over {len(rows)} random batch rows of {wl.name} (float64 NumPy "
                      f"oracle; the table rows they touch generated before timing)", "seconds": round(elapsed, 2)}


def cpu_model():
    try:
        for ln in open("/proc/cpuinfo"):
            if ln.startswith("model name"):
                return ln.split(":", 1)[1].strip()
    except OSError:
        pass
    return None


def host_params(torch, wl):
    import numpy as np
    small = {k: s.materialize("cpu") for k, s in wl.params.items() if s.numel <= 10_000_000}
    return {k: (v.view(torch.int16).numpy().view(np.uint16) if v.dtype == torch.bfloat16 else v.numpy())
            for k, v in small.items()}


def reference_arm(args):
    """--impl reference: the oracle timed on the host cores (rank 0 only)."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import torch

    from paper_conf_ipps_zhanghl21_b200 import workloads as W
    wl = W.build(args.config, dt=args.dtype)
    params_host = host_params(torch, wl)
    inputs = {k: s.materialize("cpu") for k, s in wl.inputs.items()}
    # the whole --steps K --warmup W run: ~ref_seconds of timed oracle work (each step >= one pass)
    per_step = max(0.02, min(20.0, args.ref_seconds / max(1, args.steps + args.warmup)))
    times = []
    for i in range(args.warmup + args.steps):
        cb = cpu_oracle_baseline(wl, params_host, inputs, per_step)
        if i >= args.warmup:
            times.append(cb)
    val = statistics.mean(t["value"] for t in times)
    ms = wl.batch / val * 1e3
    line = {"impl": "reference", "metric": METRIC, "value": val, "unit": "samples/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": wl.name, "global_batch": wl.batch, "parallelism": "cpu"},
            "cpu_baseline": {k: times[0][k] for k in ("cores", "kind", "sample")} | {"value": val,
                                                                                     "unit": "samples/s",
                                                                                     "cpu_model": cpu_model()},
            "e2e": {"value": val, "unit": "samples/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------------------------------------
def make_session(args, cfg, local, batch=None):
    """Load, bind, partition, profile and schedule one workload on this GPU: the measured
    greedy-correction schedule (with the recurrences' gate-tile width chosen by measurement), the
    model-mode schedule and the serial 1-stream baseline of the same kernels."""
    import torch

    from paper_conf_ipps_zhanghl21_b200 import duet
    from paper_conf_ipps_zhanghl21_b200 import workloads as W
    from paper_conf_ipps_zhanghl21_b200.harness import Session, tuned_session
    kw = {"batch": batch} if batch else {}
    wl = W.build(cfg, dt=args.dtype, **kw)
    prof_opts = dict(warmup=5, samples=args.profile_samples, reps=10, calibrate_comm=True)
    tile_ns = None
    if args.sched == "measured" and W.rnn_nodes(wl) and args.rnn_tiles:
        sess, duet_s, tile_ns, base = tuned_session(wl, n_slots=args.slots, device=local, profile=prof_opts,
                                                    tile_candidates=TILE_CANDIDATES)
    else:
        sess = base = Session(wl, n_slots=args.slots, device=local, profile=prof_opts)
        duet_s = None
    torch.cuda.synchronize()
    model_s = sess.schedule(duet.GREEDY_CORRECTION)
    if duet_s is None:
        duet_s = sess.schedule(duet.GREEDY_CORRECTION, measured=True, samples=60) if args.sched == "measured" else model_s
    serial_s = base.schedule(duet.SERIAL)
    return dict(wl=wl, sess=sess, base=base, duet_s=duet_s, model_s=model_s, serial_s=serial_s, tile_ns=tile_ns)


def measure(args, cfg, local, dev, flush, steps, warmup, headline=False):
    """Everything bench.py reports for one configuration on one GPU."""
    import torch

    from paper_conf_ipps_zhanghl21_b200 import multirank as MR
    from paper_conf_ipps_zhanghl21_b200.harness import materialize
    S = make_session(args, cfg, local)
    wl, sess, base, duet_s, model_s, serial_s = (S[k] for k in ("wl", "sess", "base", "duet_s", "model_s",
                                                                "serial_s"))
    inputs = list(materialize(wl.inputs, dev).values())
    outs = sess.outputs()
    torch.cuda.synchronize()  # inputs were generated on the default stream; duet_run uses `home`
    home = sess.home

    def step_duet():
        duet_s.run(sess.slots, inputs, outs)

    base.home.wait_stream(torch.cuda.current_stream())
    t_serial = time_steps(torch, lambda: serial_s.run(base.slots, inputs, outs), base.home, steps, warmup, flush)
    t_model = None
    if duet_s is not model_s and duet_s.export()["slot_of"] != model_s.export()["slot_of"]:
        t_model = time_steps(torch, lambda: model_s.run(sess.slots, inputs, outs), home, steps, warmup, flush)

    # --- timed region (DUET) ---
    MR.barrier()
    torch.cuda.synchronize()
    finish_clocks, _, clk_err = clock_sampler(local) if headline else (None, None, None)
    t_duet = time_steps(torch, step_duet, home, steps, warmup, flush)
    clocks = finish_clocks() if finish_clocks else clk_err
    torch.cuda.synchronize()
    total_ms = MR.max_over_ranks(sum(t_duet))
    MR.barrier()
    # tail pass (p99 / p99.9 need many samples)
    t_tail = time_steps(torch, step_duet, home, max(args.tail_samples, steps), 0, flush)

    # --- end to end through the C ABI with pinned host buffers ---
    host_in = [t.cpu().pin_memory() for t in inputs]
    host_out = sess.outputs(device=False)

    def step_e2e():
        duet_s.run(sess.slots, host_in, host_out)

    t_e2e = time_steps(torch, step_e2e, home, steps, warmup, flush)
    e2e_ms = MR.max_over_ranks(sum(t_e2e))
    t_wall = wall_steps(torch, step_e2e, home, min(steps, 200), flush)

    roof = roofline(torch, cfg, wl, sess, flush) if MR.env()[0] == 0 else None
    sched = duet_s.export()
    prof = sess.prof.export()
    p50 = statistics.median(t_duet)
    h2d = sum(t.numel() * t.element_size() for t in host_in)
    d2h = sum(t.numel() * t.element_size() for t in host_out)
    r = {
        "workload": wl.name, "baseline_config": BASELINE_IDX.get(cfg), "batch": wl.batch,
        "total_ms": total_ms, "steps": steps,
        "p50_ms": round(p50, 5), "p99_ms": round(percentile(t_tail, 99), 5),
        "p999_ms": round(percentile(t_tail, 99.9), 5), "tail_samples": len(t_tail),
        "mean_ms": round(statistics.mean(t_duet), 5),
        "serial_p50_ms": round(statistics.median(t_serial), 5),
        "speedup_vs_serial": round(statistics.median(t_serial) / p50, 4),
        "samples_per_s_p50": round(wl.batch / p50 * 1e3, 1),
        "schedule": {"step3": args.sched, "slot_of": sched["slot_of"], "fell_back": sched["fell_back"],
                     "model_makespan_ns": sched["makespan"], "profile_t_ns": prof["t_ns"][:, 0].tolist(),
                     "comm_alpha_same_ns": prof["comm"][0][0],
                     "measured_ns": getattr(duet_s, "measured_ns", None),
                     "evaluations": getattr(duet_s, "evaluations", None),
                     "model_mode_slot_of": model_s.export()["slot_of"],
                     "model_mode_p50_ms": round(statistics.median(t_model), 5) if t_model else None,
                     "rnn_tile_n": sess.wl.meta.get("rnn_tile_n"), "rnn_tile_measured_ns": S["tile_ns"]},
        "e2e": {"value": round(wl.batch * steps / (e2e_ms / 1e3), 1), "unit": "samples/s",
                "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
                "p50_ms": round(statistics.median(t_e2e), 5),
                "host_wall_p50_ms": round(statistics.median(t_wall), 5),
                "host_wall_note": "time.perf_counter around duet_run + home-stream synchronize, L2 flushed before"},
        "launches_per_step": duet_s.launch_count(),
        "roofline": roof,
        "clocks": clocks,
    }
    r["_keep"] = (wl, inputs)
    del S, sess, base, duet_s, model_s, serial_s, outs, host_in, host_out
    return r


def bench_single(args):
    import torch

    from paper_conf_ipps_zhanghl21_b200 import multirank as MR
    rank, world, local = MR.env()
    torch.cuda.set_device(local)
    MR.init("nccl", torch.device(f"cuda:{local}"))
    dev = f"cuda:{local}"
    flush = torch.empty(L2_FLUSH_BYTES // 4, dtype=torch.float32, device=dev)
    head = measure(args, args.config, local, dev, flush, args.steps, args.warmup, headline=True)
    wl, inputs = head.pop("_keep")

    extra = {}
    pcs = args.per_config
    if pcs == "auto":
        pcs = "c1,c2,c3,c4,c6" if (args.config == "c5" and world == 1) else "none"
    if pcs != "none" and rank == 0:
        for c in [c for c in pcs.split(",") if c and c != args.config]:
            torch.cuda.empty_cache()
            r = measure(args, c, local, dev, flush, min(args.steps, 200), max(args.warmup, 3))
            r.pop("_keep")
            for k in ("total_ms", "steps", "clocks"):
                r.pop(k)
            extra[c] = r

    if rank != 0:
        MR.finalize()
        return
    cpu_baseline = None
    if world == 1 and not args.no_cpu_baseline:
        ph = host_params(torch, wl)
        ih = dict(zip(wl.inputs, [t.cpu() for t in inputs]))
        cpu_baseline = cpu_oracle_baseline(wl, ph, ih, args.cpu_seconds)
        one = cpu_oracle_baseline(wl, ph, ih, max(2.0, args.cpu_seconds / 3), threads=1)
        cpu_baseline.update({"cpu_model": cpu_model(), "value_1thread": round(one["value"], 2),
                             "sample_1thread": one["sample"]})

    total_ms = head.pop("total_ms")
    line = {
        "metric": METRIC,
        "value": round(world * wl.batch * args.steps / (total_ms / 1e3), 1),
        "unit": "samples/s",
        "n_gpus": world,
        "steps": args.steps,
        "warmup": args.warmup,
        "ms_per_step": round(total_ms / args.steps, 5),
        "higher_is_better": True,
        "scaling": "weak",
        "vs_baseline": None,
        "dtype": wl.params[next(iter(wl.params))].dtype if args.dtype is None else args.dtype,
        "data": "synthetic (seeded counter-based generator; random-init weights)",
        "config": {"workload": head["workload"], "baseline_config": head["baseline_config"],
                   "global_batch": wl.batch * world, "per_gpu_batch": wl.batch, "slots": args.slots,
                   "parallelism": f"dp{world} (independent batches per rank) x {args.slots} stream slots",
                   "l2": "flushed (512 MB write) before every timed step"},
        "p50_ms": head["p50_ms"], "p99_ms": head["p99_ms"], "p999_ms": head["p999_ms"],
        "tail_samples": head["tail_samples"],
        "serial_p50_ms": head["serial_p50_ms"], "speedup_vs_serial": head["speedup_vs_serial"],
        "schedule": head["schedule"],
        "e2e": head["e2e"],
        "gpu_launches": head["launches_per_step"] * args.steps,
        "gpu_launches_per_step": head["launches_per_step"],
        "roofline": head["roofline"],
        "per_config": extra or None,
        "cpu_baseline": cpu_baseline,
        "clocks": head["clocks"],
    }
    print(json.dumps(line), flush=True)
    MR.finalize()


# ---------------------------------------------------------------------------------------------
def bench_shard(args):
    """--placement shard (N > 1 default): ONE global batch per step (BASELINE.json:11 "batch 4096
    across 1/2/4/8"); rank 0 holds the inputs in HBM, the rows are scattered over NCCL, every rank
    runs its B/N rows through its own measured DUET schedule, the outputs are gathered back to rank 0
    -- all inside the timed step (multirank.ShardExecutor)."""
    import torch

    from paper_conf_ipps_zhanghl21_b200 import multirank as MR
    from paper_conf_ipps_zhanghl21_b200 import workloads as W
    from paper_conf_ipps_zhanghl21_b200.harness import materialize
    rank, world, local = MR.env()
    torch.cuda.set_device(local)
    MR.init("nccl", torch.device(f"cuda:{local}"))
    dev = torch.device(f"cuda:{local}")
    full = W.build(args.config, dt=args.dtype)
    B = full.batch
    link = MR.calibrate_link()
    S = make_session(args, args.config, local, batch=B // world)
    sess, duet_s = S["sess"], S["duet_s"]
    tdt = {"f32": torch.float32, "bf16": torch.bfloat16}
    inputs = list(materialize(full.inputs, dev).values()) if rank == 0 else None
    in_meta = [(s.shape[1:], {"f32": torch.float32, "bf16": torch.bfloat16, "i32": torch.int32,
                              "i64": torch.int64}[s.dtype]) for s in full.inputs.values()]
    out_meta = [(tuple(shape[1:]), tdt[dt]) for _, dt, shape in full.outputs]
    ex = MR.ShardExecutor(B, in_meta, out_meta, dev)
    outs = [torch.empty((B,) + m[0], dtype=m[1], device=dev) for m in out_meta] if rank == 0 else None
    cur = torch.cuda.current_stream()

    def runner(si, so):
        sess.run(duet_s, si, so)                  # home waits on the current stream (the scatter)
        cur.wait_stream(sess.home)                # the gather sees the shard's outputs

    def step():
        ex.step(inputs, outs, runner)

    torch.cuda.synchronize()
    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    MR.barrier()
    finish_clocks, _, clk_err = clock_sampler(local)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(args.steps):
        step()
    e1.record()
    torch.cuda.synchronize()
    clocks = finish_clocks() if finish_clocks else clk_err
    ms = MR.max_over_ranks(e0.elapsed_time(e1))
    MR.barrier()
    # per-step latency (max over ranks per step is bounded by the rank-0 gather: rank 0 waits for all)
    lat = []
    for _ in range(min(args.steps, 100)):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        step()
        b.record()
        b.synchronize()
        lat.append(a.elapsed_time(b))
    # end to end: rank 0's pinned host inputs copied in, scattered, run, gathered, copied out
    host_in = [t.cpu().pin_memory() for t in inputs] if rank == 0 else None
    host_out = [torch.empty(o.shape, dtype=o.dtype).pin_memory() for o in outs] if rank == 0 else None
    dev_in = [torch.empty_like(t) for t in inputs] if rank == 0 else None

    def step_e2e():
        if rank == 0:
            for d, h in zip(dev_in, host_in):
                d.copy_(h, non_blocking=True)
        ex.step(dev_in, outs, runner)
        if rank == 0:
            for h, o in zip(host_out, outs):
                h.copy_(o, non_blocking=True)

    for _ in range(3):
        step_e2e()
    torch.cuda.synchronize()
    MR.barrier()
    e0.record()
    for _ in range(args.steps):
        step_e2e()
    e1.record()
    torch.cuda.synchronize()
    e2e_ms = MR.max_over_ranks(e0.elapsed_time(e1))
    sc, ga = ex.bytes_moved()
    n_launch = duet_s.launch_count()
    roof = None
    if rank == 0:  # the dominant kernel at this rank's B / N rows, timed alone and cold
        flush = torch.empty(L2_FLUSH_BYTES // 4, dtype=torch.float32, device=dev)
        roof = roofline(torch, args.config, S["wl"], sess, flush)
    if rank == 0:
        line = {"metric": METRIC, "value": round(B * args.steps / (ms / 1e3), 1), "unit": "samples/s",
                "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
                "ms_per_step": round(ms / args.steps, 5), "higher_is_better": True, "scaling": "strong",
                "vs_baseline": None, "dtype": args.dtype or "bf16",
                "data": "synthetic (seeded counter-based generator; random-init weights)",
                "config": {"workload": full.name, "baseline_config": BASELINE_IDX.get(args.config),
                           "global_batch": B, "per_gpu_batch": B // world, "slots": args.slots,
                           "parallelism": f"batch shards over {world} GPUs (NCCL scatter / gather of one global "
                                          f"batch inside the step) x {args.slots} stream slots",
                           "l2": "not flushed (inputs 33 MB on rank 0; every step re-scatters them)"},
                "p50_ms": round(statistics.median(lat), 5), "p99_ms": round(percentile(lat, 99), 5),
                "schedule": {"slot_of": duet_s.export()["slot_of"], "per_rank_batch": B // world},
                "collective_bytes_per_step": {"scatter_from_rank0": sc, "gather_to_rank0": ga},
                "nvlink_calibration": link,
                "e2e": {"value": round(B * args.steps / (e2e_ms / 1e3), 1), "unit": "samples/s",
                        "h2d_bytes_per_step": sum(t.numel() * t.element_size() for t in host_in),
                        "d2h_bytes_per_step": sum(t.numel() * t.element_size() for t in host_out)},
                "gpu_launches": n_launch * args.steps, "gpu_launches_per_step_per_rank": n_launch,
                "roofline": roof, "cpu_baseline": None, "clocks": clocks}
        print(json.dumps(line), flush=True)
    MR.finalize()


def bench_branch(args):
    """--placement branch: ONE batch per step; the greedy-correction schedule over one slot per GPU
    places the subgraphs, each rank runs its (GPU, phase) pieces through libduet, cut-edge tensors
    move over NCCL point-to-point (paper_conf_ipps_zhanghl21_b200/multigpu.py).
    The cross-GPU link in the comm model is measured (multirank.calibrate_link)."""
    import torch
    import torch.distributed as dist

    from paper_conf_ipps_zhanghl21_b200 import duet
    from paper_conf_ipps_zhanghl21_b200 import multigpu as MG
    from paper_conf_ipps_zhanghl21_b200 import multirank as MR
    from paper_conf_ipps_zhanghl21_b200 import workloads as W
    from paper_conf_ipps_zhanghl21_b200.harness import materialize

    rank, world, local = MR.env()
    torch.cuda.set_device(local)
    MR.init("nccl", torch.device(f"cuda:{local}"))
    dev = f"cuda:{local}"
    link = MR.calibrate_link()
    wl = W.build(args.config, dt=args.dtype)
    params = materialize(wl.params, dev)
    g = duet.Graph(wl.ir)
    g.bind_all(params)
    part = g.partition()
    ex = part.export()
    t_one = None
    if rank == 0:  # identical B200s: one GPU's per-subgraph times stand for every GPU's column
        st = torch.cuda.Stream()
        t_one = part.profile([(local, st)], warmup=3, samples=args.profile_samples, reps=5).export()["t_ns"][:, 0]
        t_one = [int(v) for v in t_one]
    if world > 1:
        obj = [t_one]
        dist.broadcast_object_list(obj, src=0)
        t_one = obj[0]
    kw = {"cross_alpha_ns": link["alpha_ns"], "cross_ps_per_byte": link["ps_per_byte"]} if link else {}
    sg_gpu, sched = MG.place_branches(ex, t_one, world, graph=g, **kw)
    pl = MG.plan(wl.ir, ex["node_to_sg"], ex["sg_phase"], sg_gpu)
    runner = MG.DuetPieces(pl, rank, params, local, n_slots=args.slots,
                           profile=dict(warmup=3, samples=max(5, args.profile_samples // 4), reps=5))
    exe = MG.Executor(pl, rank, runner, device=torch.device(dev))
    inputs = materialize(wl.inputs, dev) if rank == 0 else None
    torch.cuda.synchronize()
    for _ in range(args.warmup):
        exe.step(inputs)
    torch.cuda.synchronize()
    MR.barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    finish_clocks, _, clk_err = clock_sampler(local)
    e0.record()
    for _ in range(args.steps):
        exe.step(inputs)
    e1.record()
    torch.cuda.synchronize()
    clocks = finish_clocks() if finish_clocks else clk_err
    ms = MR.max_over_ranks(e0.elapsed_time(e1))
    n_launch = runner.launches()
    MR.barrier()
    if rank == 0:
        line = {"metric": METRIC, "value": round(wl.batch * args.steps / (ms / 1e3), 1), "unit": "samples/s",
                "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
                "ms_per_step": round(ms / args.steps, 5), "higher_is_better": True, "scaling": "strong",
                "vs_baseline": None, "dtype": args.dtype or "bf16",
                "data": "synthetic (seeded counter-based generator; random-init weights)",
                "config": {"workload": wl.name, "global_batch": wl.batch, "parallelism":
                           f"branch placement over {world} GPU(s) x {args.slots} stream slots",
                           "l2": "not flushed (multi-rank step)"},
                "placement": {"sg_gpu": sg_gpu, "model_makespan_ns": sched["makespan"],
                              "fell_back": sched["fell_back"], "profile_t_ns": t_one,
                              "comm_cross": kw or "nominal (single GPU: no link to measure)",
                              "transfers": [(t.tensor, t.src, t.dst) for t in pl.transfers]},
                "nvlink_calibration": link,
                "gpu_launches": n_launch * args.steps,
                "gpu_launches_per_step_rank0": n_launch, "roofline": None, "cpu_baseline": None, "clocks": clocks}
        print(json.dumps(line), flush=True)
    MR.finalize()


def main():
    args = parse()
    if args.impl == "reference":
        return reference_arm(args)
    world = int(os.environ.get("WORLD_SIZE", "1"))
    placement = args.placement if args.placement != "auto" else ("shard" if world > 1 else "replica")
    if placement == "branch":
        return bench_branch(args)
    if placement == "shard" and world > 1:
        return bench_shard(args)
    return bench_single(args)


if __name__ == "__main__":
    main()
