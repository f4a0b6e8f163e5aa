"""Session helper over the binding: materialise a workload's seeded weights/inputs on the GPU,
load + bind the graph, partition, profile, schedule, and run.  Plumbing only (torch allocates
memory and streams); all compute is in libduet.so."""
from __future__ import annotations

import torch

from . import duet
from .workloads import Workload


def materialize(specs: dict, device) -> dict:
    return {k: s.materialize(device) for k, s in specs.items()}


class Session:
    def __init__(self, wl: Workload, n_slots: int = 2, device: int = 0, granularity: str = "coarse",
                 params: dict | None = None, profile: dict | None = None, table=None, comm=None):
        self.wl = wl
        self.device = device
        torch.cuda.set_device(device)
        self.params = params if params is not None else materialize(wl.params, f"cuda:{device}")
        self.graph = duet.Graph(wl.ir)
        self.graph.bind_all(self.params)
        self.part = self.graph.partition(granularity)
        # slot 0 (home: inputs, outputs, the critical path after Step 1) at normal priority; the other
        # slots at high priority so their (typically latency-bound) kernels are not starved by a
        # co-running throughput branch
        lo, hi = torch.cuda.Stream.priority_range() if hasattr(torch.cuda.Stream, "priority_range") else (0, -1)
        self.streams = [torch.cuda.Stream(device=device, priority=0 if i == 0 else -1) for i in range(n_slots)]
        self.slots = [(device, s) for s in self.streams]
        if table is not None:
            self.prof = self.part.profile_from_table([device] * n_slots, table, comm or ((0, 0), (0, 0)))
        else:
            self.prof = self.part.profile(self.slots, **(profile or {}))
        self.schedules = {}

    def schedule(self, mode=duet.GREEDY_CORRECTION, measured=False, **kw) -> duet.Schedule:
        """measured=True: Step 3 / fallback compare assignments by device-measured latency over
        this session's slots (duet_schedule_measured); else by the profile's makespan model."""
        key = (mode, measured, tuple(sorted(kw.items())))
        if key not in self.schedules:
            if measured:
                torch.cuda.current_stream(self.device).synchronize()
                self.schedules[key] = self.prof.schedule_measured(self.slots, mode=mode, **kw)
            else:
                self.schedules[key] = self.prof.schedule(mode=mode, **kw)
        return self.schedules[key]

    def outputs(self, device=True):
        dev = f"cuda:{self.device}" if device else "cpu"
        out = []
        for _, dt, shape in self.wl.outputs:
            t = torch.empty(shape, dtype={"f32": torch.float32, "bf16": torch.bfloat16}[dt], device=dev)
            out.append(t.pin_memory() if not device else t)
        return out

    def run(self, sched: duet.Schedule, inputs, outputs):
        # duet_run enqueues on the home slot stream (non-blocking w.r.t. the legacy stream): order it
        # after whatever produced the inputs / last used the outputs on the caller's current stream
        self.home.wait_stream(torch.cuda.current_stream(self.device))
        sched.run(self.slots, inputs, outputs)

    @property
    def home(self) -> torch.cuda.Stream:
        return self.streams[0]


def tuned_session(wl: Workload, n_slots: int = 2, device: int = 0, profile: dict | None = None,
                  tile_candidates=(0, 128), samples: int = 60, mode=duet.GREEDY_CORRECTION):
    """Kernel-variant choice by measurement (the compiler-aware profiler's idea, §IV-B:
    each compiled variant is profiled, and the correction's, :81 §IV-C: candidate schedules are
    compared by measured latency).  The variant here is the persistent recurrence's gate-tile width,
    an SM budget when branches share one GPU:
    the workload is built with each width in `tile_candidates` (applied to every LSTM/GRU node;
    0 = the automatic choice), scheduled with measured greedy-correction, and the session with the
    lowest measured latency is kept.  The weights are materialised once and shared.

    Returns (best session, its measured schedule, {tile_n: measured ns}, the automatic-width session
    (the serial baseline's kernels: tuned for running alone), or the best one if it is that)."""
    from .workloads import rnn_nodes, with_rnn_tile_n
    base = Session(with_rnn_tile_n(wl, 0) if rnn_nodes(wl) else wl, n_slots=n_slots, device=device,
                   profile=profile)
    torch.cuda.synchronize(device)
    s0 = base.schedule(mode, measured=True, samples=samples)
    results = {0: int(s0.measured_ns)}
    best, best_s, best_ns = base, s0, s0.measured_ns
    if rnn_nodes(wl):
        for t in tile_candidates:
            if t == 0:
                continue
            sess = Session(with_rnn_tile_n(wl, t), n_slots=n_slots, device=device,
                           params=base.params, profile=profile)
            torch.cuda.synchronize(device)
            s = sess.schedule(mode, measured=True, samples=samples)
            results[t] = int(s.measured_ns)
            if s.measured_ns < best_ns:
                best, best_s, best_ns = sess, s, s.measured_ns
    return best, best_s, results, base
