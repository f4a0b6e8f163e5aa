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
