"""Branch placement across the GPUs of one node (PAPER.md:79-82 with the
paper's {CPU, GPU} device set generalised to one slot per GPU).

One process per GPU.  The greedy-correction schedule (libduet) maps every subgraph to a slot; a
slot's GPU decides which rank runs it.  The graph is cut into *pieces* = (GPU, phase): the nodes
of the subgraphs of one phase placed on one GPU.  Every piece is compiled as its own libduet graph
(its IR restricted to its nodes; a tensor produced by another piece becomes an `input`), so inside a
piece the single-GPU machinery applies unchanged (local partition, profile, greedy-correction over
that GPU's stream slots, one CUDA-graph launch).  Between phases the executor moves the cut-edge
tensors GPU -> GPU with point-to-point NCCL sends (graph inputs start on rank 0, graph outputs end
on rank 0: DESIGN.md R-10).  Phases run in order, so every cut edge crosses a phase boundary (a
multi-path phase's subgraphs are independent by construction).

The planning here is pure host logic over the IR text; `Executor` is compute-agnostic (the GPU run
uses libduet per piece, the CPU tests plug in the float64 oracle) and uses torch.distributed only
for the cut-edge transfers.
"""
from __future__ import annotations

import re
from dataclasses import dataclass, field

import torch
import torch.distributed as dist

_NODE = re.compile(r"^%([A-Za-z_][\w.]*)\s*=\s*([a-z_0-9]+)\s*\((.*?)\)\s*(\{.*?\})?\s*:\s*([a-z0-9]+)\s*\[([0-9,\s]*)\]\s*$")
_PARAM = re.compile(r"^param\s+@([A-Za-z_][\w.]*)\s*:")
_OUT = re.compile(r"^output\s+(.*)$")
TORCH_DT = {"f32": torch.float32, "bf16": torch.bfloat16, "i32": torch.int32, "i64": torch.int64}


@dataclass
class IRNode:
    id: int
    name: str
    op: str
    args: list        # %-argument names
    params: list      # @-argument names
    dtype: str
    shape: tuple
    line: str


@dataclass
class IRText:
    nodes: list
    params: dict      # name -> declaration line
    outputs: list     # node names, sorted by node id (libduet's graph output order)

    @property
    def by_name(self):
        return {n.name: n for n in self.nodes}


def parse_ir(text: str) -> IRText:
    nodes, params, outs = [], {}, []
    for raw in text.splitlines():
        line = raw.split("#", 1)[0].strip()
        if not line:
            continue
        m = _PARAM.match(line)
        if m:
            params[m.group(1)] = line
            continue
        m = _OUT.match(line)
        if m:
            outs += [t.strip().lstrip("%") for t in m.group(1).split(",") if t.strip()]
            continue
        m = _NODE.match(line)
        if not m:
            raise ValueError(f"IR line not understood: {line}")
        args = [a.strip() for a in m.group(3).split(",") if a.strip()]
        shape = tuple(int(x) for x in m.group(6).split(",") if x.strip())
        nodes.append(IRNode(len(nodes), m.group(1), m.group(2), [a[1:] for a in args if a.startswith("%")],
                            [a[1:] for a in args if a.startswith("@")], m.group(5), shape, line))
    ids = {n.name: n.id for n in nodes}
    outs = sorted(dict.fromkeys(outs), key=lambda nm: ids[nm])
    return IRText(nodes, params, outs)


@dataclass
class Piece:
    gpu: int
    phase: int
    nodes: list                      # node names (IR order)
    inputs: list = field(default_factory=list)   # cut-in tensor names (declared as `input`), IR order
    outputs: list = field(default_factory=list)  # tensors other pieces / the graph need, IR order
    ir: str = ""


@dataclass
class Transfer:
    tensor: str
    src: int      # GPU (rank) holding it
    dst: int
    phase: int    # needed before this phase runs (n_phases = after the last phase: graph outputs)


@dataclass
class Plan:
    pieces: list          # ordered by (phase, gpu)
    transfers: list       # ordered by (phase, tensor id, dst)
    n_phases: int
    home: int = 0
    tensor_meta: dict = field(default_factory=dict)  # name -> (dtype, shape)
    graph_inputs: list = field(default_factory=list)
    graph_outputs: list = field(default_factory=list)

    def pieces_on(self, gpu: int):
        return [p for p in self.pieces if p.gpu == gpu]


def plan(ir_text: str, node_to_sg, sg_phase, sg_gpu, home: int = 0) -> Plan:
    """Cut the graph into (GPU, phase) pieces and list the cut-edge transfers.

    node_to_sg: per IR node (input nodes -1, libduet's partition export), sg_phase: per subgraph,
    sg_gpu: per subgraph, the GPU of its slot (schedule slot_of mapped through the slot_gpu table)."""
    ir = parse_ir(ir_text)
    if len(node_to_sg) != len(ir.nodes):
        raise ValueError("node_to_sg does not match the IR")
    where = {}   # tensor -> (gpu, phase) of its producer; inputs: (home, -1)
    for n in ir.nodes:
        s = node_to_sg[n.id]
        where[n.name] = (home, -1) if n.op == "input" or s < 0 else (int(sg_gpu[s]), int(sg_phase[s]))
    n_phases = max([p for _, p in where.values()] + [-1]) + 1
    groups = {}
    for n in ir.nodes:
        g, p = where[n.name]
        if p >= 0:
            groups.setdefault((p, g), []).append(n)
    consumers = {n.name: [] for n in ir.nodes}
    for n in ir.nodes:
        for a in n.args:
            consumers[a].append(n)
    pieces, transfers, seen = [], [], set()
    out_set = set(ir.outputs)
    for (p, g), members in sorted(groups.items()):
        names = {m.name for m in members}
        ins = []
        for m in members:
            for a in m.args:
                if a not in names and a not in ins:
                    ins.append(a)
        ins.sort(key=lambda nm: ir.by_name[nm].id)
        outs = [m.name for m in members
                if m.name in out_set or any(where[c.name] != (g, p) for c in consumers[m.name])]
        lines = []
        used_params = []
        for m in members:
            for q in m.params:
                if q not in used_params:
                    used_params.append(q)
        lines += [ir.params[q] for q in used_params]
        for a in ins:
            src = ir.by_name[a]
            lines.append(f"%{a} = input() : {src.dtype}[{','.join(map(str, src.shape))}]")
        lines += [m.line for m in members]
        lines.append("output " + ", ".join(f"%{o}" for o in outs))
        pieces.append(Piece(g, p, [m.name for m in members], ins, outs, "\n".join(lines) + "\n"))
        for a in ins:
            sg_, _ = where[a]
            if sg_ != g and (a, g) not in seen:
                seen.add((a, g))
                transfers.append(Transfer(a, sg_, g, p))
    for o in ir.outputs:
        g, _ = where[o]
        if g != home and (o, home) not in seen:
            seen.add((o, home))
            transfers.append(Transfer(o, g, home, n_phases))
    idx = {n.name: n.id for n in ir.nodes}
    transfers.sort(key=lambda t: (t.phase, idx[t.tensor], t.dst))
    meta = {n.name: (n.dtype, n.shape) for n in ir.nodes}
    return Plan(pieces, transfers, n_phases, home, meta,
                [n.name for n in ir.nodes if n.op == "input"], list(ir.outputs))


class Executor:
    """Runs one inference across ranks: for each phase, the cut-edge transfers into it
    (torch.distributed point-to-point, rank = GPU), then this rank's piece of that phase.

    run_piece(piece, {name: tensor}) -> {name: tensor} computes a piece on this rank's device.
    Tensors live in `self.store` (this rank's copies); graph inputs must be in rank `home`'s store."""

    def __init__(self, pl: Plan, rank: int, run_piece, device=None, alloc=None):
        self.pl, self.rank, self.run_piece = pl, rank, run_piece
        self.device = device if device is not None else torch.device("cpu")
        self.alloc = alloc or (lambda dt, shape: torch.empty(shape, dtype=TORCH_DT[dt], device=self.device))
        self.store = {}

    def _exchange(self, phase: int):
        ops, landed = [], []
        # gloo moves host tensors only: device tensors are staged through host memory (the one-GPU
        # test of the multi-rank path; NCCL sends and receives device memory directly)
        staged = self.device.type == "cuda" and dist.get_backend() == "gloo"
        for t in self.pl.transfers:
            if t.phase != phase or self.rank not in (t.src, t.dst):
                continue
            if self.rank == t.src:
                x = self.store[t.tensor].contiguous()
                ops.append(dist.P2POp(dist.isend, x.cpu() if staged else x, t.dst))
            else:
                buf = self.store.get(t.tensor)
                if buf is None:
                    buf = self.store[t.tensor] = self.alloc(*self.pl.tensor_meta[t.tensor])
                tmp = torch.empty(buf.shape, dtype=buf.dtype) if staged else buf
                if staged:
                    landed.append((buf, tmp))
                ops.append(dist.P2POp(dist.irecv, tmp, t.src))
        if ops:
            for w in dist.batch_isend_irecv(ops):
                w.wait()
        for buf, tmp in landed:
            buf.copy_(tmp)

    def step(self, inputs: dict | None = None):
        if inputs:
            self.store.update(inputs)
        for phase in range(self.pl.n_phases + 1):
            self._exchange(phase)
            if phase == self.pl.n_phases:
                break
            for pc in self.pl.pieces:
                if pc.phase == phase and pc.gpu == self.rank:
                    outs = self.run_piece(pc, {a: self.store[a] for a in pc.inputs})
                    self.store.update(outs)
        if self.rank == self.pl.home:
            return [self.store[o] for o in self.pl.graph_outputs]
        return None


class DuetPieces:
    """The GPU compute of one rank: every piece placed on this rank compiled as its own libduet
    graph, partitioned, profiled and scheduled (greedy-correction) over this GPU's stream slots."""

    def __init__(self, pl: Plan, gpu: int, params: dict, device: int, n_slots: int = 2, profile=None):
        from . import duet  # noqa: PLC0415  (the binding loads libduet.so; CPU planning does not need it)
        self.device = device
        lo_hi = [0] + [-1] * (n_slots - 1)
        self.streams = [torch.cuda.Stream(device=device, priority=p) for p in lo_hi]
        self.slots = [(device, s) for s in self.streams]
        self.pieces = {}
        for pc in pl.pieces_on(gpu):
            g = duet.Graph(pc.ir)
            g.bind_all({k: params[k] for k in parse_ir(pc.ir).params})
            part = g.partition()
            prof = part.profile(self.slots, **(profile or dict(warmup=3, samples=20, reps=5)))
            sched = prof.schedule()
            outs = [torch.empty(pl.tensor_meta[o][1], dtype=TORCH_DT[pl.tensor_meta[o][0]], device=f"cuda:{device}")
                    for o in pc.outputs]
            self.pieces[(pc.phase, pc.gpu)] = (g, part, prof, sched, outs)

    def launches(self) -> int:
        return sum(v[3].launch_count() for v in self.pieces.values())

    def __call__(self, pc: Piece, ins: dict) -> dict:
        g, part, prof, sched, outs = self.pieces[(pc.phase, pc.gpu)]
        home = self.streams[0]
        home.wait_stream(torch.cuda.current_stream(self.device))  # inputs received / produced upstream
        sched.run(self.slots, [ins[a] for a in pc.inputs], outs)
        torch.cuda.current_stream(self.device).wait_stream(home)  # later sends / consumers see the results
        return dict(zip(pc.outputs, outs))


def place_branches(part_export: dict, t_ns_one_slot, n_gpu: int, cross_alpha_ns: int = 20000,
                   cross_ps_per_byte: int = 2, graph=None):
    """Greedy-correction placement of the subgraphs on one slot per GPU (identical GPUs: the
    single-GPU profile column replicated), the NVLink cut-edge cost in the comm model.
    Returns (sg_gpu, schedule export).  Deterministic: every rank derives the same placement."""
    import numpy as np  # noqa: PLC0415
    t = np.asarray(t_ns_one_slot, dtype=np.int64).reshape(-1, 1)
    table = np.repeat(t, n_gpu, axis=1)
    prof = graph.partition().profile_from_table(list(range(n_gpu)), table,
                                                ((0, 0), (cross_alpha_ns, cross_ps_per_byte)))
    s = prof.schedule().export()
    return [int(x) for x in s["slot_of"]], s
