"""Oracle coarse-grained multi-phase partitioner (test infrastructure only; see oracle/__init__.py).

PAPER.md:79 (§IV-A): a phased schedule S_1..S_t of non-overlapping node sets with a total order
between phases; a phase is *sequential* (one subgraph) or *multi-path* (several independent
subgraphs); type(S_i) != type(S_i+1); shared inputs get replicated placeholders that all point
to the same input.  Footnote 1: one level of partitioning only.

The paper does not give the cut rule; this follows SURVEY.md §8(c) C2 (DESIGN.md "Readings"
R-C2), step by step:
  1. replicate every `input` node that has k > 1 consumers into k placeholders (one per consumer,
     in ascending consumer id; the original node keeps the first consumer);
  2. add a virtual source / sink; a *separator* is a node on every source->sink path;
  3. the region between consecutive separators (in topological rank) is the set of non-separator
     nodes reachable from the first and reaching the second; its weakly connected components
     (ignoring components made only of inputs) are candidate subgraphs;
  4. a region with >= 2 components is a multi-path phase; separators and regions with <= 1
     component are merged into maximal sequential phases;
  5. granularity: coarse = one subgraph per sequential phase / per component; op = one per node;
  6. subgraph ids sorted by (phase, smallest topological rank); boundary tensors and bytes.
Input nodes are not compute and belong to no subgraph (node_to_sg = -1).
"""
from __future__ import annotations

import heapq
from dataclasses import dataclass

from .ir import Graph, parse

SEQ, MULTI = 0, 1


@dataclass
class Partition:
    n_nodes: int
    node_to_sg: list        # over the IR's nodes; -1 for inputs
    sg_nodes: list          # per subgraph: IR node ids (ascending topological rank)
    sg_phase: list
    phase_kind: list        # SEQ / MULTI
    edges: dict             # (src_sg, dst_sg) -> bytes; -1 = graph input / output
    n_placeholders: int

    @property
    def n_sg(self):
        return len(self.sg_nodes)

    @property
    def n_phase(self):
        return len(self.phase_kind)

    def edge_list(self):
        return sorted(self.edges.items())


def _topo_rank(n, preds, succs):
    indeg = [len(p) for p in preds]
    ready = [v for v in range(n) if indeg[v] == 0]
    heapq.heapify(ready)
    rank = [0] * n
    k = 0
    while ready:
        u = heapq.heappop(ready)
        rank[u] = k
        k += 1
        for v in succs[u]:
            indeg[v] -= 1
            if indeg[v] == 0:
                heapq.heappush(ready, v)
    assert k == n
    return rank


def _reach(start, adj, n_total, blocked=None):
    seen = [False] * n_total
    stack = [start]
    seen[start] = True
    while stack:
        u = stack.pop()
        for v in adj[u]:
            if not seen[v] and v != blocked:
                seen[v] = True
                stack.append(v)
    return seen


def partition(ir, granularity: str = "coarse") -> Partition:
    g: Graph = parse(ir) if isinstance(ir, str) else ir
    n0 = len(g.nodes)
    is_input = [nd.op == "input" for nd in g.nodes]
    cons = g.consumers()

    # ---- step 1: replicated placeholders for shared inputs ----
    preds = [list(nd.inputs) for nd in g.nodes]
    alias = list(range(n0))            # working node -> IR node whose tensor it carries
    succs = [list(c) for c in cons]
    n_ph = 0
    for i in range(n0):
        if is_input[i] and len(cons[i]) > 1:
            first, rest = cons[i][0], cons[i][1:]
            succs[i] = [first]
            for c in rest:
                w = len(preds)
                preds.append([])
                succs.append([c])
                alias.append(i)
                is_input.append(True)
                preds[c] = [w if u == i else u for u in preds[c]]
                n_ph += 1
    N = len(preds)
    compute = [not is_input[v] for v in range(N)]
    rank = _topo_rank(N, preds, succs)

    # ---- step 2: virtual source / sink, separators ----
    S, T = N, N + 1
    fwd = [list(s) for s in succs] + [[], []]
    bwd = [list(p) for p in preds] + [[], []]
    for v in range(N):
        if not preds[v]:
            fwd[S].append(v)
            bwd[v].append(S)
        if not succs[v]:        # only sinks; outputs with consumers keep just their boundary edge
            fwd[v].append(T)
            bwd[T].append(v)
    seps = [v for v in range(N) if not _reach(S, fwd, N + 2, blocked=v)[T]]
    seps.sort(key=lambda v: rank[v])
    sepset = set(seps)

    # ---- step 3: regions and their weakly connected components ----
    bounds = [S] + seps + [T]
    down = {b: _reach(b, fwd, N + 2) for b in bounds}
    up = {b: _reach(b, bwd, N + 2) for b in bounds}
    items = []  # sequence of ("region", [components]) and ("sep", v)
    for bi in range(len(bounds) - 1):
        a, b = bounds[bi], bounds[bi + 1]
        region = [v for v in range(N) if v not in sepset and down[a][v] and up[b][v]]
        rset = set(region)
        comp_of = {}
        comps = []
        for v in sorted(region, key=lambda x: rank[x]):
            if v in comp_of:
                continue
            cid = len(comps)
            comps.append([])
            stack = [v]
            comp_of[v] = cid
            while stack:
                u = stack.pop()
                comps[cid].append(u)
                for w in succs[u] + preds[u]:
                    if w in rset and w not in comp_of:
                        comp_of[w] = cid
                        stack.append(w)
        comps = [sorted(c, key=lambda x: rank[x]) for c in comps]
        comps = [c for c in comps if any(compute[v] for v in c)]
        comps.sort(key=lambda c: min(rank[v] for v in c if compute[v]))
        items.append(("region", comps))
        if bi + 1 < len(bounds) - 1:
            items.append(("sep", b))

    # ---- step 4: phases ----
    phases = []   # (kind, [node lists])
    cur = []

    def flush():
        nonlocal cur
        if any(compute[v] for v in cur):
            phases.append((SEQ, [sorted(cur, key=lambda x: rank[x])]))
        cur = []

    for kind, payload in items:
        if kind == "sep":
            cur.append(payload)
        elif len(payload) >= 2:
            flush()
            phases.append((MULTI, payload))
        else:
            for c in payload:
                cur.extend(c)
    flush()

    # ---- step 5: granularity ----
    sgs = []   # (phase, [compute nodes by rank])
    for p, (kind, groups) in enumerate(phases):
        for grp in groups:
            nodes = [v for v in grp if compute[v]]
            if granularity == "coarse":
                sgs.append((p, nodes))
            elif granularity == "op":
                sgs.extend((p, [v]) for v in nodes)
            else:
                raise ValueError(granularity)
    # ---- step 6: ids in (phase, min rank) order; boundary tensors ----
    sgs.sort(key=lambda t: (t[0], min(rank[v] for v in t[1])))
    sg_of = [-1] * N
    for s, (_, nodes) in enumerate(sgs):
        for v in nodes:
            sg_of[v] = s
    tensors = {}
    for v in range(N):
        if not compute[v]:
            continue
        for u in preds[v]:
            src = sg_of[u] if compute[u] else -1
            if src == sg_of[v]:
                continue
            tensors.setdefault((src, sg_of[v]), set()).add(alias[u])
    for o in g.outputs:
        if compute[o]:
            tensors.setdefault((sg_of[o], -1), set()).add(o)
    edges = {k: sum(g.nodes[t].nbytes for t in ts) for k, ts in tensors.items()}
    return Partition(
        n_nodes=n0,
        node_to_sg=[sg_of[v] for v in range(n0)],
        sg_nodes=[nodes for _, nodes in sgs],
        sg_phase=[p for p, _ in sgs],
        phase_kind=[k for k, _ in phases],
        edges=edges,
        n_placeholders=n_ph,
    )
