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
  6. subgraph ids sorted by (phase, smallest topological rank); boundary tensors and bytes;
  7. batch_shards = k > 1 (multi-GPU): every subgraph of a multi-path
     phase becomes k row-shard subgraphs (ids consecutive, shard j = rows [j B / k, (j+1) B / k)),
     each priced separately by the profile; a tensor crossing into or out of shard j carries
     share_j(b) = floor(b (j+1) / k) - floor(b j / k) of its b bytes (the shares sum to b);
     shard-to-shard edges connect equal shard indices only (rows are independent).
Input nodes are not compute and belong to no subgraph (node_to_sg = -1; a sharded node maps to
its shard 0).
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
    sg_shard: list = None   # per subgraph: row-shard index, -1 = unsharded (batch_shards = 1 or seq phase)
    sg_origin: list = None  # per subgraph: id of the unsharded subgraph it is a shard of

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


def share(b: int, j: int, k: int) -> int:
    """Bytes of a b-byte row-major tensor that fall in row shard j of k (step 7)."""
    return b * (j + 1) // k - b * j // k


def partition(ir, granularity: str = "coarse", batch_shards: int = 1) -> Partition:
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
    # ---- step 7: row shards of the multi-path subgraphs ----
    k = int(batch_shards)
    if k < 1:
        raise ValueError("batch_shards must be >= 1")
    ids = []                      # unsharded subgraph -> its new ids (k of them if sharded)
    sg_shard, sg_origin = [], []
    for s, (p, _) in enumerate(sgs):
        shard = k > 1 and phases[p][0] == MULTI
        ids.append([])
        for j in range(k if shard else 1):
            ids[s].append(len(sg_shard))
            sg_shard.append(j if shard else -1)
            sg_origin.append(s)

    def pairs(src, dst):
        """(new src, new dst, shard index of the bytes or -1) for an edge between two unsharded ids."""
        S = ids[src] if src >= 0 else [-1]
        D = ids[dst] if dst >= 0 else [-1]
        if len(S) > 1 and len(D) > 1:
            return [(S[j], D[j], j) for j in range(k)]
        if len(D) > 1:
            return [(S[0], D[j], j) for j in range(k)]
        if len(S) > 1:
            return [(S[i], D[0], i) for i in range(k)]
        return [(S[0], D[0], -1)]

    tensors = {}                  # (new src, new dst) -> (shard index, {tensor ids})
    for v in range(N):
        if not compute[v]:
            continue
        for u in preds[v]:
            src = sg_of[u] if compute[u] else -1
            if src == sg_of[v]:
                continue
            for a, b, j in pairs(src, sg_of[v]):
                tensors.setdefault((a, b), (j, set()))[1].add(alias[u])
    for o in g.outputs:
        if compute[o]:
            for a, b, j in pairs(sg_of[o], -1):
                tensors.setdefault((a, b), (j, set()))[1].add(o)
    edges = {key: sum(g.nodes[t].nbytes if j < 0 else share(g.nodes[t].nbytes, j, k) for t in ts)
             for key, (j, ts) in tensors.items()}
    sg_nodes, sg_phase = [], []
    for s_new, s in enumerate(sg_origin):
        sg_nodes.append(sgs[s][1])
        sg_phase.append(sgs[s][0])
    return Partition(
        n_nodes=n0,
        node_to_sg=[ids[sg_of[v]][0] if sg_of[v] >= 0 else -1 for v in range(n0)],
        sg_nodes=sg_nodes,
        sg_phase=sg_phase,
        phase_kind=[kk for kk, _ in phases],
        edges=edges,
        n_placeholders=n_ph,
        sg_shard=sg_shard,
        sg_origin=sg_origin,
    )
