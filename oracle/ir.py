"""Oracle IR reader (test infrastructure only; see oracle/__init__.py).

Reads the DUET text IR (grammar in include/duet.h) into an adjacency-list graph, the analogue of
the paper's Relay -> adjacency-list translation (Fig. 10): nodes are operators,
an edge (v_i, v_j) means v_j consumes v_i's output.
"""
from __future__ import annotations

import re
from dataclasses import dataclass, field

DTYPE_BYTES = {"f32": 4, "bf16": 2, "i32": 4, "i64": 8}


class IRError(ValueError):
    pass


@dataclass
class Node:
    id: int
    name: str
    op: str
    args: list            # list of ("%", name) or ("@", name)
    attrs: dict
    dtype: str
    shape: tuple
    inputs: list = field(default_factory=list)   # producer node ids (unique, ascending)
    params: list = field(default_factory=list)   # parameter names in argument order

    @property
    def nbytes(self) -> int:
        n = DTYPE_BYTES[self.dtype]
        for s in self.shape:
            n *= s
        return n


@dataclass
class Graph:
    nodes: list
    params: dict            # name -> (dtype, shape)
    outputs: list           # node ids
    by_name: dict

    def consumers(self):
        cons = [[] for _ in self.nodes]
        for n in self.nodes:
            for u in n.inputs:
                cons[u].append(n.id)
        return [sorted(set(c)) for c in cons]


_NODE = re.compile(r"^%([A-Za-z_][\w.]*)\s*=\s*([a-z_0-9]+)\s*\((.*?)\)\s*(\{(.*?)\})?\s*:\s*"
                   r"([a-z0-9]+)\s*\[([0-9,\s]*)\]\s*$")
_PARAM = re.compile(r"^param\s+@([A-Za-z_][\w.]*)\s*:\s*([a-z0-9]+)\s*\[([0-9,\s]*)\]\s*$")
_OUT = re.compile(r"^output\s+(.*)$")


def _shape(s: str) -> tuple:
    s = s.strip()
    if not s:
        return ()
    return tuple(int(x) for x in s.split(","))


def _attr_val(v: str):
    v = v.strip()
    try:
        return int(v)
    except ValueError:
        pass
    try:
        return float(v)
    except ValueError:
        return v


def parse(text: str) -> Graph:
    nodes, params, outputs, by_name = [], {}, [], {}
    out_names = []
    for raw in text.splitlines():
        line = raw.split("#", 1)[0].strip()
        if not line:
            continue
        m = _PARAM.match(line)
        if m:
            name, dt, shp = m.groups()
            if dt not in DTYPE_BYTES or name in params:
                raise IRError(f"bad param: {line}")
            params[name] = (dt, _shape(shp))
            continue
        m = _OUT.match(line)
        if m:
            for tok in m.group(1).split(","):
                tok = tok.strip()
                if not tok.startswith("%"):
                    raise IRError(f"bad output: {line}")
                out_names.append(tok[1:])
            continue
        m = _NODE.match(line)
        if not m:
            raise IRError(f"cannot parse: {line}")
        name, op, args, _, attrs, dt, shp = m.groups()
        if dt not in DTYPE_BYTES or name in by_name:
            raise IRError(f"bad node: {line}")
        arglist = []
        for a in (x.strip() for x in args.split(",")):
            if not a:
                continue
            if a[0] not in "%@" or len(a) < 2:
                raise IRError(f"bad argument {a!r}: {line}")
            arglist.append((a[0], a[1:]))
        ad = {}
        if attrs:
            for kv in attrs.split(","):
                if not kv.strip():
                    continue
                k, v = kv.split("=", 1)
                ad[k.strip()] = _attr_val(v)
        n = Node(len(nodes), name, op, arglist, ad, dt, _shape(shp))
        by_name[name] = n.id
        nodes.append(n)
    for n in nodes:
        ins = []
        for kind, nm in n.args:
            if kind == "%":
                if nm not in by_name:
                    raise IRError(f"undefined value %{nm}")
                ins.append(by_name[nm])
            else:
                if nm not in params:
                    raise IRError(f"undefined parameter @{nm}")
                n.params.append(nm)
        n.inputs = sorted(set(ins))
    for nm in out_names:
        if nm not in by_name:
            raise IRError(f"undefined output %{nm}")
        outputs.append(by_name[nm])
    g = Graph(nodes, params, sorted(set(outputs)), by_name)
    topo_order(g)  # raises on cycles
    return g


def topo_order(g: Graph) -> list:
    """Kahn's algorithm, always taking the smallest ready node id (the rank used everywhere)."""
    import heapq
    indeg = [len(n.inputs) for n in g.nodes]
    cons = g.consumers()
    ready = [i for i, d in enumerate(indeg) if d == 0]
    heapq.heapify(ready)
    order = []
    while ready:
        u = heapq.heappop(ready)
        order.append(u)
        for v in cons[u]:
            indeg[v] -= 1
            if indeg[v] == 0:
                heapq.heappush(ready, v)
    if len(order) != len(g.nodes):
        raise IRError("graph has a cycle")
    return order
