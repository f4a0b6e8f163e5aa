"""Oracle makespan model, greedy-correction scheduler, fallback and brute force
(test infrastructure only; see oracle/__init__.py).

PAPER.md:81 (§IV-C) and Algorithm 1: Step 1 places the critical path on the
fastest device, Step 2 greedily places the remaining subgraphs "to the device that minimizes the
increase of the critical path", Step 3 refines each multi-path phase by KL-like swaps / single
moves, terminating after x rounds without a decrease.  PAPER.md:71/:90: fall back to the best
single device.  PAPER.md:88: the exhaustive optimum ("Ideal").

Devices generalise to D slots (slot = (gpu, stream)).  The paper's `measure latency` is the
integer makespan model C3 (R-6, "model mode").  All arithmetic is int64 ns with the
explicit tie-breaks of SURVEY.md §8(c) C3/C4 (R-1..R-16).
"""
from __future__ import annotations

import itertools
from dataclasses import dataclass

from .partition import MULTI, SEQ, Partition


@dataclass
class Link:
    alpha_ns: int = 0
    ps_per_byte: int = 0


@dataclass
class Comm:
    same_gpu: Link
    cross_gpu: Link


@dataclass
class Schedule:
    slot_of: list
    order: list
    makespan: int
    fell_back: int


class Model:
    """C3: phase-barriered list schedule over independent slots (integer ns)."""

    def __init__(self, part: Partition, T, slot_gpu, comm: Comm):
        self.p = part
        self.T = [list(map(int, row)) for row in T]
        self.D = len(slot_gpu)
        self.slot_gpu = list(slot_gpu)
        self.comm = comm
        n = part.n_sg
        self.preds = [[] for _ in range(n)]
        self.succs = [[] for _ in range(n)]
        self.in_bytes = [None] * n
        self.out_bytes = [None] * n
        for (u, v), b in part.edge_list():
            if u == -1:
                self.in_bytes[v] = b
            elif v == -1:
                self.out_bytes[u] = b
            else:
                self.preds[v].append((u, b))
                self.succs[u].append((v, b))
        self.phases = [[] for _ in range(part.n_phase)]
        for s in range(n):
            self.phases[part.sg_phase[s]].append(s)

    def c(self, d_from: int, d_to: int, nbytes: int) -> int:
        """Comm cost: 0 on the same slot, alpha + ceil(bytes * ps / 1000) otherwise."""
        if d_from == d_to:
            return 0
        link = self.comm.same_gpu if self.slot_gpu[d_from] == self.slot_gpu[d_to] else self.comm.cross_gpu
        return link.alpha_ns + (nbytes * link.ps_per_byte + 999) // 1000

    def _simulate_phase(self, a, p, phase_start, finish, only=None):
        free = [phase_start] * self.D
        pe = phase_start
        for s in self.phases[p]:
            if a[s] < 0 or (only is not None and s not in only):
                continue
            d = a[s]
            ready = 0
            if self.in_bytes[s] is not None:
                ready = self.c(0, d, self.in_bytes[s])
            for u, b in self.preds[s]:
                if u in finish:
                    ready = max(ready, finish[u] + self.c(a[u], d, b))
            start = max(free[d], ready)
            finish[s] = start + self.T[s][d]
            free[d] = finish[s]
            pe = max(pe, finish[s])
        return pe, free

    def makespan(self, a) -> int:
        finish = {}
        t = 0
        for p in range(len(self.phases)):
            t, _ = self._simulate_phase(a, p, t, finish)
        m = t
        for s, b in enumerate(self.out_bytes):
            if b is not None:
                m = max(m, finish[s] + self.c(a[s], 0, b))
        return m

    def partial(self, a, p):
        """Step 2's objective: phases < p complete; phase p with placed subgraphs only.
        Returns (phase_end, free-per-slot)."""
        finish = {}
        t = 0
        for q in range(p):
            t, _ = self._simulate_phase(a, q, t, finish)
        return self._simulate_phase(a, p, t, finish)

    def comm_in(self, a, s, d) -> int:
        r = 0
        if self.in_bytes[s] is not None:
            r = self.c(0, d, self.in_bytes[s])
        for u, b in self.preds[s]:
            if a[u] >= 0:
                r = max(r, self.c(a[u], d, b))
        return r

    def critical_path_lb(self) -> int:
        """Longest path with weights min_d T[s][d] and no comm (lower bound on any makespan)."""
        n = self.p.n_sg
        best = [0] * n
        for s in range(n):  # ids are topological
            w = min(self.T[s])
            best[s] = w + max((best[u] for u, _ in self.preds[s]), default=0)
        return max(best, default=0)

    def phase_cp_sum(self) -> int:
        tot = 0
        for ph in self.phases:
            best = {}
            for s in ph:
                w = min(self.T[s])
                best[s] = w + max((best[u] for u, _ in self.preds[s] if u in best), default=0)
            tot += max(best.values())
        return tot


def _argmin_place(m: Model, a, s):
    return min(range(m.D), key=lambda d: (m.T[s][d], m.comm_in(a, s, d), d))


def _phase_chain(m: Model, p, cost):
    """Step 1 (multi-path): s* = argmax cost (ties: smallest id) and the longest intra-phase
    chain through it by cost (ties: smallest id)."""
    ph = m.phases[p]
    inph = set(ph)
    s_star = max(ph, key=lambda s: (cost[s], -s))
    dp_in, dp_out = {}, {}
    for s in ph:
        dp_in[s] = cost[s] + max((dp_in[u] for u, _ in m.preds[s] if u in inph), default=0)
    for s in reversed(ph):
        dp_out[s] = cost[s] + max((dp_out[v] for v, _ in m.succs[s] if v in inph), default=0)
    chain = [s_star]
    cur = s_star
    while True:
        ps = [u for u, _ in m.preds[cur] if u in inph]
        if not ps:
            break
        cur = max(ps, key=lambda u: (dp_in[u], -u))
        chain.append(cur)
    cur = s_star
    while True:
        ss = [v for v, _ in m.succs[cur] if v in inph]
        if not ss:
            break
        cur = max(ss, key=lambda v: (dp_out[v], -v))
        chain.append(cur)
    return sorted(set(chain))


def greedy(m: Model):
    """Steps 1 and 2 for every phase in order."""
    n = m.p.n_sg
    a = [-1] * n
    for p, ph in enumerate(m.phases):
        if m.p.phase_kind[p] == SEQ:
            for s in ph:
                a[s] = _argmin_place(m, a, s)
            continue
        cost = {s: min(m.T[s]) for s in ph}
        for s in _phase_chain(m, p, cost):
            a[s] = _argmin_place(m, a, s)
        # Step 2: Kahn over the unplaced, priority (cost desc, id asc)
        rem = [s for s in ph if a[s] < 0]
        remset = set(rem)
        indeg = {s: sum(1 for u, _ in m.preds[s] if u in remset) for s in rem}
        done = set()
        while len(done) < len(rem):
            ready = [s for s in rem if s not in done and indeg[s] == 0]
            s = min(ready, key=lambda x: (-cost[x], x))
            before, _ = m.partial(a, p)
            best = None
            for d in range(m.D):
                a[s] = d
                after, free = m.partial(a, p)
                key = (after - before, free[d], m.T[s][d], d)
                if best is None or key < best:
                    best = key
            a[s] = best[3]
            done.add(s)
            for v, _ in m.succs[s]:
                if v in indeg:
                    indeg[v] -= 1
    return a


def correct(m: Model, a, p, rounds: int = 1, trace=None):
    """Step 3 (Algorithm 1) on multi-path phase p, in model mode.  `trace` (a list, optional)
    receives one (M, kind, i, d-or-j, accepted) tuple per inner iteration, in order."""
    a = list(a)
    t_old = m.makespan(a)
    ph = m.phases[p]
    idle = 0
    while True:
        improved = False
        U = list(ph)
        while U:
            best = None
            for i in U:
                for d in range(m.D):
                    if d == a[i]:
                        continue
                    b = list(a)
                    b[i] = d
                    key = (m.makespan(b), 0, i, d)
                    if best is None or key < best:
                        best = key
            for x, i in enumerate(U):
                for j in U[x + 1:]:
                    if a[i] == a[j]:
                        continue
                    b = list(a)
                    b[i], b[j] = a[j], a[i]
                    key = (m.makespan(b), 1, i, j)
                    if best is None or key < best:
                        best = key
            if best is None:
                break
            t_new, kind, i, y = best
            U = [s for s in U if s != i and not (kind == 1 and s == y)]
            if trace is not None:
                trace.append((t_new, kind, i, y, t_new < t_old))
            if t_new < t_old:
                if kind == 0:
                    a[i] = y
                else:
                    a[i], a[y] = a[y], a[i]
                t_old = t_new
                improved = True
        idle = 0 if improved else idle + 1
        if idle >= rounds:
            break
    return a


def lowbias32(x: int) -> int:
    """32-bit integer hash (the seeded random placement of the Fig. 13 baselines, R-29)."""
    x &= 0xFFFFFFFF
    x ^= x >> 16
    x = (x * 0x7FEB352D) & 0xFFFFFFFF
    x ^= x >> 15
    x = (x * 0x846CA68B) & 0xFFFFFFFF
    x ^= x >> 16
    return x


def schedule(part: Partition, T, slot_gpu, comm: Comm, mode: int = 0, correction_rounds: int = 1,
             allow_fallback: bool = True, fixed=None, seed: int = 0, trace=None) -> Schedule:
    """mode 0 greedy-correction, 1 greedy only, 2 serial (home slot 0), 3 fixed; Fig. 13
    baselines: 4 random, 5 round-robin, 6 random + correction."""
    m = Model(part, T, slot_gpu, comm)
    n = part.n_sg
    fell = 0
    if mode == 2:
        a = [0] * n
    elif mode == 3:
        a = [int(x) for x in fixed]
    else:
        if mode in (4, 6):
            a = [lowbias32((seed * 0x9E3779B1 + s) & 0xFFFFFFFF) % m.D for s in range(n)]
        elif mode == 5:
            a = [s % m.D for s in range(n)]
        else:
            a = greedy(m)
        if mode in (0, 6):
            for p in range(part.n_phase):
                if part.phase_kind[p] == MULTI:
                    a = correct(m, a, p, correction_rounds, trace)
        if allow_fallback:
            m_gc = m.makespan(a)
            singles = [(m.makespan([d] * n), d) for d in range(m.D)]
            m1, d1 = min(singles)
            if m1 <= m_gc:
                a = [d1] * n
                fell = 1
    return Schedule(a, list(range(n)), m.makespan(a), fell)


def brute_force(part: Partition, T, slot_gpu, comm: Comm):
    """C5 'Ideal': min over all D^n assignments; ties -> lexicographically first."""
    m = Model(part, T, slot_gpu, comm)
    best = None
    for a in itertools.product(range(m.D), repeat=part.n_sg):
        ms = m.makespan(list(a))
        if best is None or ms < best[0]:
            best = (ms, list(a))
    return best


def brute_force_symmetric(part: Partition, T, slot_gpu, comm: Comm):
    """C5 for D interchangeable non-home slots (8 identical GPUs x 1 stream
    over NVSwitch).  Only canonical assignments are evaluated: set partitions of the subgraphs
    with one distinguished home block (slot 0, where graph inputs live and outputs must return,
    C3) and at most D-1 unlabeled non-home blocks, labeled 1, 2, ... in order of first use
    (restricted growth strings).  Valid only when relabeling slots 1..D-1 changes no cost: every
    subgraph has equal T on those slots and they are all on distinct GPUs other than slot 0's, or
    all on slot 0's GPU.  Returns (min makespan, first canonical assignment reaching it)."""
    m = Model(part, T, slot_gpu, comm)
    D, n = m.D, part.n_sg
    for row in m.T:
        if any(row[d] != row[1] for d in range(2, D)):
            raise ValueError("non-home slots must have identical costs")
    rest = m.slot_gpu[1:]
    if not (all(g == m.slot_gpu[0] for g in rest)
            or (len(set(rest)) == len(rest) and m.slot_gpu[0] not in rest)):
        raise ValueError("non-home slots must all share slot 0's GPU or all sit on distinct other GPUs")
    best = None
    a = [0] * n

    def rec(s, used):
        nonlocal best
        if s == n:
            ms = m.makespan(a)
            if best is None or ms < best[0]:
                best = (ms, list(a))
            return
        for d in range(0, min(used + 1, D - 1) + 1):
            a[s] = d
            rec(s + 1, max(used, d))

    rec(0, 0)
    return best


def canonical_count(n: int, D: int) -> int:
    """Number of assignments brute_force_symmetric evaluates (the enumeration alone)."""
    cnt = 0

    def rec(s, used):
        nonlocal cnt
        if s == n:
            cnt += 1
            return
        for d in range(0, min(used + 1, D - 1) + 1):
            rec(s + 1, max(used, d))

    rec(0, 0)
    return cnt
