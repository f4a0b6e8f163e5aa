"""Golden fixtures under tests/golden/ (each file cites its passage): the paper's Table II numbers
(PAPER.md:87), the hand-traced LPT counter-example and the hand-computed 2-layer
toy net (BASELINE.json:5).  Checked against the oracle and, for the schedules, against libduet
through the C ABI (host-side, no GPU)."""
import os

import numpy as np
import pytest
import torch

from oracle import forward as F
from oracle.partition import partition
from oracle.schedule import Comm, Link, brute_force, schedule
from paper_conf_ipps_zhanghl21_b200 import duet

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")
ZERO = Comm(Link(0, 0), Link(0, 0))


def load(name):
    d, t = {}, []
    for line in open(os.path.join(GOLDEN, name)):
        line = line.split("#", 1)[0].split()
        if not line:
            continue
        if line[0] == "t_ns":
            t.append((int(line[1]), [int(v) for v in line[2:]]))
        else:
            d[line[0]] = [float(v) if "." in v or "e" in v else int(v) for v in line[1:]]
    if t:
        d["t_ns"] = [row for _, row in sorted(t)]
    return d


def branches_ir(n):
    lines = ["%x = input() : f32[4,4]"] + [f"%b{i} = opaque(%x) : f32[4,{i + 1}]" for i in range(n)]
    return "\n".join(lines + ["output " + ", ".join(f"%b{i}" for i in range(n))]) + "\n"


@pytest.mark.parametrize("name", ["table2_cpu_gpu.txt", "lpt_counterexample.txt"])
def test_schedule_golden_oracle_and_abi(name):
    g = load(name)
    T, slot_gpu = g["t_ns"], g["slot_gpu"]
    ir = branches_ir(len(T))
    p = partition(ir)
    s = schedule(p, T, slot_gpu, ZERO)
    assert s.slot_of == g["expect_slot_of"]
    assert s.makespan == g["expect_makespan_ns"][0]
    assert s.fell_back == g["expect_fell_back"][0]
    assert brute_force(p, T, slot_gpu, ZERO)[0] == g["expect_brute_force_ns"][0]
    if "expect_greedy_slot_of" in g:
        gr = schedule(p, T, slot_gpu, ZERO, mode=1, allow_fallback=False)
        assert gr.slot_of == g["expect_greedy_slot_of"]
        assert gr.makespan == g["expect_greedy_makespan_ns"][0]
    # the C++ scheduler through the C ABI
    pr = duet.Graph(ir).partition().profile_from_table(slot_gpu, T)
    e = pr.schedule().export()
    assert e["slot_of"] == g["expect_slot_of"] and e["makespan"] == g["expect_makespan_ns"][0]
    assert e["fell_back"] == g["expect_fell_back"][0]


TOY = """
param @W1 : {dt}[2,2]
param @b1 : f32[2]
param @W2 : {dt}[1,2]
param @b2 : f32[1]
%x = input() : {dt}[1,2]
%h = linear(%x, @W1, @b1) {{act=relu}} : {dt}[1,2]
%y = linear(%h, @W2, @b2) {{act=sigmoid}} : f32[1,1]
output %y
"""


@pytest.mark.parametrize("dt", ["f32", "bf16"])
def test_toy_mlp_golden(dt):
    g = load("toy_mlp.txt")

    def enc(v, shape):
        a = np.asarray(v, dtype=np.float32).reshape(shape)
        if dt == "bf16":
            return torch.tensor(a).to(torch.bfloat16).view(torch.int16).numpy().view(np.uint16)
        return a

    params = {"W1": enc(g["W1"], (2, 2)), "b1": np.float32(g["b1"]), "W2": enc(g["W2"], (1, 2)),
              "b2": np.float32(g["b2"])}
    out = F.run(TOY.format(dt=dt), params, {"x": enc(g["x"], (1, 2))}, keep_all=True)
    np.testing.assert_array_equal(np.asarray(out["h"], dtype=np.float64).ravel(), g["expect_h"])
    assert out["y"][0, 0] == pytest.approx(g["expect_y"][0], rel=1e-15)


def fig8_ir():
    """The constructed Fig. 8 graph (tests/golden/fig8_swap.txt): head, branches b1..b6 (subgraph
    ids 1..6 = the figure's), join; b6's output is 2000 B, every other tensor 4 B."""
    lines = ["%x = input() : f32[1]", "%h = opaque(%x) : f32[1]"]
    lines += [f"%b{k} = opaque(%h) : f32[{500 if k == 6 else 1}]" for k in range(1, 7)]
    lines += ["%j = opaque(" + ", ".join(f"%b{k}" for k in range(1, 7)) + ") : f32[1]", "output %j"]
    return "\n".join(lines) + "\n"


def test_fig8_swap_golden():
    """PAPER.md:81 §IV-C Step 3 / Fig. 8: initial GPU = {1,3,6}, CPU = {2,4,5}; the first accepted
    correction is the pair (6, 5), avoiding b6's large output crossing devices."""
    from oracle.schedule import Model
    g = load("fig8_swap.txt")
    ir = fig8_ir()
    p = partition(ir)
    assert p.n_sg == 8 and p.sg_phase == [0, 1, 1, 1, 1, 1, 1, 2]
    assert p.edges[(6, 7)] == 2000 and p.edges[(5, 7)] == 4
    T, slot_gpu = g["t_ns"], g["slot_gpu"]
    comm = Comm(Link(0, 0), Link(g["comm_cross_alpha_ns"][0], g["comm_cross_ps_per_byte"][0]))
    gr = schedule(p, T, slot_gpu, comm, mode=1, allow_fallback=False)
    assert gr.slot_of == g["expect_greedy_slot_of"] and gr.makespan == g["expect_greedy_makespan_ns"][0]
    gpu = {s for s in range(1, 7) if gr.slot_of[s] == 1}
    cpu = {s for s in range(1, 7) if gr.slot_of[s] == 0}
    assert gpu == {1, 3, 6} and cpu == {2, 4, 5}
    trace = []
    s = schedule(p, T, slot_gpu, comm, trace=trace)
    m_first, kind, i, j, accepted = trace[0]
    assert [m_first, kind, i, j] == g["expect_first_correction"] and accepted
    assert [t for t in trace[1:] if t[4]] == []           # nothing else accepted
    assert s.slot_of == g["expect_slot_of"] and s.makespan == g["expect_makespan_ns"][0]
    assert s.fell_back == g["expect_fell_back"][0]
    m = Model(p, T, slot_gpu, comm)
    assert m.critical_path_lb() == g["expect_critical_path_lb_ns"][0]
    assert [m.makespan([d] * 8) for d in (0, 1)] == g["expect_single_slot_ns"]
    assert brute_force(p, T, slot_gpu, comm)[0] <= s.makespan
    # the C++ scheduler through the C ABI
    dp = duet.Graph(ir).partition()
    cm = ((0, 0), (g["comm_cross_alpha_ns"][0], g["comm_cross_ps_per_byte"][0]))
    pr = dp.profile_from_table(slot_gpu, T, comm=cm)
    e = pr.schedule(mode=duet.GREEDY_ONLY, allow_fallback=False).export()
    assert e["slot_of"] == g["expect_greedy_slot_of"]
    e = pr.schedule().export()
    assert e["slot_of"] == g["expect_slot_of"] and e["makespan"] == g["expect_makespan_ns"][0]
