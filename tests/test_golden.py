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
