"""CPU-side checks of the C ABI (no GPU needed): libduet.so loads and exports every entry point
declared in include/duet.h; IR errors map to status codes; partitions and schedules computed by
the C++ library are bit-identical to the oracle (BASELINE.json:5 "Schedules and partitions must be
bit-exact for the same profile table")."""
import os
import random
import re

import pytest

from oracle.partition import partition as o_partition
from oracle.schedule import Comm, Link, schedule as o_schedule
from paper_conf_ipps_zhanghl21_b200 import duet
from paper_conf_ipps_zhanghl21_b200 import workloads as W

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_exports_every_declared_symbol():
    hdr = open(os.path.join(ROOT, "include", "duet.h")).read()
    hdr = re.sub(r"/\*.*?\*/", "", hdr, flags=re.S)
    declared = set(re.findall(r"\b(duet_[a-z_]+)\s*\(", hdr))
    assert len(declared) >= 19
    import ctypes
    lib = ctypes.CDLL(duet.LIB_PATH)
    for name in declared:
        assert hasattr(lib, name), name
    assert set(duet.EXPORTED) == declared
    assert duet.abi_version() == 2


@pytest.mark.parametrize("ir,code", [
    ("%a = add(%b, %b) : f32[1]\n%b = add(%a, %a) : f32[1]\n", "ECYCLE"),
    ("%a = linear(%x, @W, @b) : f32[1]\n", "EPARSE"),
    ("%a = input() : f16[1]\n", "EPARSE"),
    ("%a input() : f32[1]\n", "EPARSE"),
])
def test_ir_errors(ir, code):
    with pytest.raises(duet.DuetError) as e:
        duet.Graph(ir)
    assert e.value.name == code


def test_bind_checks_shape_dtype():
    import torch
    g = duet.Graph("param @W : f32[2,3]\n%x = input() : f32[1,3]\n%y = linear(%x, @W, @b) : f32[1,2]\n"
                   "param @b : f32[2]\noutput %y\n")
    with pytest.raises(duet.DuetError) as e:
        g.bind("W", torch.zeros(3, 2))  # host tensor and wrong shape
    assert e.value.name in ("ESHAPE", "EINVAL")
    with pytest.raises(duet.DuetError) as e:
        g.bind("W", torch.zeros(2, 3, dtype=torch.bfloat16))
    assert e.value.name == "EDTYPE"
    with pytest.raises(duet.DuetError) as e:
        g.bind("nope", torch.zeros(2))
    assert e.value.name == "EINVAL"
    assert g.info() == {"n_nodes": 2, "n_inputs": 1, "n_outputs": 1, "n_params": 2}


def _same_partition(ir, gran):
    p = duet.Graph(ir).partition(gran).export()
    o = o_partition(ir, gran)
    assert p["node_to_sg"] == o.node_to_sg
    assert p["sg_phase"] == o.sg_phase
    assert p["phase_kind"] == o.phase_kind
    assert p["edges"] == o.edges
    return p, o


@pytest.mark.parametrize("cfg", list(W.CONFIGS))
@pytest.mark.parametrize("small", [True, False])
@pytest.mark.parametrize("gran", ["coarse", "op"])
def test_partition_bit_exact_configs(cfg, small, gran):
    _same_partition(W.build(cfg, small=small).ir, gran)


@pytest.mark.parametrize("var", [dict(rnn_layers=8), dict(resnet=34), dict(resnet=50), dict(resnet=101),
                                 dict(ffn_layers=8), dict(batch=2)])
@pytest.mark.parametrize("gran", ["coarse", "op"])
def test_partition_bit_exact_model_variations(var, gran):
    """PAPER.md:89 §VI-D variations of c4 (full size): libduet's partition == the oracle's; at
    coarse granularity the branches stay one subgraph each (CNN, RNN, FFN + join)."""
    p, _ = _same_partition(W.build("c4", **var).ir, gran)
    if gran == "coarse":
        assert p["n_sg"] == 4


def random_dag_ir(rng, n_nodes, n_inputs=2):
    lines = [f"%x{i} = input() : f32[8,{4 + i}]" for i in range(n_inputs)]
    names = []
    for i in range(n_nodes):
        k = rng.randint(0, min(3, len(names)))
        srcs = rng.sample(names, k) if k else []
        if not srcs or rng.random() < 0.2:
            srcs.append(f"x{rng.randrange(n_inputs)}")
        lines.append(f"%n{i} = opaque({', '.join('%' + s for s in srcs)}) : f32[8,{rng.randint(1, 64)}]")
        names.append(f"n{i}")
    outs = rng.sample(names, min(len(names), rng.randint(1, 3)))
    lines.append("output " + ", ".join("%" + n for n in outs))
    rng.shuffle(lines)  # definitions may come in any order
    return "\n".join(lines) + "\n"


@pytest.mark.parametrize("seed", range(60))
def test_partition_and_schedule_bit_exact_fuzz(seed):
    rng = random.Random(1000 + seed)
    ir = random_dag_ir(rng, rng.randint(2, 16), rng.randint(1, 3))
    gran = rng.choice(["coarse", "op"])
    p, o = _same_partition(ir, gran)
    n = o.n_sg
    D = rng.choice([1, 2, 3, 4, 8])
    slot_gpu = sorted(rng.randint(0, 2) for _ in range(D))
    slot_gpu[0] = 0
    T = [[rng.randint(0, 60) * 997 for _ in range(D)] for _ in range(n)]
    comm = ((rng.randint(0, 3000), rng.randint(0, 5)), (rng.randint(0, 9000), rng.randint(0, 700)))
    part = duet.Graph(ir).partition(gran)
    prof = part.profile_from_table(slot_gpu, T, comm)
    oc = Comm(Link(*comm[0]), Link(*comm[1]))
    for mode in (0, 1, 2, 4, 5, 6):
        for rounds in ((1, 2) if mode in (0, 6) else (1,)):
            for fb in (True, False):
                s = prof.schedule(mode=mode, correction_rounds=rounds, allow_fallback=fb, seed=seed).export()
                os_ = o_schedule(o, T, slot_gpu, oc, mode=mode, correction_rounds=rounds, allow_fallback=fb,
                                 seed=seed)
                assert s["slot_of"] == os_.slot_of, (mode, rounds, fb)
                assert s["makespan"] == os_.makespan
                assert s["fell_back"] == os_.fell_back
                assert s["order"] == os_.order
    fixed = [rng.randrange(D) for _ in range(n)]
    s = prof.schedule(mode=3, fixed=fixed).export()
    assert s["slot_of"] == fixed
    assert s["makespan"] == o_schedule(o, T, slot_gpu, oc, mode=3, fixed=fixed).makespan


def test_table2_and_lpt_fixtures_through_abi():
    ir2 = "%x = input() : f32[4,4]\n%rnn = opaque(%x) : f32[4,1]\n%cnn = opaque(%x) : f32[4,2]\noutput %rnn, %cnn\n"
    pr = duet.Graph(ir2).partition().profile_from_table([0, 1], [[2_400_000, 6_400_000], [14_900_000, 900_000]])
    s = pr.schedule().export()
    assert s["slot_of"] == [0, 1] and s["makespan"] == 2_400_000 and s["fell_back"] == 0
    ir5 = "%x = input() : f32[4,4]\n" + "".join(f"%b{i} = opaque(%x) : f32[4,{i + 1}]\n" for i in range(5))
    ir5 += "output " + ", ".join(f"%b{i}" for i in range(5)) + "\n"
    pr = duet.Graph(ir5).partition().profile_from_table([0, 0], [[t, t] for t in (7000, 6000, 5000, 4000, 3000)])
    assert pr.schedule(mode=1, allow_fallback=False).export()["slot_of"] == [0, 1, 1, 0, 0]
    s = pr.schedule().export()
    assert s["slot_of"] == [1, 0, 1, 0, 0] and s["makespan"] == 13000


def test_state_errors():
    part = duet.Graph("%x = input() : f32[2]\n%y = opaque(%x) : f32[2]\noutput %y\n").partition()
    with pytest.raises(duet.DuetError) as e:
        part.profile_from_table([0], [[-1]])
    assert e.value.name == "EINVAL"
    with pytest.raises(duet.DuetError) as e:
        duet.Graph("%x = input() : f32[2]\n").partition(batch_shards=2)
    assert e.value.name == "EUNSUPPORTED"
    s = part.profile_from_table([0], [[5]]).schedule()
    with pytest.raises(duet.DuetError) as e:
        s.launch_count()
    assert e.value.name == "ESTATE"


@pytest.mark.parametrize("cfg", ["c3", "c4", "c5"])
def test_rnn_tile_n_rewrite(cfg):
    """with_rnn_tile_n sets / clears the tile_n attribute on exactly the LSTM/GRU nodes, keeps
    their other attributes, and leaves the partition (the IR's structure) unchanged."""
    wl = W.build(cfg, small=True, **({"rnn_layers": 2} if cfg == "c4" else {}))
    rnn = W.rnn_nodes(wl)
    assert rnn
    w128 = W.with_rnn_tile_n(wl, 128)
    lines0, lines1 = wl.ir.splitlines(), w128.ir.splitlines()
    assert len(lines0) == len(lines1)
    for a, b in zip(lines0, lines1):
        if any(a.startswith(f"%{n} = ") for n in rnn):
            assert "tile_n=128" in b and b.replace(", tile_n=128", "").replace(" {tile_n=128}", "") == a
        else:
            assert a == b
    assert W.with_rnn_tile_n(w128, 0).ir == wl.ir
    assert w128.meta["rnn_tile_n"] == 128
    p0 = duet.Graph(wl.ir).partition("coarse").export()
    p1 = duet.Graph(w128.ir).partition("coarse").export()
    assert p0 == p1
