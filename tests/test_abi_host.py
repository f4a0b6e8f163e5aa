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
    for k in (0, 65):  # batch_shards in [1, 64]
        with pytest.raises(duet.DuetError) as e:
            duet.Graph("%x = input() : f32[2]\n").partition(batch_shards=k)
        assert e.value.name == "EINVAL"
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


# ---- batch_shards = k ---------------------------------------------------
def _same_sharded(ir, gran, k):
    dp = duet.Graph(ir).partition(gran, batch_shards=k)
    p = dp.export()
    o = o_partition(ir, gran, batch_shards=k)
    assert p["node_to_sg"] == o.node_to_sg and p["sg_phase"] == o.sg_phase
    assert p["phase_kind"] == o.phase_kind and p["edges"] == o.edges
    sh = dp.shards()
    assert sh["sg_shard"] == o.sg_shard and sh["sg_origin"] == o.sg_origin
    return dp, o


@pytest.mark.parametrize("cfg", ["c1", "c2", "c3", "c4", "c5", "c6"])
@pytest.mark.parametrize("k", [2, 3, 8])
def test_batch_shards_bit_exact_configs(cfg, k):
    """libduet's row-shard transform == the oracle's, on every config; c5 at k = 8 has the 8k + 1 = 65
    subgraphs of SURVEY.md §8(a) A0."""
    ir = W.build(cfg, small=not (cfg == "c5" and k == 8)).ir
    dp, o = _same_sharded(ir, "coarse", k)
    base = o_partition(ir)
    n_multi = sum(1 for s in range(base.n_sg) if base.phase_kind[base.sg_phase[s]] == 1)
    assert o.n_sg == base.n_sg + (k - 1) * n_multi
    if cfg == "c5":
        assert o.n_sg == 8 * k + 1
    # the shares of every boundary tensor add back up to the unsharded bytes
    agg = {}
    for (a, b), nb in o.edges.items():
        key = (o.sg_origin[a] if a >= 0 else -1, o.sg_origin[b] if b >= 0 else -1)
        agg[key] = agg.get(key, 0) + nb
    # (an edge between a sharded and an unsharded subgraph splits into k shares; shard-to-shard
    # edges pair equal indices: either way the parts sum to the unsharded bytes)
    assert agg == base.edges


@pytest.mark.parametrize("seed", range(30))
def test_batch_shards_bit_exact_fuzz(seed):
    rng = random.Random(5000 + seed)
    ir = random_dag_ir(rng, rng.randint(2, 14), rng.randint(1, 3))
    gran = rng.choice(["coarse", "op"])
    k = rng.choice([2, 3, 4, 7])
    dp, o = _same_sharded(ir, gran, k)
    if o.n_sg > 24:   # the Python greedy-correction is O(n^3) model evaluations: partition only
        return
    D = rng.choice([2, 3, 4])
    slot_gpu = list(range(D))
    T = [[rng.randint(1, 40) * 1000 for _ in range(D)] for _ in range(o.n_sg)]
    comm = Comm(Link(rng.randint(0, 3000), rng.randint(0, 3)), Link(rng.randint(0, 9000), rng.randint(0, 500)))
    os_ = o_schedule(o, T, slot_gpu, comm)
    e = dp.profile_from_table(slot_gpu, T, ((comm.same_gpu.alpha_ns, comm.same_gpu.ps_per_byte),
                                            (comm.cross_gpu.alpha_ns, comm.cross_gpu.ps_per_byte))).schedule().export()
    assert e["slot_of"] == os_.slot_of and e["makespan"] == os_.makespan and e["fell_back"] == os_.fell_back


def test_batch_shards_hand_case():
    """x -> {a, b} -> j with k = 3: a and b become shards 0..2 (ids 0-2 and 3-5), j is 6.
    x is f32[6,4] (96 B): each shard of a reads 32 B; a's output f32[6,2] (48 B) reaches j as
    16 B per shard; the unsharded output j f32[6,1] leaves whole (24 B).  Shares of 10 B over
    k = 3 are 3, 3, 4 (floor(10 (j+1) / 3) - floor(10 j / 3))."""
    from oracle.partition import share
    ir = ("%x = input() : f32[6,4]\n%a = opaque(%x) : f32[6,2]\n%b = opaque(%x) : f32[6,3]\n"
          "%j = opaque(%a, %b) : f32[6,1]\noutput %j\n")
    dp, o = _same_sharded(ir, "coarse", 3)
    assert o.n_sg == 7 and o.sg_shard == [0, 1, 2, 0, 1, 2, -1] and o.sg_origin == [0, 0, 0, 1, 1, 1, 2]
    assert o.node_to_sg == [-1, 0, 3, 6]
    assert o.edges[(-1, 0)] == 32 and o.edges[(-1, 5)] == 32
    assert o.edges[(1, 6)] == 16 and o.edges[(4, 6)] == 24 and o.edges[(6, -1)] == 24
    assert [share(10, j, 3) for j in range(3)] == [3, 3, 4]
    with pytest.raises(duet.DuetError) as e:
        dp.profile([(0, 0)])
    assert e.value.name == "EUNSUPPORTED"
    with pytest.raises(duet.DuetError):
        duet.Graph(ir).partition(batch_shards=0)
