"""Branch placement across GPUs (paper_conf_ipps_zhanghl21_b200/multigpu.py):
host-side planning checked on CPU.  The pieces are evaluated with the float64 oracle (no GPU here),
so "split == whole" pins the cut: a dropped edge, a wrong phase order or a missing transfer
changes the result.  World-size-2 gloo run of the executor's point-to-point protocol."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

from oracle import forward as OF
from paper_conf_ipps_zhanghl21_b200 import duet
from paper_conf_ipps_zhanghl21_b200 import multigpu as MG
from paper_conf_ipps_zhanghl21_b200 import workloads as W
from tests.helpers import to_np


def _c5_plan(n_gpu=2, home=0):
    wl = W.build("c5", small=True)
    part = duet.Graph(wl.ir).partition().export()
    kinds = part["phase_kind"]
    # multi-path subgraphs round-robin over the GPUs, sequential ones (the join) at home
    sg_gpu = [(s % n_gpu) if kinds[part["sg_phase"][s]] == 1 else home for s in range(part["n_sg"])]
    return wl, part, sg_gpu, MG.plan(wl.ir, part["node_to_sg"], part["sg_phase"], sg_gpu, home)


def test_plan_covers_every_node_once_and_pieces_compile():
    wl, part, sg_gpu, pl = _c5_plan(2)
    ir = MG.parse_ir(wl.ir)
    placed = [n for pc in pl.pieces for n in pc.nodes]
    compute = [n.name for n in ir.nodes if n.op != "input"]
    assert sorted(placed) == sorted(compute) and len(placed) == len(set(placed))
    assert {pc.gpu for pc in pl.pieces} == {0, 1}
    for pc in pl.pieces:
        g = duet.Graph(pc.ir)           # libduet parses every piece
        info = g.info()
        assert info["n_inputs"] == len(pc.inputs) and info["n_outputs"] == len(pc.outputs)
    # inputs go home -> the branch's GPU before phase 0, branch logits come back before the join
    for t in pl.transfers:
        assert t.src != t.dst
        if t.tensor in pl.graph_inputs:
            assert t.src == 0 and t.dst == 1 and t.phase == 0
        else:
            assert t.src == 1 and t.dst == 0
    assert pl.n_phases == len(part["phase_kind"])


def _oracle_params(wl):
    return {k: to_np(s.materialize()) for k, s in wl.params.items()}


def _piece_runner(params):
    def run(pc, ins):
        sub = {k: params[k] for k in MG.parse_ir(pc.ir).params}
        out = OF.run(pc.ir, sub, {k: to_np(v) if isinstance(v, torch.Tensor) else v for k, v in ins.items()},
                     keep_all=True)
        return {o: out[o] for o in pc.outputs}
    return run


@pytest.mark.parametrize("n_gpu", [2, 3, 8])
def test_split_equals_whole_oracle(n_gpu):
    wl, part, sg_gpu, pl = _c5_plan(n_gpu)
    params = _oracle_params(wl)
    inputs = {k: to_np(s.materialize()) for k, s in wl.inputs.items()}
    run = _piece_runner(params)
    store = dict(inputs)
    for phase in range(pl.n_phases):
        for pc in pl.pieces:
            if pc.phase == phase:
                store.update(run(pc, {a: store[a] for a in pc.inputs}))
    whole = OF.run(wl.ir, params, inputs)
    # a cut-edge tensor crosses as a piece input in its declared dtype (f32 logits here), which the
    # oracle rounds like stored data; the unsplit oracle keeps it in float64: fp32-rounding agreement
    for o in pl.graph_outputs:
        np.testing.assert_allclose(np.asarray(store[o]), np.asarray(whole[o]), rtol=1e-6, atol=0)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out_dir):
    os.environ.update(RANK=str(rank), WORLD_SIZE=str(world), LOCAL_RANK=str(rank), MASTER_ADDR="127.0.0.1",
                      MASTER_PORT=str(port))
    from paper_conf_ipps_zhanghl21_b200 import multirank as MR
    assert MR.init("gloo")
    wl, part, sg_gpu, pl = _c5_plan(world)
    params = _oracle_params(wl)
    run = _piece_runner(params)

    # the executor moves torch tensors: bf16 graph inputs as their int16 bit patterns, computed
    # tensors as the oracle's float64 values
    def np_of(t):
        return t.numpy().view(np.uint16) if t.dtype == torch.int16 else t.numpy()

    def run_t(pc, ins):
        return {k: torch.from_numpy(np.ascontiguousarray(v)) for k, v in run(pc, {a: np_of(t) for a, t in ins.items()}).items()}

    def alloc(dt, shape):
        if dt == "bf16" and any(t for t in pl.graph_inputs if pl.tensor_meta[t] == (dt, tuple(shape))):
            return torch.empty(shape, dtype=torch.int16)
        return torch.empty(shape, dtype=torch.float64 if dt in ("f32", "bf16") else MG.TORCH_DT[dt])

    ex = MG.Executor(pl, rank, run_t, alloc=alloc)
    ins = None
    if rank == 0:
        ins = {}
        for k, s in wl.inputs.items():
            a = np.ascontiguousarray(to_np(s.materialize()))
            ins[k] = torch.from_numpy(a.view(np.int16) if a.dtype == np.uint16 else a)
    outs = ex.step(ins)
    res = {}
    if rank == 0:
        inputs = {k: to_np(s.materialize()) for k, s in wl.inputs.items()}
        whole = OF.run(wl.ir, params, inputs)
        res["equal"] = all(np.allclose(o.numpy(), whole[n], rtol=1e-6, atol=0) for o, n in zip(outs, pl.graph_outputs))
    res["ran"] = sorted(n for pc in pl.pieces_on(rank) for n in pc.nodes)
    MR.barrier()
    MR.finalize()
    torch.save(res, os.path.join(out_dir, f"r{rank}.pt"))


def test_world2_gloo_branch_placement(tmp_path):
    port = _free_port()
    mp.spawn(_worker, args=(2, port, str(tmp_path)), nprocs=2, join=True)
    r0 = torch.load(tmp_path / "r0.pt")
    r1 = torch.load(tmp_path / "r1.pt")
    assert r0["equal"]
    assert r0["ran"] and r1["ran"] and not set(r0["ran"]) & set(r1["ran"])
