"""World-size-2 gloo tests (CPU) of the multi-rank host path: max-over-ranks timing, contiguous row
shards, gathering shards on rank 0, and that every rank derives the identical partition/schedule
from the same profile table.  The per-shard compute is the oracle here (no
GPU on this box); inference rows are independent, so sharded == unsharded."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

from paper_conf_ipps_zhanghl21_b200 import multirank as MR


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out_dir):
    os.environ.update(RANK=str(rank), WORLD_SIZE=str(world), LOCAL_RANK=str(rank), MASTER_ADDR="127.0.0.1",
                      MASTER_PORT=str(port))
    from oracle import forward as OF
    from paper_conf_ipps_zhanghl21_b200 import duet
    from paper_conf_ipps_zhanghl21_b200 import workloads as W
    from tests.helpers import to_np

    assert MR.init("gloo")
    res = {}
    res["max"] = MR.max_over_ranks(10.0 + rank)
    # identical schedule on every rank from the same (partition, profile table)
    wl = W.build("c5", small=True)
    part = duet.Graph(wl.ir).partition()
    n = part.n_sg
    T = [[1000 * (s + 1), 1000 * (s + 1)] for s in range(n)]
    sched = part.profile_from_table([0, 0], T).schedule().export()
    objs = [None] * world
    torch.distributed.all_gather_object(objs, sched)
    res["same_schedule"] = all(o == objs[0] for o in objs)
    # row-sharded inference of c2-small: each rank evaluates its shard, rank 0 gathers
    wl2 = W.build("c2", small=True, dt="f32")
    params = {k: to_np(s.materialize()) for k, s in wl2.params.items()}
    raw = to_np(wl2.inputs["raw"].materialize())
    a, b = MR.shard_range(wl2.batch, world, rank)
    y_local = torch.tensor(OF.run(wl2.ir, params, {"raw": raw[a:b]})["y"])
    y = MR.gather_rows(y_local, wl2.batch)
    if rank == 0:
        full = OF.run(wl2.ir, params, {"raw": raw})["y"]
        res["gather_equal"] = bool(np.allclose(y.numpy(), full, rtol=1e-12, atol=0))  # BLAS blocking may differ by M
        res["rows"] = int(y.shape[0])
    MR.barrier()
    MR.finalize()
    torch.save(res, os.path.join(out_dir, f"r{rank}.pt"))


def test_world2_gloo(tmp_path):
    world = 2
    mp.spawn(_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world, join=True)
    r0 = torch.load(tmp_path / "r0.pt")
    r1 = torch.load(tmp_path / "r1.pt")
    assert r0["max"] == 11.0 and r1["max"] == 11.0
    assert r0["same_schedule"] and r1["same_schedule"]
    assert r0["gather_equal"] and r0["rows"] == 300


def _shard_worker(rank, world, port, out_dir):
    """ShardExecutor (bench.py's N > 1 strong-scaling step): rank 0's full c5-small batch is
    scattered in row blocks, each rank runs the float64 oracle on its rows (the GPU run uses
    libduet), the outputs are gathered back; the result must equal the oracle on the whole batch."""
    os.environ.update(RANK=str(rank), WORLD_SIZE=str(world), LOCAL_RANK=str(rank), MASTER_ADDR="127.0.0.1",
                      MASTER_PORT=str(port))
    from oracle import forward as OF
    from paper_conf_ipps_zhanghl21_b200 import workloads as W
    from tests.helpers import to_np

    assert MR.init("gloo")
    wl = W.build("c5", small=True, dt="f32", batch=8 * world)
    params = {k: to_np(s.materialize()) for k, s in wl.params.items()}
    full_in = [s.materialize() for s in wl.inputs.values()]
    in_meta = [(t.shape[1:], t.dtype) for t in full_in]
    out_meta = [(tuple(shape[1:]), torch.float32) for _, _, shape in wl.outputs]
    ex = MR.ShardExecutor(wl.batch, in_meta, out_meta, torch.device("cpu"))
    seen = {}

    def runner(shard_in, shard_out):
        seen["rows"] = int(shard_in[0].shape[0])
        got = OF.run(wl.ir, params, {k: to_np(t) for k, t in zip(wl.inputs, shard_in)})
        for (name, _, _), o in zip(wl.outputs, shard_out):
            o.copy_(torch.from_numpy(got[name]).to(o.dtype))

    outs = [torch.full((wl.batch,) + tuple(m[0]), float("nan")) for m in out_meta] if rank == 0 else None
    ex.step(full_in if rank == 0 else None, outs, runner)
    res = {"rows": seen["rows"], "bytes": ex.bytes_moved()}
    if rank == 0:
        want = OF.run(wl.ir, params, {k: to_np(t) for k, t in zip(wl.inputs, full_in)})
        res["equal"] = all(np.allclose(o.numpy(), want[name], rtol=1e-6, atol=1e-7)
                           for (name, _, _), o in zip(wl.outputs, outs))
        res["shard0_exact"] = bool(np.array_equal(outs[0][:8].numpy(), torch.from_numpy(
            OF.run(wl.ir, params, {k: to_np(t)[:8] for k, t in zip(wl.inputs, full_in)})[wl.outputs[0][0]]).float().numpy()))
    MR.barrier()
    MR.finalize()
    torch.save(res, os.path.join(out_dir, f"s{rank}.pt"))


@pytest.mark.parametrize("world", [2])
def test_shard_executor_gloo(tmp_path, world):
    mp.spawn(_shard_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world, join=True)
    r = [torch.load(tmp_path / f"s{k}.pt") for k in range(world)]
    assert all(x["rows"] == 8 for x in r)
    assert r[0]["equal"] and r[0]["shard0_exact"]
    sc, ga = r[0]["bytes"]
    assert sc > 0 and ga == (world - 1) * 8 * 4


def test_shard_executor_rejects_uneven_batch():
    ex = MR.ShardExecutor(7, [((3,), torch.float32)], [((1,), torch.float32)], torch.device("cpu"))
    assert ex.rows == 7 and ex.world == 1


@pytest.mark.parametrize("n,world", [(2048, 8), (300, 7), (5, 8), (0, 3), (4096, 1)])
def test_shard_range_partitions_rows(n, world):
    spans = [MR.shard_range(n, world, r) for r in range(world)]
    assert spans[0][0] == 0 and spans[-1][1] == n
    assert all(spans[i][1] == spans[i + 1][0] for i in range(world - 1))
    sizes = [b - a for a, b in spans]
    assert max(sizes) - min(sizes) <= 1


def test_single_process_noops():
    assert MR.max_over_ranks(3.5) == 3.5
    t = torch.arange(4)
    assert MR.gather_rows(t, 4) is t


@pytest.mark.gpu
def test_bench_two_ranks_on_one_gpu():
    """bench.py under torchrun with 2 ranks (the driver's N>1 launch): barrier, max-over-ranks timing
    and rank 0's single JSON line.  This box has one GPU, so both ranks sit on GPU 0 and the process
    group is gloo (DUET_FORCE_DEVICE / DUET_DIST_BACKEND; NCCL refuses two ranks per GPU)."""
    import json
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, DUET_DIST_BACKEND="gloo", DUET_FORCE_DEVICE="0")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2", "--master-addr",
           "127.0.0.1", "--master-port", "29541", "bench.py", "--config", "c1", "--gpus", "2", "--steps", "5",
           "--warmup", "3", "--no-cpu-baseline", "--profile-samples", "5", "--placement", "replica",
           "--tail-samples", "20"]
    r = subprocess.run(cmd, env=env, cwd=root, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-2000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["config"]["global_batch"] == 2 and d["value"] > 0


@pytest.mark.gpu
def test_bench_shard_two_ranks_on_one_gpu():
    """bench.py's N > 1 default (--placement shard) under torchrun with 2 ranks on GPU 0 over gloo:
    one global c2 batch scattered from rank 0 in row blocks, each rank's libduet schedule on its
    1024 rows, outputs gathered on rank 0 inside the timed step; one JSON line, strong scaling."""
    import json
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, DUET_DIST_BACKEND="gloo", DUET_FORCE_DEVICE="0")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2", "--master-addr",
           "127.0.0.1", "--master-port", "29545", "bench.py", "--config", "c2", "--gpus", "2", "--steps", "5",
           "--warmup", "3", "--profile-samples", "5"]
    r = subprocess.run(cmd, env=env, cwd=root, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-2000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["scaling"] == "strong" and d["config"]["global_batch"] == 2048
    assert d["config"]["per_gpu_batch"] == 1024 and d["collective_bytes_per_step"]["gather_to_rank0"] == 1024 * 4
    assert d["value"] > 0 and d["e2e"]["value"] > 0


@pytest.mark.gpu
def test_shard_parity_two_ranks_on_one_gpu(tmp_path):
    """The strong-scaling shard step's result: 2 ranks on GPU 0 (gloo) each run libduet on half of
    c5-small's batch; rank 0's gathered outputs must meet the float64 oracle on the whole batch."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, DUET_DIST_BACKEND="gloo", DUET_FORCE_DEVICE="0", OUT=str(tmp_path))
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2", "--master-addr",
           "127.0.0.1", "--master-port", "29547", os.path.join(root, "tests", "shard_parity_worker.py")]
    r = subprocess.run(cmd, env=env, cwd=root, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
    assert "shard parity ok" in r.stdout, r.stdout[-3000:]


@pytest.mark.gpu
def test_bench_branch_placement_two_ranks_on_one_gpu():
    """bench.py --placement branch under torchrun with 2 ranks (both on GPU 0 over gloo, tensors staged
    through host memory): c3's two towers placed on the 2 ranks by greedy-correction, cut edges sent
    point-to-point, rank 0 prints one JSON line with the placement."""
    import json
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, DUET_DIST_BACKEND="gloo", DUET_FORCE_DEVICE="0")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2", "--master-addr",
           "127.0.0.1", "--master-port", "29543", "bench.py", "--config", "c3", "--placement", "branch", "--gpus",
           "2", "--steps", "3", "--warmup", "3", "--profile-samples", "5"]
    r = subprocess.run(cmd, env=env, cwd=root, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-2000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["scaling"] == "strong" and len(set(d["placement"]["sg_gpu"])) >= 1
