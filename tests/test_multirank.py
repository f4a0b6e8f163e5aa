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
           "--warmup", "3", "--no-cpu-baseline", "--profile-samples", "5"]
    r = subprocess.run(cmd, env=env, cwd=root, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-2000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["config"]["global_batch"] == 2 and d["value"] > 0


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
