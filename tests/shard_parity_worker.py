"""torchrun worker for tests/test_multirank.py::test_shard_parity_two_ranks_on_one_gpu: c5-small's
batch sharded over the ranks (multirank.ShardExecutor), each rank's rows through libduet, gathered on
rank 0 and checked against the float64 oracle of the whole batch."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from oracle import forward as OF  # noqa: E402
from paper_conf_ipps_zhanghl21_b200 import multirank as MR  # noqa: E402
from paper_conf_ipps_zhanghl21_b200 import workloads as W  # noqa: E402
from paper_conf_ipps_zhanghl21_b200.harness import Session, materialize  # noqa: E402
from tests.helpers import TOL, check, oracle_arrays  # noqa: E402

rank, world, local = MR.env()
torch.cuda.set_device(local)
MR.init("nccl", torch.device(f"cuda:{local}"))
dev = torch.device(f"cuda:{local}")
full = W.build("c5", small=True, batch=96 * world)
wl = W.build("c5", small=True, batch=96)
sess = Session(wl, n_slots=2, device=local, profile=dict(warmup=1, samples=3, reps=1))
sched = sess.schedule()
inputs = list(materialize(full.inputs, dev).values())
tdt = {"f32": torch.float32, "bf16": torch.bfloat16, "i32": torch.int32, "i64": torch.int64}
in_meta = [(t.shape[1:], t.dtype) for t in inputs]
out_meta = [(tuple(shape[1:]), tdt[dt]) for _, dt, shape in full.outputs]
ex = MR.ShardExecutor(full.batch, in_meta, out_meta, dev)
outs = [torch.full((full.batch,) + m[0], float("nan"), dtype=m[1], device=dev) for m in out_meta]
cur = torch.cuda.current_stream()


def runner(si, so):
    sess.run(sched, si, so)
    cur.wait_stream(sess.home)


ex.step(inputs, outs, runner)
torch.cuda.synchronize()
if rank == 0:
    want = OF.run(full.ir, oracle_arrays(sess.params), oracle_arrays(dict(zip(full.inputs, inputs))))
    for (name, _, _), o in zip(full.outputs, outs):
        check(o.float().cpu().numpy(), want[name], TOL["bf16"], f"shard x{world} {name}")
    print("shard parity ok", flush=True)
MR.barrier()
MR.finalize()
