import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_ipps_zhanghl21_b200 import workloads as W
from paper_conf_ipps_zhanghl21_b200.harness import Session, materialize
from oracle import forward as OF
from tests.helpers import to_np, lazy_rows, rel_err
wl = W.build("c4", branch_outputs=True)
sess = Session(wl, n_slots=2, profile=dict(warmup=2, samples=3, reps=2))
inputs = list(materialize(wl.inputs, "cuda").values())
outs = sess.outputs()
sess.run(sess.schedule(), inputs, outs)
torch.cuda.synchronize()
names = [o[0] for o in wl.outputs]
O = dict(zip(names, outs))
w = sess.params["head_w"].double().cpu().numpy(); b = sess.params["head_b"].double().cpu().numpy()
feats = [O[n].float().double().cpu().numpy() for n in ("cnn_gap", "gru", "mlp_fc")]
z = np.concatenate(feats, 1) @ w + b[0]
y_from_gpu_feats = 1 / (1 + np.exp(-z))
print("head kernel vs f64 head on GPU features:", rel_err(O["y"].cpu().numpy()[:, 0], y_from_gpu_feats))
print("z range", z.min(), z.max(), "y range", y_from_gpu_feats.min(), y_from_gpu_feats.max())
rows = np.array([63, 5])
oparams = {k: (lazy_rows(s) if s.numel > 10_000_000 else to_np(sess.params[k])) for k, s in wl.params.items()}
oin = {k: to_np(t)[rows] for k, t in zip(wl.inputs, inputs)}
want = OF.run(wl.ir, oparams, oin)
for n in names:
    g = O[n].float().cpu().numpy()[rows]
    print(n, "err", rel_err(g, want[n]), "max|oracle|", np.abs(want[n]).max(), "max abs diff", np.abs(g - want[n]).max())
zo = np.concatenate([want["cnn_gap"], want["gru"], want["mlp_fc"]], 1) @ w + b[0]
print("z oracle", zo, "z gpu", z[rows])
