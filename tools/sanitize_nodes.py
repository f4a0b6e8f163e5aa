"""Small launches of the hand-synchronised kernels for compute-sanitizer (tests/test_sanitizer.py):
the pair GEMM (gemm2_kernel: TMA + mbarrier ring + tcgen05 + TMEM), the persistent recurrence
(rnn_persist_kernel: grid barrier + h hand-off), the implicit-GEMM conv (conv_tma_kernel) and the
stem conv, each once, plus one two-slot schedule of c2-small (gathers, joins).  Run as
`compute-sanitizer --tool racecheck python tools/sanitize_nodes.py`."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

from paper_conf_ipps_zhanghl21_b200 import duet  # noqa: E402
from paper_conf_ipps_zhanghl21_b200 import workloads as W  # noqa: E402
from paper_conf_ipps_zhanghl21_b200.harness import Session, materialize  # noqa: E402


def node(ir, params, args, out_shape, out_dt=torch.bfloat16):
    g = duet.Graph(ir)
    g.bind_all({k: v.cuda() for k, v in params.items()})
    y = torch.empty(out_shape, dtype=out_dt, device="cuda")
    g.node_run("y", [a.cuda() for a in args], y)
    torch.cuda.synchronize()
    assert torch.isfinite(y.float()).all()


def main():
    which = sys.argv[1:] or ["gemm", "rnn", "conv", "stem", "conv7", "c2"]
    gen = torch.Generator().manual_seed(0)
    r = lambda *s, sc=1.0: ((torch.rand(*s, generator=gen) * 2 - 1) * sc).to(torch.bfloat16)
    if "gemm" in which:
        M, N, K = 300, 136, 320
        node(f"param @W : bf16[{N},{K}]\nparam @b : f32[{N}]\n%x = input() : bf16[{M},{K}]\n"
             f"%y = linear(%x, @W, @b) {{act=relu}} : bf16[{M},{N}]\noutput %y\n",
             {"W": r(N, K, sc=K ** -0.5), "b": torch.zeros(N)}, [r(M, K)], (M, N))
        print("gemm ok", flush=True)
    if "rnn" in which:
        S, B, E, H = 4, 200, 64, 72
        node(f"param @Wih : bf16[{3 * H},{E}]\nparam @Whh : bf16[{3 * H},{H}]\nparam @bih : f32[{3 * H}]\n"
             f"param @bhh : f32[{3 * H}]\n%x = input() : bf16[{S},{B},{E}]\n"
             f"%y = gru(%x, @Wih, @Whh, @bih, @bhh) : bf16[{B},{H}]\noutput %y\n",
             {"Wih": r(3 * H, E, sc=H ** -0.5), "Whh": r(3 * H, H, sc=H ** -0.5), "bih": torch.zeros(3 * H),
              "bhh": torch.zeros(3 * H)}, [r(S, B, E)], (B, H))
        print("rnn ok", flush=True)
    for key, (N_, H_, C, Co, k, s, p) in (("conv", (2, 14, 64, 64, 3, 1, 1)), ("stem", (1, 64, 3, 64, 7, 2, 3)),
                                              ("conv7", (16, 7, 512, 512, 3, 1, 1))):
        if key not in which:
            continue
        Ho, Wo = (H_ + 2 * p - k) // s + 1, (H_ + 2 * p - k) // s + 1
        node(f"param @W : bf16[{Co},{k},{k},{C}]\nparam @g : f32[{Co}]\nparam @b : f32[{Co}]\nparam @m : f32[{Co}]\n"
             f"param @v : f32[{Co}]\n%x = input() : bf16[{N_},{H_},{H_},{C}]\n"
             f"%y = conv2d_bn(%x, @W, @g, @b, @m, @v) {{stride={s}, pad={p}, act=relu}} : bf16[{N_},{Ho},{Wo},{Co}]\n"
             "output %y\n",
             {"W": r(Co, k, k, C, sc=(2.0 / (k * k * C)) ** 0.5), "g": torch.ones(Co), "b": torch.zeros(Co),
              "m": torch.zeros(Co), "v": torch.ones(Co)}, [r(N_, H_, H_, C)], (N_, Ho, Wo, Co))
        print(key, "ok", flush=True)
    if "c2" in which:
        wl = W.build("c2", small=True)
        sess = Session(wl, n_slots=2, profile=dict(warmup=1, samples=2, reps=1))
        inputs = list(materialize(wl.inputs, "cuda").values())
        outs = sess.outputs()
        sess.run(sess.prof.schedule(mode=duet.FIXED, fixed=[0, 1, 0, 0]), inputs, outs)
        torch.cuda.synchronize()
        print("c2 ok", flush=True)


if __name__ == "__main__":
    main()
