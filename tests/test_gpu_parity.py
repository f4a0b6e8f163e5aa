"""GPU parity: the CUDA path (through the C ABI) vs the float64 oracle on the same seeded inputs.

Bar (BASELINE.json:5): relative error <= 1e-5 (fp32) / 2e-2 (bf16 inputs, fp32
accumulate); bit-exact for integer / byte work (hashing, gathers).  Sizes span several tiles with
ragged tails; the full c2 size (the bench workload) is checked on sampled rows."""
import numpy as np
import pytest
import torch

from oracle import forward as OF
from paper_conf_ipps_zhanghl21_b200 import duet
from paper_conf_ipps_zhanghl21_b200 import workloads as W
from paper_conf_ipps_zhanghl21_b200.harness import Session, materialize
from tests.helpers import TOL, check, lazy_rows, oracle_arrays, rel_err, to_np

pytestmark = pytest.mark.gpu

FAST_PROFILE = dict(warmup=2, samples=5, reps=2)


def _single_node_graph(op_line, params, inputs):
    lines = [f"param @{k} : {dt}[{','.join(map(str, s))}]" for k, (dt, s) in params.items()]
    lines += [f"%{k} = input() : {dt}[{','.join(map(str, s))}]" for k, (dt, s) in inputs.items()]
    lines += [op_line, "output %y"]
    return "\n".join(lines) + "\n"


def _rand(shape, dt, scale=1.0, seed=0):
    g = torch.Generator().manual_seed(seed)
    t = (torch.rand(shape, generator=g, dtype=torch.float64) * 2 - 1) * scale
    return t.to(torch.float32).to(torch.bfloat16 if dt == "bf16" else torch.float32)


@pytest.mark.parametrize("M,N,K,dt,out", [
    (128, 128, 64, "bf16", "bf16"),
    (300, 136, 320, "bf16", "bf16"),
    (2048, 1024, 1664, "bf16", "bf16"),
    (77, 48, 72, "bf16", "f32"),
    (513, 272, 200, "bf16", "f32"),
    (300, 136, 320, "f32", "f32"),      # fp32 on the tensor cores (3xTF32, gemm_tf32.cu)
    (2048, 1024, 1664, "f32", "f32"),   # c2's fc1 in fp32: 128-wide tiles
    (130, 17, 36, "f32", "f32"),        # ragged M / N, K one 32-wide block + 4
    (4096, 64, 1024, "f32", "f32"),
    (5, 3, 7, "f32", "f32"),            # K % 4 != 0, N < 16: CUDA-core path
    (128, 768, 3072, "bf16", "bf16"),   # split-K (12 splits of 4 k-blocks) + reduce
    (120, 136, 2500, "bf16", "f32"),    # split-K, ragged M / N / K
    (3, 768, 768, "bf16", "bf16"),      # MT-DNN task pooler at batch 3
])
def test_linear_node(M, N, K, dt, out):
    ir = _single_node_graph(f"%y = linear(%x, @W, @b) {{act=relu}} : {out}[{M},{N}]",
                            {"W": (dt, (N, K)), "b": ("f32", (N,))}, {"x": (dt, (M, K))})
    x = _rand((M, K), dt, 1.0, 1)
    Wt = _rand((N, K), dt, 1.0 / np.sqrt(K), 2)
    b = _rand((N,), "f32", 0.1, 3)
    g = duet.Graph(ir)
    g.bind_all({"W": Wt.cuda(), "b": b.cuda()})
    y = torch.empty((M, N), dtype=torch.bfloat16 if out == "bf16" else torch.float32, device="cuda")
    g.node_run("y", [x.cuda()], y)
    torch.cuda.synchronize()
    want = OF.linear(OF.to_f64(to_np(x), dt), OF.to_f64(to_np(Wt), dt), OF.to_f64(to_np(b), "f32"), "relu")
    err = rel_err(y.float().cpu().numpy(), want)
    assert err <= (TOL["f32"] if dt == "f32" else 1e-2), err


def test_gathers_and_hash_bit_exact():
    wl = W.build("c2", small=True)
    params = materialize(wl.params, "cuda")
    raw = wl.inputs["raw"].materialize("cuda")
    g = duet.Graph(wl.ir)
    g.bind_all(params)
    B, F = raw.shape
    ids = torch.empty((B, F), dtype=torch.int32, device="cuda")
    g.node_run("ids", [raw], ids)
    X = torch.empty((B, F * 64), dtype=torch.bfloat16, device="cuda")
    g.node_run("deep_x", [ids], X)
    wide = torch.empty((B, 1), dtype=torch.float32, device="cuda")
    g.node_run("wide", [ids], wide)
    torch.cuda.synchronize()
    V = 1000
    o_ids = OF.hash_mod(to_np(raw), V)
    np.testing.assert_array_equal(ids.cpu().numpy(), o_ids)
    E = to_np(params["deep_E"])
    np.testing.assert_array_equal(to_np(X), E[np.arange(F)[None, :], o_ids].reshape(B, -1))
    o_wide = OF.gather_sum(o_ids, to_np(params["wide_T"]), "bf16", to_np(params["wide_b"]).astype(np.float64))
    assert rel_err(wide.cpu().numpy(), o_wide) < 1e-6


def _oracle_outputs(wl, params, inputs):
    return OF.run(wl.ir, oracle_arrays(params), oracle_arrays(inputs))


CASES = [("c1", "f32"), ("c1", "bf16"), ("c2", "bf16"), ("c2", "f32"), ("c3", "bf16"), ("c3", "f32"),
         ("c4", "bf16"), ("c4", "f32"), ("c5", "bf16"), ("c5", "f32"), ("c6", "bf16"), ("c6", "f32")]


@pytest.mark.parametrize("cfg,dt", CASES)
def test_config_small_parity(cfg, dt):
    wl = W.build(cfg, small=True, dt=dt, branch_outputs=True)
    sess = Session(wl, n_slots=2, profile=FAST_PROFILE)
    assert sess.part.n_sg > 1  # branch outputs keep the multi-path phases (only sinks reach C2's sink)
    inputs = list(materialize(wl.inputs, "cuda").values())
    want = _oracle_outputs(wl, sess.params, dict(zip(wl.inputs, inputs)))
    results = {}
    for mode in (duet.GREEDY_CORRECTION, duet.SERIAL):
        outs = sess.outputs()
        sess.run(sess.schedule(mode), inputs, outs)
        torch.cuda.synchronize()
        results[mode] = [o.float().cpu().numpy() for o in outs]
        for (name, _, _), y in zip(wl.outputs, results[mode]):
            check(y, want[name], TOL[dt], f"{cfg} {dt} mode={mode} {name}")
    # same kernels, any placement -> bit-identical outputs
    for a, b in zip(results[duet.GREEDY_CORRECTION], results[duet.SERIAL]):
        np.testing.assert_array_equal(a, b)


def _input_consumers(ir, node_to_sg):
    """graph input name -> sorted subgraph ids of the nodes reading it (node ids = IR node order)."""
    import re
    names, args = [], []
    for ln in ir.splitlines():
        m = re.match(r"^%([\w.]+) = (\w+)\((.*?)\)", ln)
        if m:
            names.append((m.group(1), m.group(2)))
            args.append([a.strip()[1:] for a in m.group(3).split(",") if a.strip().startswith("%")])
    out = {nm: set() for nm, op in names if op == "input"}
    for i, a in enumerate(args):
        for x in a:
            if x in out:
                out[x].add(node_to_sg[i])
    return {k: sorted(v) for k, v in out.items()}


def _assignments(n, inputs_first_last, limit=64, seed=0):
    """All 2^n slot assignments when n is small, else a seeded random sample plus, for every input
    read by several subgraphs, the assignments that put its first consumer on slot 1 and a later
    one on slot 0 and vice versa (the H2D copy's event is then waited on across streams)."""
    import itertools
    import random
    if 2 ** n <= limit:
        return [list(a) for a in itertools.product(range(2), repeat=n)]
    rng = random.Random(seed)
    out = [[rng.randrange(2) for _ in range(n)] for _ in range(limit)]
    for first, last in inputs_first_last:
        for d in (0, 1):
            a = [rng.randrange(2) for _ in range(n)]
            a[first], a[last] = 1 - d, d
            out.append(a)
    return out


@pytest.mark.parametrize("cfg", ["c1", "c3", "c4", "c5"])
def test_host_buffers_every_assignment(cfg):
    """Slot assignments with pinned host buffers: each H2D copy is issued at the fork on its own
    copy stream and every consumer waits on its event (runtime.cu capture) -- the outputs equal the
    device-buffer run of the serial schedule byte for byte.  c5's raw features feed two subgraphs."""
    wl = W.build(cfg, small=True, branch_outputs=True)
    sess = Session(wl, n_slots=2, profile=FAST_PROFILE)
    n = sess.part.n_sg
    assert n > 1
    inputs = list(materialize(wl.inputs, "cuda").values())
    ref = sess.outputs()
    sess.run(sess.schedule(duet.SERIAL), inputs, ref)
    torch.cuda.synchronize()
    ref = [r.float().cpu().numpy() for r in ref]
    host_in = [t.cpu().pin_memory() for t in inputs]
    shared = [(min(sgs), max(sgs)) for sgs in _input_consumers(wl.ir, sess.part.export()["node_to_sg"]).values()
              if len(sgs) > 1]
    if cfg == "c5":
        assert shared
    for a in _assignments(n, shared):
        s = sess.prof.schedule(mode=duet.FIXED, fixed=list(a))
        host_out = sess.outputs(device=False)
        for o in host_out:
            o.fill_(float("nan")) if o.is_floating_point() else o.fill_(-1)
        sess.run(s, host_in, host_out)
        sess.home.synchronize()
        torch.cuda.synchronize()
        for r, h in zip(ref, host_out):
            np.testing.assert_array_equal(r, h.float().numpy(), err_msg=str(a))


@pytest.mark.parametrize("cfg", ["c1", "c2", "c3", "c4", "c5", "c6"])
def test_host_buffers_e2e_equal_device(cfg):
    """Pinned HOST inputs/outputs through duet_run (zero-copy reads/stores where eligible, memcpy
    nodes elsewhere; branch outputs exercise both) give the same bytes as device tensors."""
    wl = W.build(cfg, small=True, branch_outputs=True)
    sess = Session(wl, n_slots=2, profile=FAST_PROFILE)
    inputs = list(materialize(wl.inputs, "cuda").values())
    s = sess.schedule()
    dev_out = sess.outputs()
    sess.run(s, inputs, dev_out)
    host_in = [t.cpu().pin_memory() for t in inputs]
    for rep in range(2):
        host_out = sess.outputs(device=False)
        for o in host_out:
            o.fill_(float("nan")) if o.is_floating_point() else o.fill_(-1)
        sess.run(s, host_in, host_out)
        sess.home.synchronize()
        torch.cuda.synchronize()
        for d, h in zip(dev_out, host_out):
            np.testing.assert_array_equal(d.float().cpu().numpy(), h.float().numpy())
    assert s.launch_count() >= 3
    with pytest.raises(duet.DuetError) as e:
        sess.run(s, [t.cpu() for t in inputs], sess.outputs(device=False))  # pageable inputs
    assert e.value.name == "EINVAL"


def tile_rows(batch, seed, tile=128, extra=()):
    """One random row from every 128-row M tile (the GEMM / recurrence tile height), the first and
    the last row, plus `extra`: a bug confined to one tile cannot escape."""
    rng = np.random.default_rng(seed)
    rows = {0, batch - 1, *extra}
    for t0 in range(0, batch, tile):
        rows.add(int(rng.integers(t0, min(batch, t0 + tile))))
    return np.array(sorted(rows))


@pytest.mark.parametrize("cfg", ["c3", "c4", "c5"])
def test_full_size_sampled(cfg):
    """c3/c4/c5 at their BASELINE.json sizes (bench launch configuration: 2 slots, greedy-correction);
    the oracle evaluates one sampled row per 128-row tile plus the ends (rows are independent) --
    every branch output."""
    wl = W.build(cfg, branch_outputs=True)
    sess = Session(wl, n_slots=2, profile=FAST_PROFILE)
    inputs = list(materialize(wl.inputs, "cuda").values())
    outs = sess.outputs()
    sess.run(sess.schedule(), inputs, outs)
    torch.cuda.synchronize()
    rows = tile_rows(wl.batch, 1, extra=(17,) if wl.batch > 17 else ())
    oparams = {k: (lazy_rows(spec) if spec.numel > 10_000_000 else to_np(sess.params[k]))
               for k, spec in wl.params.items()}
    oin = {k: to_np(t)[rows] for k, t in zip(wl.inputs, inputs)}
    want = OF.run(wl.ir, oparams, oin)
    for (name, _, _), y in zip(wl.outputs, outs):
        check(y.float().cpu().numpy()[rows], want[name], TOL["bf16"], f"full {cfg} {name} ({len(rows)} rows)")


def test_c2_full_size_sampled():
    """The bench workload (BASELINE.json:8 at full size) in the bench's launch configuration;
    the oracle evaluates 96 sampled rows (rows are independent), reading only the table rows they
    touch."""
    wl = W.build("c2")
    sess = Session(wl, n_slots=2, profile=FAST_PROFILE)
    inputs = list(materialize(wl.inputs, "cuda").values())
    outs = sess.outputs()
    sess.run(sess.schedule(), inputs, outs)
    torch.cuda.synchronize()
    rows = tile_rows(wl.batch, 0, extra=np.random.default_rng(0).choice(wl.batch, 64, replace=False).tolist())
    oparams = {}
    for k, spec in wl.params.items():
        oparams[k] = lazy_rows(spec) if spec.numel > 10_000_000 else to_np(sess.params[k])
    oin = {"raw": to_np(inputs[0])[rows]}
    want = OF.run(wl.ir, oparams, oin)["y"]
    check(outs[0].cpu().numpy()[rows], want, TOL["bf16"], f"full c2 ({len(rows)} rows)")


@pytest.mark.parametrize("N,H,W,C,Co,k,stride,pad", [
    (2, 23, 19, 3, 64, 7, 2, 3),      # W*C % 8 != 0: explicit im2col + pair GEMM, K padded to 8
    (1, 224, 224, 3, 64, 7, 2, 3),    # ResNet stem at full size: smem-im2col kernel (conv_stem.cu)
    (2, 64, 64, 3, 64, 7, 2, 3),      # stem kernel, one TMA box per input row
    (3, 40, 24, 3, 32, 7, 2, 3),      # stem kernel, Wo = 12, Co = 32, rows outside the image
    (2, 30, 16, 4, 48, 5, 2, 2),      # stem kernel with no dummy element (pad*C even), Co = 48
    (3, 14, 14, 64, 64, 3, 1, 1),     # 3x3, vector path, ragged M tile
    (2, 15, 13, 128, 256, 3, 2, 1),   # stride 2, Co = 256
    (2, 9, 9, 64, 128, 1, 2, 0),      # 1x1 downsample
    (4, 1, 1, 512, 512, 3, 1, 1),     # 1x1 map: only the centre tap (tap rectangle)
    (16, 2, 2, 256, 512, 3, 2, 1),    # c5 layer-4 downsampling conv: 2 x 2 of 9 taps
    (64, 7, 7, 512, 512, 3, 1, 1),    # c4 layer 4: 25 m tiles
    (30, 7, 7, 512, 256, 3, 1, 1),    # ragged last m tile
    (8, 14, 14, 256, 256, 3, 1, 1),   # layer-3 shape
    (2, 56, 56, 64, 64, 3, 1, 1),     # c4 layer 1 (three CTAs per SM)
    (3, 28, 28, 128, 128, 3, 1, 1),   # layer-2 shape
    (7, 8, 8, 64, 64, 3, 1, 1),       # c5 layer-1 shape
    (3, 12, 20, 64, 48, 3, 1, 1),     # W != H, Co < tile
    (32, 28, 28, 128, 128, 3, 1, 1),  # 196 128-wide tiles > SMs: two CTAs per SM
    (64, 14, 14, 256, 256, 3, 1, 1),  # c4 layer 3 (two CTAs per SM)
])

def test_conv_node(N, H, W, C, Co, k, stride, pad, dt="bf16"):
    Ho, Wo = (H + 2 * pad - k) // stride + 1, (W + 2 * pad - k) // stride + 1
    ir = _single_node_graph(
        f"%y = conv2d_bn(%x, @W, @g, @b, @m, @v) {{stride={stride}, pad={pad}, act=relu}} : {dt}[{N},{Ho},{Wo},{Co}]",
        {"W": (dt, (Co, k, k, C)), "g": ("f32", (Co,)), "b": ("f32", (Co,)), "m": ("f32", (Co,)),
         "v": ("f32", (Co,))}, {"x": (dt, (N, H, W, C))})
    x = _rand((N, H, W, C), dt, 1.0, 5)
    Wt = _rand((Co, k, k, C), dt, (2.0 / (k * k * C)) ** 0.5, 6)
    g_ = (_rand((Co,), "f32", 0.5, 7) + 1.0)
    b_ = _rand((Co,), "f32", 0.1, 8)
    m_ = _rand((Co,), "f32", 0.1, 9)
    v_ = (_rand((Co,), "f32", 0.5, 10) + 1.0)
    g = duet.Graph(ir)
    g.bind_all({"W": Wt.cuda(), "g": g_.cuda(), "b": b_.cuda(), "m": m_.cuda(), "v": v_.cuda()})
    y = torch.empty((N, Ho, Wo, Co), dtype=torch.bfloat16 if dt == "bf16" else torch.float32, device="cuda")
    g.node_run("y", [x.cuda()], y)
    torch.cuda.synchronize()
    f = lambda t, d: OF.to_f64(to_np(t), d)
    want = OF.conv2d_bn(f(x, dt), f(Wt, dt), f(g_, "f32"), f(b_, "f32"), f(m_, "f32"), f(v_, "f32"),
                        stride, pad, "relu")
    check(y.float().cpu().numpy(), want, TOL[dt], f"conv {N}x{H}x{W}x{C}->{Co} k{k}s{stride} {dt}")


@pytest.mark.parametrize("N,H,W,C,Co,k,stride,pad", [
    (2, 23, 19, 3, 64, 7, 2, 3),      # C % 32 != 0: explicit fp32 im2col + 3xTF32 GEMM
    (1, 224, 224, 3, 64, 7, 2, 3),    # ResNet stem at full size
    (2, 30, 16, 4, 48, 5, 2, 2),
    (3, 14, 14, 64, 64, 3, 1, 1),     # 3xTF32 implicit GEMM (im2col TMA, 32-channel k-blocks)
    (2, 15, 13, 128, 256, 3, 2, 1),   # stride 2, 128-wide tiles
    (2, 9, 9, 64, 128, 1, 2, 0),      # 1x1 downsample
    (4, 1, 1, 512, 512, 3, 1, 1),     # tap rectangle: centre tap only
    (16, 2, 2, 256, 512, 3, 2, 1),
    (30, 7, 7, 512, 256, 3, 1, 1),    # ragged last m tile, K = 4608
    (2, 56, 56, 64, 64, 3, 1, 1),     # c4 layer-1 shape
    (3, 12, 20, 32, 48, 3, 1, 1),     # one 32-channel block, Co < tile
])
def test_conv_node_f32(N, H, W, C, Co, k, stride, pad):
    """fp32 mode on the tensor cores (gemm_tf32.cu) against the float64 oracle at the fp32 bar."""
    test_conv_node(N, H, W, C, Co, k, stride, pad, dt="f32")

@pytest.mark.parametrize("N,H,W,C", [
    (5, 1, 1, 512),     # c5's layer-4 map: the small-map average pool is a per-chunk copy
    (3, 2, 3, 64),      # HW < 8: small-map kernel
    (2, 7, 7, 512),     # c4's layer-4 map (HW >= 8: split-HW kernel)
    (3, 9, 5, 24),      # C % 8 == 0 (3 chunks)
    (2, 3, 3, 20),      # C % 8 != 0: scalar kernel
    (2, 112, 112, 64),  # c4's max pool input: staged bands of output rows
    (5, 16, 16, 64),    # c5's: a whole image per CTA
    (3, 15, 9, 64),     # odd H / W: the last window is clipped
])
def test_pool_nodes(N, H, W, C):
    """Global average pool and 3x3/2 max pool nodes against the oracle (bf16 storage)."""
    Hp, Wp = (H - 1) // 2 + 1, (W - 1) // 2 + 1
    ir = "\n".join([f"%x = input() : bf16[{N},{H},{W},{C}]", f"%a = avgpool(%x) : bf16[{N},{C}]",
                     f"%y = maxpool(%x) {{k=3, stride=2, pad=1}} : bf16[{N},{Hp},{Wp},{C}]", "output %a",
                     "output %y"]) + "\n"
    x = _rand((N, H, W, C), "bf16", 2.0, 41)
    g = duet.Graph(ir)
    a = torch.empty((N, C), dtype=torch.bfloat16, device="cuda")
    y = torch.empty((N, Hp, Wp, C), dtype=torch.bfloat16, device="cuda")
    g.node_run("a", [x.cuda()], a)
    g.node_run("y", [x.cuda()], y)
    torch.cuda.synchronize()
    xf = OF.to_f64(to_np(x), "bf16")
    check(a.float().cpu().numpy(), OF.avgpool(xf), TOL["bf16"], f"avgpool {N}x{H}x{W}x{C}")
    # a max of bf16 values is one of them: exact
    np.testing.assert_array_equal(y.float().cpu().numpy(), OF.maxpool(xf, 3, 2, 1))


@pytest.mark.parametrize("kind,S,B,E,H,dt", [
    ("lstm", 7, 300, 64, 48, "bf16"),    # ragged B (3 M tiles), H not a multiple of the unit tile
    ("lstm", 5, 64, 40, 136, "bf16"),    # E padded to 64, H > one tile
    ("gru", 6, 200, 64, 72, "bf16"),
    ("gru", 4, 130, 24, 256, "bf16"),
    ("lstm", 5, 33, 24, 40, "f32"),      # fp32: 3xTF32 fused step (gemm_tf32.cu)
    ("gru", 5, 33, 24, 40, "f32"),
    ("lstm", 6, 300, 64, 136, "f32"),    # 3 M tiles, H over several 16-unit tiles
    ("gru", 5, 260, 100, 72, "f32"),     # E padded to 128
    ("lstm", 4, 20, 23, 40, "f32"),      # E % 4 != 0: CUDA-core parity path
    ("gru", 4, 20, 24, 42, "f32"),       # H % 4 != 0: CUDA-core parity path
])
def test_rnn_node(kind, S, B, E, H, dt):
    G = 4 if kind == "lstm" else 3
    ir = _single_node_graph(
        f"%y = {kind}(%x, @Wih, @Whh, @bih, @bhh) : {dt}[{B},{H}]",
        {"Wih": (dt, (G * H, E)), "Whh": (dt, (G * H, H)), "bih": ("f32", (G * H,)), "bhh": ("f32", (G * H,))},
        {"x": (dt, (S, B, E))})
    sc = 1.0 / np.sqrt(H)
    x = _rand((S, B, E), dt, 1.0, 11)
    Wih, Whh = _rand((G * H, E), dt, sc, 12), _rand((G * H, H), dt, sc, 13)
    bih, bhh = _rand((G * H,), "f32", sc, 14), _rand((G * H,), "f32", sc, 15)
    g = duet.Graph(ir)
    g.bind_all({"Wih": Wih.cuda(), "Whh": Whh.cuda(), "bih": bih.cuda(), "bhh": bhh.cuda()})
    y = torch.empty((B, H), dtype=torch.bfloat16 if dt == "bf16" else torch.float32, device="cuda")
    g.node_run("y", [x.cuda()], y)
    torch.cuda.synchronize()
    f = lambda t, d: OF.to_f64(to_np(t), d)
    want = (OF.lstm if kind == "lstm" else OF.gru)(f(x, dt), f(Wih, dt), f(Whh, dt), f(bih, "f32"), f(bhh, "f32"))
    err = rel_err(y.float().cpu().numpy(), want)
    print(f"[parity] {kind} S{S} B{B} E{E} H{H} {dt}: rel err {err:.3e}")
    assert err <= TOL[dt], err


@pytest.mark.parametrize("kind,S,B,E,H,dt", [
    ("gru", 5, 200, 64, 72, "bf16"),      # persistent kernel, one tile per CTA
    ("lstm", 4, 300, 64, 136, "bf16"),
    ("lstm", 3, 2048, 128, 256, "bf16"),  # persistent kernel, several tiles per CTA (state in HBM)
    ("lstm", 3, 4096, 256, 512, "bf16"),  # several 128 x 256 tiles per CTA
    ("gru", 3, 4000, 136, 520, "bf16"),   # 128 x 256 tiles, ragged B, H and E
    ("lstm", 4, 2304, 128, 264, "bf16"),  # one 128 x 256 tile per CTA (90 tiles), ragged H
    ("gru", 3, 4096, 128, 256, "bf16"),   # one 128 x 256 tile per CTA (c5's b3 shape, GRU)
    ("gru", 4, 33, 24, 40, "f32"),        # 3xTF32 fused step
    ("lstm", 3, 40, 23, 40, "f32"),       # CUDA-core parity path
])
def test_rnn_node_seq_output(kind, S, B, E, H, dt):
    rnn_seq_case(kind, S, B, E, H, dt)


_PAIR_SCRIPT = r'''
import os, sys
sys.path.insert(0, os.environ["REPO"])
from tests.test_gpu_parity import rnn_seq_case
for case in [("lstm", 3, 4096, 256, 512, "bf16"), ("gru", 3, 4000, 136, 520, "bf16"), ("lstm", 4, 3840, 128, 264, "bf16")]:
    rnn_seq_case(*case)
    print("ok", case)
'''


def test_rnn_pair_lstm_forced():
    """The CTA-pair recurrence on LSTM (DUET_RNN_PAIR=2; by default only GRU uses it), ragged H,
    every h_t against the oracle; a subprocess because the switch is read once."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, DUET_RNN_PAIR="2", REPO=root)
    r = subprocess.run([sys.executable, "-c", _PAIR_SCRIPT], env=env, capture_output=True, text=True, timeout=300,
                       cwd=root)
    assert r.returncode == 0 and r.stdout.count("ok") == 3, r.stdout[-3000:] + r.stderr[-3000:]


_MSYNC_SCRIPT = r'''
import os, sys
sys.path.insert(0, os.environ["REPO"])
from tests.test_gpu_parity import rnn_seq_case
for case in [("lstm", 6, 300, 64, 136, "bf16"), ("gru", 5, 1000, 64, 72, "bf16"), ("lstm", 4, 2304, 128, 264, "bf16"),
             ("lstm", 4, 4096, 256, 512, "bf16"), ("gru", 4, 4000, 136, 520, "bf16")]:
    rnn_seq_case(*case)
    print("ok", case)
'''


@pytest.mark.parametrize("msync", ["0", "2"])
def test_rnn_row_block_sync_forced(msync):
    """The recurrence's step synchronisation both ways (DUET_RNN_MSYNC=2: every 128-row block waits
    only for its own h_{t-1}; 0: one grid barrier), on one-tile (2 and 8 row blocks), several-tile
    and CTA-pair launches; every h_t against the oracle.  A subprocess: the switch is read once."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, DUET_RNN_MSYNC=msync, REPO=root)
    r = subprocess.run([sys.executable, "-c", _MSYNC_SCRIPT], env=env, capture_output=True, text=True, timeout=300,
                       cwd=root)
    assert r.returncode == 0 and r.stdout.count("ok") == 5, r.stdout[-3000:] + r.stderr[-3000:]


def rnn_seq_case(kind, S, B, E, H, dt):
    """Stacked-RNN lower layer (seq=1, Fig. 14): every h_t, [S, B, H] time-major."""
    G = 4 if kind == "lstm" else 3
    ir = _single_node_graph(
        f"%y = {kind}(%x, @Wih, @Whh, @bih, @bhh) {{seq=1}} : {dt}[{S},{B},{H}]",
        {"Wih": (dt, (G * H, E)), "Whh": (dt, (G * H, H)), "bih": ("f32", (G * H,)), "bhh": ("f32", (G * H,))},
        {"x": (dt, (S, B, E))})
    sc = 1.0 / np.sqrt(H)
    x = _rand((S, B, E), dt, 1.0, 21)
    Wih, Whh = _rand((G * H, E), dt, sc, 22), _rand((G * H, H), dt, sc, 23)
    bih, bhh = _rand((G * H,), "f32", sc, 24), _rand((G * H,), "f32", sc, 25)
    g = duet.Graph(ir)
    g.bind_all({"Wih": Wih.cuda(), "Whh": Whh.cuda(), "bih": bih.cuda(), "bhh": bhh.cuda()})
    y = torch.empty((S, B, H), dtype=torch.bfloat16 if dt == "bf16" else torch.float32, device="cuda")
    g.node_run("y", [x.cuda()], y)
    torch.cuda.synchronize()
    f = lambda t, d: OF.to_f64(to_np(t), d)
    want = (OF.lstm if kind == "lstm" else OF.gru)(f(x, dt), f(Wih, dt), f(Whh, dt), f(bih, "f32"), f(bhh, "f32"),
                                                   seq=True)
    assert want.shape == (S, B, H)
    err = rel_err(y.float().cpu().numpy(), want)
    print(f"[parity] {kind} seq S{S} B{B} E{E} H{H} {dt}: rel err {err:.3e}")
    assert err <= TOL[dt], err


VARIATIONS = [  # PAPER.md:89 §VI-D on c4 (Figs. 14-17): (rnn_layers, resnet, ffn_layers, batch, dt)
    (2, 18, 1, 3, "bf16"), (4, 18, 1, 3, "bf16"), (1, 34, 1, 3, "bf16"), (1, 50, 1, 3, "bf16"),
    (1, 101, 1, 2, "bf16"), (1, 18, 4, 3, "bf16"), (1, 18, 1, 32, "bf16"), (2, 50, 3, 2, "f32"),
]


@pytest.mark.parametrize("layers,resnet,ffn,batch,dt", VARIATIONS)
def test_model_variation_parity(layers, resnet, ffn, batch, dt):
    wl = W.build("c4", small=True, dt=dt, branch_outputs=True, rnn_layers=layers, resnet=resnet,
                 ffn_layers=ffn, batch=batch)
    sess = Session(wl, n_slots=2, profile=FAST_PROFILE)
    inputs = list(materialize(wl.inputs, "cuda").values())
    want = _oracle_outputs(wl, sess.params, dict(zip(wl.inputs, inputs)))
    outs = sess.outputs()
    sess.run(sess.schedule(), inputs, outs)
    torch.cuda.synchronize()
    for (name, _, _), y in zip(wl.outputs, outs):
        check(y.float().cpu().numpy(), want[name], TOL[dt], f"c4 L{layers} R{resnet} F{ffn} B{batch} {dt} {name}")


@pytest.mark.parametrize("tile_n,layers", [(64, 1), (256, 1), (128, 2)])
def test_rnn_tile_n_parity(tile_n, layers):
    """The persistent recurrence's gate-tile width as a node attribute (c4's GRU runs 128-wide
    tiles by default): every width gives the oracle's answer."""
    wl = W.build("c4", small=True, branch_outputs=True, rnn_layers=layers, gru_tile_n=tile_n)
    assert f"tile_n={tile_n}" in wl.ir
    sess = Session(wl, n_slots=2, profile=FAST_PROFILE)
    inputs = list(materialize(wl.inputs, "cuda").values())
    want = _oracle_outputs(wl, sess.params, dict(zip(wl.inputs, inputs)))
    outs = sess.outputs()
    sess.run(sess.schedule(), inputs, outs)
    torch.cuda.synchronize()
    for (name, _, _), y in zip(wl.outputs, outs):
        err = rel_err(y.float().cpu().numpy(), want[name])
        print(f"[parity] c4 gru tile_n={tile_n} L{layers} {name}: rel err {err:.3e}")
        assert err <= TOL["bf16"], (name, err)


@pytest.mark.parametrize("cfg", ["c3", "c4"])
def test_tuned_session_parity(cfg):
    """harness.tuned_session (bench.py's default for workloads with recurrences): both gate-tile
    widths are measured, the kept session is the faster one, and its outputs match the oracle."""
    from paper_conf_ipps_zhanghl21_b200.harness import tuned_session
    wl = W.build(cfg, small=True, branch_outputs=True)
    sess, s, tiles, base = tuned_session(wl, n_slots=2, profile=FAST_PROFILE, samples=5)
    assert set(tiles) == {0, 128} and all(v > 0 for v in tiles.values())
    assert tiles[sess.wl.meta["rnn_tile_n"]] == min(tiles.values())
    assert base.wl.meta["rnn_tile_n"] == 0 and base.params is sess.params
    inputs = list(materialize(wl.inputs, "cuda").values())
    want = _oracle_outputs(wl, sess.params, dict(zip(wl.inputs, inputs)))
    for sch, ss in ((s, sess), (base.schedule(duet.SERIAL), base)):
        outs = ss.outputs()
        ss.run(sch, inputs, outs)
        torch.cuda.synchronize()
        for (name, _, _), y in zip(wl.outputs, outs):
            err = rel_err(y.float().cpu().numpy(), want[name])
            print(f"[parity] {cfg} tuned tile_n={ss.wl.meta['rnn_tile_n']} {name}: rel err {err:.3e}")
            assert err <= TOL["bf16"], (name, err)


def test_rnn_tile_n_invalid():
    wl = W.build("c4", small=True, gru_tile_n=96)
    with pytest.raises(duet.DuetError) as e:
        Session(wl, n_slots=2, profile=FAST_PROFILE)
    assert e.value.name == "EINVAL"
    assert "tile_n" in str(e.value)


@pytest.mark.parametrize("layers,resnet,ffn", [(8, 18, 1), (1, 101, 1), (1, 18, 8)])
def test_model_variation_full_size_sampled(layers, resnet, ffn):
    """The deepest Fig. 14-16 variations at c4's full size (bench launch configuration); the oracle
    evaluates 2 sampled rows."""
    wl = W.build("c4", branch_outputs=True, rnn_layers=layers, resnet=resnet, ffn_layers=ffn)
    sess = Session(wl, n_slots=2, profile=FAST_PROFILE)
    inputs = list(materialize(wl.inputs, "cuda").values())
    outs = sess.outputs()
    sess.run(sess.schedule(), inputs, outs)
    torch.cuda.synchronize()
    rows = np.array([0, 17, wl.batch - 1])
    oparams = {k: (lazy_rows(spec) if spec.numel > 10_000_000 else to_np(sess.params[k]))
               for k, spec in wl.params.items()}
    oin = {k: to_np(t)[rows] for k, t in zip(wl.inputs, inputs)}
    want = OF.run(wl.ir, oparams, oin)
    for (name, _, _), y in zip(wl.outputs, outs):
        check(y.float().cpu().numpy()[rows], want[name], TOL["bf16"], f"full c4 L{layers} R{resnet} F{ffn} {name}")


@pytest.mark.parametrize("B,S,heads,dh,dt", [(2, 40, 2, 64, "bf16"), (1, 128, 12, 64, "bf16"), (3, 77, 3, 32, "f32"),
                                              (2, 300, 2, 64, "bf16"), (1, 5, 4, 32, "f32"),
                                              (2, 128, 2, 128, "bf16"), (1, 512, 1, 32, "f32"),
                                              (4, 128, 12, 64, "bf16"), (3, 1, 2, 64, "bf16"), (5, 100, 3, 64, "bf16")])
def test_attention_node(B, S, heads, dh, dt):
    """MT-DNN self-attention against the float64 oracle.  bf16 / dh = 64 /
    S <= 128 runs the tcgen05 kernel (attention_tc.cu; S = 1, 40, 100, 128, several sequences per
    launch), the rest the CUDA-core kernel."""
    H = heads * dh
    ir = _single_node_graph(f"%y = attention(%x) {{heads={heads}, seq={S}}} : {dt}[{B * S},{H}]", {},
                            {"x": (dt, (B * S, 3 * H))})
    x = _rand((B * S, 3 * H), dt, 1.5, 31)
    g = duet.Graph(ir)
    y = torch.empty((B * S, H), dtype=torch.bfloat16 if dt == "bf16" else torch.float32, device="cuda")
    g.node_run("y", [x.cuda()], y)
    torch.cuda.synchronize()
    want = OF.attention(OF.to_f64(to_np(x), dt), heads, S)
    err = rel_err(y.float().cpu().numpy(), want)
    print(f"[parity] attention B{B} S{S} h{heads} dh{dh} {dt}: rel err {err:.3e}")
    assert err <= TOL[dt], err


@pytest.mark.parametrize("rows,H,dt", [(120, 128, "bf16"), (128, 768, "bf16"), (33, 1000, "f32"), (7, 40, "f32")])
def test_add_layernorm_node(rows, H, dt):
    ir = _single_node_graph(f"%y = add_layernorm(%a, %b, @g, @be) : {dt}[{rows},{H}]",
                            {"g": ("f32", (H,)), "be": ("f32", (H,))}, {"a": (dt, (rows, H)), "b": (dt, (rows, H))})
    a, b = _rand((rows, H), dt, 2.0, 41), _rand((rows, H), dt, 1.0, 42)
    gm, be = _rand((H,), "f32", 0.5, 43) + 1.0, _rand((H,), "f32", 0.2, 44)
    g = duet.Graph(ir)
    g.bind_all({"g": gm.cuda(), "be": be.cuda()})
    y = torch.empty((rows, H), dtype=torch.bfloat16 if dt == "bf16" else torch.float32, device="cuda")
    g.node_run("y", [a.cuda(), b.cuda()], y)
    torch.cuda.synchronize()
    f = lambda t, d: OF.to_f64(to_np(t), d)
    want = OF.add_layernorm(f(a, dt), f(b, dt), f(gm, "f32"), f(be, "f32"))
    assert rel_err(y.float().cpu().numpy(), want) <= TOL[dt]


def test_c6_full_size():
    """MT-DNN at its full (proposed) model size (BERT-base encoder + 4 task heads) in the bench's
    launch configuration: every task output and the [CLS] vector against the float64 oracle."""
    wl = W.build("c6", branch_outputs=True, batch=4)  # batch 4: 1-element task outputs make R-25 degenerate
    sess = Session(wl, n_slots=2, profile=FAST_PROFILE)
    inputs = list(materialize(wl.inputs, "cuda").values())
    want = _oracle_outputs(wl, sess.params, dict(zip(wl.inputs, inputs)))
    outs = sess.outputs()
    sess.run(sess.schedule(), inputs, outs)
    torch.cuda.synchronize()
    for (name, _, _), y in zip(wl.outputs, outs):
        check(y.float().cpu().numpy(), want[name], TOL["bf16"], f"full c6 {name}")


@pytest.mark.parametrize("cfg,mode", [("c5", duet.GREEDY_CORRECTION), ("c5", duet.RANDOM_CORRECTION),
                                      ("c3", duet.GREEDY_CORRECTION)])
def test_measured_correction(cfg, mode):
    """Step 3 with device-measured latency returns a valid assignment whose
    outputs equal the serial schedule's bit for bit and still meet the oracle bar."""
    wl = W.build(cfg, small=True, dt="bf16")
    sess = Session(wl, n_slots=2, profile=FAST_PROFILE)
    s = sess.schedule(mode, measured=True, samples=5, warmup=1, seed=3)
    e = s.export()
    assert len(e["slot_of"]) == sess.part.n_sg and all(0 <= d < 2 for d in e["slot_of"])
    assert s.measured_ns > 0 and s.evaluations >= 1
    if mode == duet.RANDOM_CORRECTION and not e["fell_back"]:
        assert s.evaluations >= 2
    inputs = list(materialize(wl.inputs, "cuda").values())
    want = _oracle_outputs(wl, sess.params, dict(zip(wl.inputs, inputs)))
    got = {}
    for key, sch in (("measured", s), ("serial", sess.schedule(duet.SERIAL))):
        outs = sess.outputs()
        sess.run(sch, inputs, outs)
        torch.cuda.synchronize()
        got[key] = [o.float().cpu().numpy() for o in outs]
    for (name, _, _), y, z in zip(wl.outputs, got["measured"], got["serial"]):
        np.testing.assert_array_equal(y, z)
        assert rel_err(y, want[name]) <= TOL["bf16"]


def test_concurrent_slots_no_deadlock():
    """Regression guard: random two-slot assignments of c5 co-run tcgen05 GEMMs,
    RNN steps and persistent convs; with TMEM allocated before griddepcontrol.wait this hung within
    ~100-1300 replays.  Runs in a subprocess under a hard timeout."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, CFG="c5", ITERS="800", MODE="random")
    try:
        r = subprocess.run([sys.executable, os.path.join(root, "tools", "stress.py")], env=env, cwd=root,
                           capture_output=True, text=True, timeout=240)
    except subprocess.TimeoutExpired:
        pytest.fail("c5 random-assignment stress did not finish in 240 s (deadlock?)")
    assert r.returncode == 0 and "done" in r.stdout, r.stdout[-2000:] + r.stderr[-2000:]


def test_branch_placement_pieces_on_device():
    """c5's branches placed on 2 GPUs by greedy-correction over one slot per
    GPU, cut into (GPU, phase) pieces, each piece compiled and run by libduet.  On this one-GPU box
    both 'GPUs' are cuda:0 and the cut-edge transfers are identity (the store is shared); the
    result must match the float64 oracle of the whole graph."""
    from paper_conf_ipps_zhanghl21_b200 import multigpu as MG
    wl = W.build("c5", small=True)
    params = materialize(wl.params, "cuda")
    g = duet.Graph(wl.ir)
    g.bind_all(params)
    part = g.partition()
    ex = part.export()
    t_one = [1_000_000 * (s + 1) for s in range(ex["n_sg"])]  # ms-scale: cross-GPU cost does not dominate
    sg_gpu, _ = MG.place_branches(ex, t_one, 2, graph=g)
    assert set(sg_gpu) == {0, 1}
    pl = MG.plan(wl.ir, ex["node_to_sg"], ex["sg_phase"], sg_gpu)
    runners = {gpu: MG.DuetPieces(pl, gpu, params, 0, n_slots=2, profile=FAST_PROFILE) for gpu in (0, 1)}
    inputs = materialize(wl.inputs, "cuda")
    torch.cuda.synchronize()
    store = dict(inputs)
    for phase in range(pl.n_phases):
        for pc in pl.pieces:
            if pc.phase == phase:
                store.update(runners[pc.gpu](pc, {a: store[a] for a in pc.inputs}))
    torch.cuda.synchronize()
    want = OF.run(wl.ir, oracle_arrays(params), oracle_arrays(inputs))
    for o in pl.graph_outputs:
        err = rel_err(store[o].float().cpu().numpy(), want[o])
        assert err <= TOL["bf16"], (o, err)


def test_bench_contract_keys():
    """`python bench.py` (the driver's default N=1 run, shortened): one JSON line with the contract's
    keys for the c5 headline, the cold roofline of its dominant kernel, a per-config block, the
    CPU-oracle baseline and the e2e leg (device-event and host wall clock)."""
    import json
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, "bench.py", "--steps", "10", "--warmup", "3", "--cpu-seconds", "1",
                        "--profile-samples", "5", "--tail-samples", "30", "--per-config", "c2"],
                       cwd=root, capture_output=True, text=True, timeout=1500)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-2000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout
    d = json.loads(lines[0])
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
              "vs_baseline", "dtype", "data", "config", "e2e", "gpu_launches", "roofline", "cpu_baseline", "clocks",
              "per_config", "p99_ms", "p999_ms"):
        assert k in d, k
    assert d["steps"] == 10 and d["warmup"] == 3 and d["n_gpus"] == 1 and d["value"] > 0
    assert d["config"]["workload"] == "c5_ensemble" and d["tail_samples"] == 30
    assert d["roofline"]["bound"] == "tensor" and 0 < d["roofline"]["frac"] < 1
    assert d["roofline"]["timing"].startswith("cold")
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["value"] > 0
    assert d["cpu_baseline"]["value_1thread"] > 0
    assert d["e2e"]["h2d_bytes_per_step"] > 30e6 and d["e2e"]["d2h_bytes_per_step"] == 4096 * 4
    assert d["e2e"]["host_wall_p50_ms"] >= d["e2e"]["p50_ms"] * 0.9
    assert d["gpu_launches"] >= d["steps"]
    c2 = d["per_config"]["c2"]
    assert c2["workload"] == "c2_wide_deep" and c2["roofline"]["frac"] > 0 and c2["speedup_vs_serial"] > 0
    assert c2["e2e"]["h2d_bytes_per_step"] == 2048 * 26 * 8


@pytest.mark.parametrize("cfg", ["c2", "c4", "c5"])
def test_executor_trace_dependencies(cfg):
    """The executor's dependency contract on the device (§IV-D): with tracing on,
    duet_run records each subgraph's start / end; every partition edge u -> v has start(v) >=
    end(u), subgraphs on one slot never overlap, and the traced run's outputs equal the untraced
    run's bit for bit (tracing adds event nodes only)."""
    import os
    import sys
    sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tools"))
    import trace_json as TJ
    wl = W.build(cfg, small=True)
    sess = Session(wl, n_slots=2, profile=FAST_PROFILE)
    inputs = list(materialize(wl.inputs, "cuda").values())
    for sched in (sess.schedule(), sess.prof.schedule(mode=duet.ROUND_ROBIN)):
        ref = sess.outputs()
        sess.run(sched, inputs, ref)
        torch.cuda.synchronize()
        with pytest.raises(duet.DuetError):
            sched.trace()  # the last run was not traced
        sched.set_trace(True)
        outs = sess.outputs()
        sess.run(sched, inputs, outs)
        torch.cuda.synchronize()
        start, end = sched.trace()
        assert (end >= start).all() and (start >= 0).all()
        assert TJ.violations(sess, start, end) == []
        slot_of = sched.export()["slot_of"]
        for d in set(slot_of):
            iv = sorted((int(start[s]), int(end[s])) for s in range(len(slot_of)) if slot_of[s] == d)
            assert all(b[0] >= a[1] for a, b in zip(iv, iv[1:])), iv
        for r, o in zip(ref, outs):
            assert torch.equal(r.cpu(), o.cpu())
        sched.set_trace(False)

