"""Synthetic multi-branch inference workloads c1..c5 (BASELINE.json:7-11) as DUET IR text plus
seeded parameter/input specs.

Structure only: this module writes the IR text (include/duet.h, "IR text") and says how each
parameter and input is drawn (paper_conf_ipps_zhanghl21_b200/inputs.py).  It contains none of
the method's arithmetic.  Shapes marked "(p)" in SURVEY.md §8(d) are the proposed readings of
the paper's lost Table I.

Every builder takes size keywords so the same topology can be instantiated at the full
BASELINE size (bench) and at small sizes the oracle finishes in seconds (tests).
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

from . import inputs as _gen


@dataclass
class TensorSpec:
    dtype: str
    shape: tuple
    init: tuple
    seed: int

    @property
    def numel(self) -> int:
        n = 1
        for s in self.shape:
            n *= int(s)
        return n

    def materialize(self, device="cpu"):
        return _gen.materialize(self.dtype, self.shape, self.init, self.seed, device=device)

    def rows(self, *lead_index):
        return _gen.materialize_rows(self.dtype, self.shape, self.init, self.seed, lead_index)


@dataclass
class Workload:
    name: str
    ir: str
    params: dict = field(default_factory=dict)   # name -> TensorSpec (declaration order)
    inputs: dict = field(default_factory=dict)   # name -> TensorSpec (declaration order)
    outputs: list = field(default_factory=list)  # (name, dtype, shape)
    batch: int = 1
    meta: dict = field(default_factory=dict)


class _Builder:
    def __init__(self, name: str, cfg_id: int, dt: str):
        self.name = name
        self.cfg = cfg_id
        self.dt = dt
        self.lines: list[str] = []
        self.params: dict = {}
        self.inputs: dict = {}
        self.outputs: list = []
        self._n = 0

    def _seed(self) -> int:
        self._n += 1
        return self.cfg * 100003 + self._n * 7919

    def param(self, name, dtype, shape, init):
        assert name not in self.params, name
        self.params[name] = TensorSpec(dtype, tuple(int(s) for s in shape), init, self._seed())
        self.lines.append(f"param @{name} : {dtype}[{','.join(str(int(s)) for s in shape)}]")
        return "@" + name

    def input(self, name, dtype, shape, init):
        self.inputs[name] = TensorSpec(dtype, tuple(int(s) for s in shape), init, self._seed())
        self.node(name, "input", [], dtype, shape)
        return "%" + name

    def node(self, name, op, args, dtype, shape, **attrs):
        a = ", ".join(args)
        at = ""
        if attrs:
            at = " {" + ", ".join(f"{k}={v}" for k, v in attrs.items()) + "}"
        self.lines.append(f"%{name} = {op}({a}){at} : {dtype}[{','.join(str(int(s)) for s in shape)}]")
        return "%" + name

    def output(self, *names):
        self.lines.append("output " + ", ".join(names))

    def build(self, batch, **meta) -> Workload:
        return Workload(self.name, "\n".join(self.lines) + "\n", self.params, self.inputs,
                        self.outputs, batch, meta)

    # ---- layer helpers -------------------------------------------------------------------
    def linear(self, name, x, k, n, m, act="relu", out_dt=None):
        b = 1.0 / math.sqrt(k)
        W = self.param(f"{name}_W", self.dt, (n, k), ("uniform", b))
        bias = self.param(f"{name}_b", "f32", (n,), ("uniform", b))
        return self.node(name, "linear", [x, W, bias], out_dt or self.dt, (m, n), act=act)

    def mlp(self, name, x, dims, m, act="relu", last_act="none", out_dt=None):
        args = [x]
        for i in range(len(dims) - 1):
            b = 1.0 / math.sqrt(dims[i])
            args.append(self.param(f"{name}_W{i}", self.dt, (dims[i + 1], dims[i]), ("uniform", b)))
            args.append(self.param(f"{name}_b{i}", "f32", (dims[i + 1],), ("uniform", b)))
        return self.node(name, "mlp", args, out_dt or self.dt, (m, dims[-1]), act=act,
                         last_act=last_act)

    def rnn(self, name, kind, x, e, h, s, b, seq=False, tile_n=0):
        """seq=True: output every h_t as [S, B, H] (a lower layer of a stacked RNN).  tile_n: the
        persistent recurrence's gate-tile width (0 = automatic)."""
        kw = {"tile_n": tile_n} if tile_n else {}
        g = 4 if kind == "lstm" else 3
        bd = 1.0 / math.sqrt(h)
        Wih = self.param(f"{name}_Wih", self.dt, (g * h, e), ("uniform", bd))
        Whh = self.param(f"{name}_Whh", self.dt, (g * h, h), ("uniform", bd))
        bih = self.param(f"{name}_bih", "f32", (g * h,), ("uniform", bd))
        bhh = self.param(f"{name}_bhh", "f32", (g * h,), ("uniform", bd))
        if seq:
            return self.node(name, kind, [x, Wih, Whh, bih, bhh], self.dt, (s, b, h), seq=1, **kw)
        return self.node(name, kind, [x, Wih, Whh, bih, bhh], self.dt, (b, h), **kw)

    def stacked_rnn(self, name, kind, x, e, h, s, b, layers=1, tile_n=0):
        """`layers` stacked RNNs (Fig. 14): layers 0..L-2 return their whole output
        sequence, the top layer h_S.  The top layer keeps the plain name (layers=1 is the plain RNN)."""
        for li in range(layers - 1):
            x = self.rnn(f"{name}_l{li}", kind, x, e if li == 0 else h, h, s, b, seq=True,
                         tile_n=tile_n)
        return self.rnn(name, kind, x, e if layers == 1 else h, h, s, b, tile_n=tile_n)

    def conv_bn(self, name, x, n, h, w, cin, cout, k, stride, pad, act, gamma=(0.5, 1.5)):
        ho = (h + 2 * pad - k) // stride + 1
        wo = (w + 2 * pad - k) // stride + 1
        std = math.sqrt(2.0 / (cin * k * k))  # Kaiming-normal (fan_in, ReLU gain)
        W = self.param(f"{name}_W", self.dt, (cout, k, k, cin), ("normal", std))
        g = self.param(f"{name}_gamma", "f32", (cout,), ("uniform_range", *gamma))
        be = self.param(f"{name}_beta", "f32", (cout,), ("normal", 0.1))
        mu = self.param(f"{name}_mean", "f32", (cout,), ("normal", 0.1))
        var = self.param(f"{name}_var", "f32", (cout,), ("uniform_range", 0.5, 1.5))
        out = self.node(name, "conv2d_bn", [x, W, g, be, mu, var], self.dt, (n, ho, wo, cout),
                        stride=stride, pad=pad, act=act)
        return out, ho, wo

    def resnet18(self, prefix, x, n, h, w):
        """torchvision ResNet-18 topology in NHWC -> [n, 512]."""
        return self.resnet(prefix, x, n, h, w, 18)

    RESNET_BLOCKS = {18: ("basic", (2, 2, 2, 2)), 34: ("basic", (3, 4, 6, 3)),
                     50: ("bottleneck", (3, 4, 6, 3)), 101: ("bottleneck", (3, 4, 23, 3))}

    def resnet(self, prefix, x, n, h, w, depth=18):
        """torchvision ResNet-`depth` (He et al.; 18/34 BasicBlock, 50/101 Bottleneck with the stride
        on the 3x3 conv, "v1.5") in NHWC -> [n, 512] (18/34) or [n, 2048] (50/101).  The depths
        are Fig. 15's ("Varying the CNN depths")."""
        kind, blocks = self.RESNET_BLOCKS[depth]
        exp = 1 if kind == "basic" else 4
        c, h, w = self.conv_bn(f"{prefix}_stem", x, n, h, w, 3, 64, 7, 2, 3, "relu")
        ho, wo = (h + 2 - 3) // 2 + 1, (w + 2 - 3) // 2 + 1
        c = self.node(f"{prefix}_pool", "maxpool", [c], self.dt, (n, ho, wo, 64), k=3, stride=2, pad=1)
        h, w, cin = ho, wo, 64
        # depth-scaled residual-branch gamma (R-28): the residual stream's variance grows
        # with the number of blocks L, so the branch scale goes with sqrt(8 / L) (8 = ResNet-18's L,
        # unchanged there; the 1/sqrt(L) residual scaling of Fixup / SkipInit) and the pooled
        # features stay O(1) at every depth, as in a trained network
        rs = math.sqrt(8.0 / sum(blocks))
        rg = (0.1 * rs, 0.3 * rs)
        for li, width in enumerate([64, 128, 256, 512]):
            cout = width * exp
            for bi in range(blocks[li]):
                stride = 2 if (li > 0 and bi == 0) else 1
                nm = f"{prefix}_l{li + 1}b{bi}"
                # residual-branch BN gamma ~ U(0.1, 0.3) on the block's last conv: keeps activations
                # O(1) through the stack like a trained network (an untrained Kaiming ResNet doubles
                # the variance per block)
                if kind == "basic":
                    y, h2, w2 = self.conv_bn(nm + "_c1", c, n, h, w, cin, cout, 3, stride, 1, "relu")
                    y, h2, w2 = self.conv_bn(nm + "_c2", y, n, h2, w2, cout, cout, 3, 1, 1, "none",
                                             gamma=rg)
                else:
                    y, _, _ = self.conv_bn(nm + "_c1", c, n, h, w, cin, width, 1, 1, 0, "relu")
                    y, h2, w2 = self.conv_bn(nm + "_c2", y, n, h, w, width, width, 3, stride, 1, "relu")
                    y, h2, w2 = self.conv_bn(nm + "_c3", y, n, h2, w2, width, cout, 1, 1, 0, "none",
                                             gamma=rg)
                if stride != 1 or cin != cout:
                    sc, _, _ = self.conv_bn(nm + "_ds", c, n, h, w, cin, cout, 1, stride, 0, "none")
                else:
                    sc = c
                c = self.node(nm + "_add", "add", [y, sc], self.dt, (n, h2, w2, cout), act="relu")
                h, w, cin = h2, w2, cout
        return self.node(f"{prefix}_gap", "avgpool", [c], self.dt, (n, cin))


# ------------------------------------------------------------------------------------------
# c1 — tiny 2-branch wide&deep (BASELINE.json:7): vocab 1k, emb 16, MLP 64-32-1, batch 1,
# 6 fused-op nodes -> 6 subgraphs at op granularity, 4 at coarse.
# ------------------------------------------------------------------------------------------
def c1_tiny_wd(batch=1, fields=8, vocab=1000, emb=16, hidden=(64, 32), dt="f32") -> Workload:
    B = _Builder("c1_tiny_wd", 1, dt)
    raw = B.input("raw", "i64", (batch, fields), ("randint", 1 << 31))
    ids = B.node("ids", "hash_mod", [raw], "i32", (batch, fields), V=vocab)
    wt = B.param("wide_T", dt, (fields, vocab, 1), ("normal", 0.05))
    wg = B.node("wide_g", "gather_concat", [ids, wt], dt, (batch, fields))
    wb = B.param("wide_b", "f32", (1,), ("uniform", 0.1))
    wide = B.node("wide", "reduce_sum", [wg, wb], "f32", (batch, 1))
    et = B.param("deep_E", dt, (fields, vocab, emb), ("normal", 1.0))
    x = B.node("deep_x", "gather_concat", [ids, et], dt, (batch, fields * emb))
    deep = B.mlp("deep", x, [fields * emb, *hidden, 1], batch, out_dt="f32")
    y = B.node("y", "sum_join", [wide, deep], "f32", (batch, 1))
    B.output(y)
    B.outputs = [("y", "f32", (batch, 1))]
    return B.build(batch, config=1)


# ------------------------------------------------------------------------------------------
# c2 — wide&deep recommender (BASELINE.json:8): 26 sparse tables x64, MLP 1024-512-256, B=2048.
# Join sigma(wide + w.a + b) (Cheng et al.).  R = 10^6 rows (p).
# ------------------------------------------------------------------------------------------
def c2_wide_deep(batch=2048, fields=26, rows=1_000_000, emb=64, hidden=(1024, 512, 256),
                 dt="bf16") -> Workload:
    B = _Builder("c2_wide_deep", 2, dt)
    raw = B.input("raw", "i64", (batch, fields), ("randint", 1 << 31))
    ids = B.node("ids", "hash_mod", [raw], "i32", (batch, fields), V=rows)
    wt = B.param("wide_T", dt, (fields, rows), ("normal", 0.05))
    wb = B.param("wide_b", "f32", (1,), ("uniform", 0.1))
    wide = B.node("wide", "gather_sum", [ids, wt, wb], "f32", (batch, 1))
    et = B.param("deep_E", dt, (fields, rows, emb), ("normal", 1.0))
    h = B.node("deep_x", "gather_concat", [ids, et], dt, (batch, fields * emb))
    k = fields * emb
    for i, n in enumerate(hidden):
        h = B.linear(f"fc{i + 1}", h, k, n, batch, act="relu")
        k = n
    jw = B.param("join_w", "f32", (k,), ("uniform", 1.0 / math.sqrt(k)))
    jb = B.param("join_b", "f32", (1,), ("uniform", 0.1))
    y = B.node("y", "dot_join", [wide, h, jw, jb], "f32", (batch, 1))
    B.output(y)
    B.outputs = [("y", "f32", (batch, 1))]
    return B.build(batch, config=2)


# ------------------------------------------------------------------------------------------
# c3 — two-tower DSSM/Siamese (BASELINE.json:9): 2 LSTM encoders H=512, seq 64, B=256;
# separate weights, cosine join.  V=32768, E=256 (p).
# ------------------------------------------------------------------------------------------
def c3_two_tower(batch=256, seq=64, vocab=32768, emb=256, hidden=512, dt="bf16") -> Workload:
    B = _Builder("c3_two_tower", 3, dt)
    towers = []
    for t in ("A", "B"):
        tok = B.input(f"tok{t}", "i32", (batch, seq), ("randint", vocab))
        E = B.param(f"E{t}", dt, (vocab, emb), ("normal", 1.0))
        x = B.node(f"x{t}", "embed_seq", [tok, E], dt, (seq, batch, emb))
        towers.append(B.rnn(f"lstm{t}", "lstm", x, emb, hidden, seq, batch))
    y = B.node("y", "cosine_join", towers, "f32", (batch, 1))
    B.output(y)
    B.outputs = [("y", "f32", (batch, 1))]
    return B.build(batch, config=3)


# ------------------------------------------------------------------------------------------
# c4 — hybrid CNN + RNN + MLP (BASELINE.json:10): ResNet-18 branch + GRU 1024, B=64.
# Image 224x224x3, GRU(256->1024) S=64, MLP 8 tables x 10^5 x 64 -> 512 -> 256 (p).
# Join sigma(w . concat[512, 1024, 256] + b).
# ------------------------------------------------------------------------------------------
def c4_hybrid(batch=64, image=224, seq=64, vocab=32768, emb=256, gru_hidden=1024, fields=8,
              rows=100_000, mlp_out=256, rnn_layers=1, resnet=18, ffn_layers=1, dt="bf16",
              gru_tile_n=0) -> Workload:
    """`rnn_layers`, `resnet` and `ffn_layers` are the model variations of PAPER.md:89 (§VI-D,
    Figs. 14-16: stacked RNN 1/2/4/8, ResNet 18/34/50/101, FFN depth); `batch` is Fig. 17's.
    The defaults are BASELINE.json:10's configuration.  gru_tile_n: the GRU's gate-tile width
    (0 = automatic; `with_rnn_tile_n` / `harness.tuned_session` choose it by measurement)."""
    B = _Builder("c4_hybrid", 4, dt)
    img = B.input("image", dt, (batch, image, image, 3), ("normal", 1.0))
    cnn = B.resnet("cnn", img, batch, image, image, resnet)
    d_cnn = 512 if resnet in (18, 34) else 2048
    tok = B.input("tok", "i32", (batch, seq), ("randint", vocab))
    E = B.param("tok_E", dt, (vocab, emb), ("normal", 1.0))
    x = B.node("tok_x", "embed_seq", [tok, E], dt, (seq, batch, emb))
    rnn = B.stacked_rnn("gru", "gru", x, emb, gru_hidden, seq, batch, rnn_layers, gru_tile_n)
    raw = B.input("raw", "i64", (batch, fields), ("randint", 1 << 31))
    ids = B.node("ids", "hash_mod", [raw], "i32", (batch, fields), V=rows)
    T = B.param("mlp_E", dt, (fields, rows, 64), ("normal", 1.0))
    f = B.node("mlp_x", "gather_concat", [ids, T], dt, (batch, fields * 64))
    m = B.linear("mlp_fc", f, fields * 64, mlp_out, batch, act="relu")
    for li in range(1, ffn_layers):
        m = B.linear(f"mlp_fc{li}", m, mlp_out, mlp_out, batch, act="relu")
    d = d_cnn + gru_hidden + mlp_out
    hw = B.param("head_w", "f32", (d,), ("uniform", 1.0 / math.sqrt(d)))
    hb = B.param("head_b", "f32", (1,), ("uniform", 0.1))
    y = B.node("y", "concat_head", [cnn, rnn, m, hw, hb], "f32", (batch, 1), act="sigmoid")
    B.output(y)
    B.outputs = [("y", "f32", (batch, 1))]
    return B.build(batch, config=4, rnn_layers=rnn_layers, resnet=resnet, ffn_layers=ffn_layers)


# ------------------------------------------------------------------------------------------
# c5 — 8-way heterogeneous ensemble (BASELINE.json:11), B=4096 (all branch shapes (p)):
# b0 c2 deep tower (+head), b1 c2 wide, b2 LSTM512 (E256,S32), b3 LSTM256 (E128,S64),
# b4 GRU1024 (E256,S16), b5 GRU512 (E256,S32), b6 ResNet-18 at 32x32, b7 MLP 512-2048-1024-512-1.
# Join sigma(mean of 8 logits).  b0/b1 hash the shared raw ids separately so that the
# replicated input placeholders keep them independent branches.
# ------------------------------------------------------------------------------------------
def c5_ensemble(batch=4096, fields=26, rows=1_000_000, vocab=32768, image=32,
                scale=1.0, dt="bf16") -> Workload:
    """`scale` shrinks widths/lengths for small parity cases (1.0 = BASELINE size)."""
    def sc(v, lo=8):
        return max(lo, int(round(v * scale / 8)) * 8) if scale != 1.0 else v
    B = _Builder("c5_ensemble", 5, dt)
    logits = []
    raw = B.input("raw", "i64", (batch, fields), ("randint", 1 << 31))
    # b0 deep tower
    ids0 = B.node("b0_ids", "hash_mod", [raw], "i32", (batch, fields), V=rows)
    E0 = B.param("b0_E", dt, (fields, rows, 64), ("normal", 1.0))
    h = B.node("b0_x", "gather_concat", [ids0, E0], dt, (batch, fields * 64))
    k = fields * 64
    for i, n in enumerate([sc(1024), sc(512), sc(256)]):
        h = B.linear(f"b0_fc{i + 1}", h, k, n, batch, act="relu")
        k = n
    logits.append(B.linear("b0_head", h, k, 1, batch, act="none", out_dt="f32"))
    # b1 wide
    ids1 = B.node("b1_ids", "hash_mod", [raw], "i32", (batch, fields), V=rows)
    wt = B.param("b1_T", dt, (fields, rows), ("normal", 0.05))
    wb = B.param("b1_b", "f32", (1,), ("uniform", 0.1))
    logits.append(B.node("b1_wide", "gather_sum", [ids1, wt, wb], "f32", (batch, 1)))
    # b2..b5 recurrent branches
    for bi, (kind, e, hdim, s) in zip(
            range(2, 6), [("lstm", 256, 512, 32), ("lstm", 128, 256, 64),
                          ("gru", 256, 1024, 16), ("gru", 256, 512, 32)]):
        e, hdim = sc(e), sc(hdim)
        s = max(2, int(s * scale)) if scale != 1.0 else s
        tok = B.input(f"b{bi}_tok", "i32", (batch, s), ("randint", vocab))
        E = B.param(f"b{bi}_E", dt, (vocab, e), ("normal", 1.0))
        x = B.node(f"b{bi}_x", "embed_seq", [tok, E], dt, (s, batch, e))
        r = B.rnn(f"b{bi}_{kind}", kind, x, e, hdim, s, batch)
        logits.append(B.linear(f"b{bi}_head", r, hdim, 1, batch, act="none", out_dt="f32"))
    # b6 ResNet-18 at 32x32
    img = B.input("b6_image", dt, (batch, image, image, 3), ("normal", 1.0))
    g = B.resnet18("b6", img, batch, image, image)
    logits.append(B.linear("b6_head", g, 512, 1, batch, act="none", out_dt="f32"))
    # b7 dense MLP
    dense = B.input("b7_dense", dt, (batch, sc(512)), ("normal", 1.0))
    h = dense
    k = sc(512)
    for i, n in enumerate([sc(2048), sc(1024), sc(512)]):
        h = B.linear(f"b7_fc{i + 1}", h, k, n, batch, act="relu")
        k = n
    logits.append(B.linear("b7_head", h, k, 1, batch, act="none", out_dt="f32"))
    y = B.node("y", "mean_join", logits, "f32", (batch, 1))
    B.output(y)
    B.outputs = [("y", "f32", (batch, 1))]
    return B.build(batch, config=5)


# ------------------------------------------------------------------------------------------
# c6 — MT-DNN (Fig. 3; not a BASELINE.json config): shared
# lexicon encoder + L-layer bidirectional Transformer encoder (BERT-base: L=12, H=768, 12 heads,
# FFN 3072, post-LN, GELU) over S=128 tokens, then independent task-specific heads on the [CLS]
# vector (MT-DNN's four GLUE task types: single-sentence classification (2), pairwise similarity
# (1), pairwise classification (3), relevance ranking (1)), each pooler linear + tanh -> linear.
# Batch 1 is the paper's inference setting.  All sizes (p).
# ------------------------------------------------------------------------------------------
def c6_mtdnn(batch=1, seq=128, layers=12, hidden=768, heads=12, ffn=3072, vocab=30522, tasks=(2, 1, 3, 1),
             dt="bf16") -> Workload:
    B = _Builder("c6_mtdnn", 6, dt)
    M = batch * seq
    tok = B.input("tok", "i32", (batch, seq), ("randint", vocab))
    seg = B.input("seg", "i32", (batch, seq), ("randint", 2))
    args = [tok, seg, B.param("tok_E", dt, (vocab, hidden), ("normal", 1.0)),
            B.param("pos_E", dt, (seq, hidden), ("normal", 1.0)),
            B.param("seg_E", dt, (2, hidden), ("normal", 1.0)),
            B.param("emb_g", "f32", (hidden,), ("uniform_range", 0.8, 1.2)),
            B.param("emb_b", "f32", (hidden,), ("normal", 0.1))]
    x = B.node("emb", "bert_embed", args, dt, (M, hidden))

    def ln_params(name):
        return [B.param(f"{name}_g", "f32", (hidden,), ("uniform_range", 0.8, 1.2)),
                B.param(f"{name}_b", "f32", (hidden,), ("normal", 0.1))]

    for li in range(layers):
        nm = f"L{li}"
        qkv = B.linear(f"{nm}_qkv", x, hidden, 3 * hidden, M, act="none")
        a = B.node(f"{nm}_att", "attention", [qkv], dt, (M, hidden), heads=heads, seq=seq)
        o = B.linear(f"{nm}_o", a, hidden, hidden, M, act="none")
        x1 = B.node(f"{nm}_ln1", "add_layernorm", [o, x] + ln_params(f"{nm}_ln1"), dt, (M, hidden))
        f = B.linear(f"{nm}_ff1", x1, hidden, ffn, M, act="gelu")
        f2 = B.linear(f"{nm}_ff2", f, ffn, hidden, M, act="none")
        x = B.node(f"{nm}_ln2", "add_layernorm", [f2, x1] + ln_params(f"{nm}_ln2"), dt, (M, hidden))
    cls = B.node("cls", "select_rows", [x], dt, (batch, hidden), stride=seq, offset=0)
    outs = []
    for ti, c in enumerate(tasks):
        p = B.linear(f"task{ti}_pool", cls, hidden, hidden, batch, act="tanh")
        outs.append(B.linear(f"task{ti}", p, hidden, c, batch, act="none", out_dt="f32"))
    B.output(*outs)
    B.outputs = [(f"task{ti}", "f32", (batch, c)) for ti, c in enumerate(tasks)]
    return B.build(batch, config=6)


CONFIGS = {
    "c1": c1_tiny_wd,
    "c2": c2_wide_deep,
    "c3": c3_two_tower,
    "c4": c4_hybrid,
    "c5": c5_ensemble,
    "c6": c6_mtdnn,
}

# Small instances (oracle in seconds; several tiles + ragged tails) used by the parity tests.
SMALL = {
    "c1": dict(),
    "c2": dict(batch=300, fields=5, rows=1000, emb=64, hidden=(192, 136, 72)),
    "c3": dict(batch=72, seq=6, vocab=500, emb=64, hidden=48),
    "c4": dict(batch=3, image=40, seq=5, vocab=400, emb=64, gru_hidden=72, fields=3, rows=500,
               mlp_out=40),
    "c5": dict(batch=200, fields=4, rows=800, vocab=300, image=32, scale=0.125),
    "c6": dict(batch=3, seq=40, layers=2, hidden=128, heads=2, ffn=256, vocab=500),
}


def with_branch_outputs(wl: Workload) -> Workload:
    """Also expose every branch result feeding the final join as a graph output (parity tests check
    each branch, not only the join)."""
    import re
    lines = wl.ir.splitlines()
    decl = {}
    for ln in lines:
        m = re.match(r"^%([\w.]+) = (\w+)\((.*?)\).*: (\w+)\[([0-9,]*)\]$", ln)
        if m:
            decl[m.group(1)] = (m.group(2), [a.strip()[1:] for a in m.group(3).split(",") if a.strip().startswith("%")],
                                m.group(4), tuple(int(x) for x in m.group(5).split(",")))
    join = wl.outputs[0][0]
    extra = [a for a in decl[join][1] if a not in [o[0] for o in wl.outputs]]
    out_idx = next(i for i, ln in enumerate(lines) if ln.startswith("output "))
    lines[out_idx] += "".join(f", %{a}" for a in extra)
    outs = list(wl.outputs) + [(a, decl[a][2], decl[a][3]) for a in extra]
    # duet_run / the oracle order outputs by node declaration order
    order = {nm: i for i, nm in enumerate(decl)}
    outs.sort(key=lambda o: order[o[0]])
    return Workload(wl.name, "\n".join(lines) + "\n", wl.params, wl.inputs, outs, wl.batch, dict(wl.meta))


def rnn_nodes(wl: Workload) -> list:
    import re
    return [m.group(1) for m in (re.match(r"^%([\w.]+) = (?:lstm|gru)\(", ln) for ln in wl.ir.splitlines()) if m]


def with_rnn_tile_n(wl: Workload, tile_n: int) -> Workload:
    """Every LSTM/GRU node with gate-tile width `tile_n` (0 = automatic; include/duet.h `tile_n`).
    The width is an SM budget when branches share the GPU (DESIGN.md "SM sharing between concurrent
    branches"): fewer, wider tiles leave SMs to a co-running branch but lengthen the recurrence."""
    import re
    out = []
    for ln in wl.ir.splitlines():
        if re.match(r"^%[\w.]+ = (?:lstm|gru)\(", ln):
            head, tail = ln.rsplit(" : ", 1)
            m = re.search(r" \{(.*)\}$", head)
            attrs = [a for a in (m.group(1).split(", ") if m else []) if not a.startswith("tile_n=")]
            if tile_n:
                attrs.append(f"tile_n={tile_n}")
            head = head[:m.start()] if m else head
            ln = head + (" {" + ", ".join(attrs) + "}" if attrs else "") + " : " + tail
        out.append(ln)
    meta = dict(wl.meta, rnn_tile_n=tile_n)
    return Workload(wl.name, "\n".join(out) + "\n", wl.params, wl.inputs, list(wl.outputs), wl.batch, meta)


def build(name: str, small: bool = False, dt: str | None = None, branch_outputs: bool = False,
          **kw) -> Workload:
    args = dict(SMALL[name]) if small else {}
    args.update(kw)
    if dt is not None:
        args["dt"] = dt
    wl = CONFIGS[name](**args)
    return with_branch_outputs(wl) if branch_outputs else wl
