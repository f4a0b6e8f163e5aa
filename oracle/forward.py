"""Oracle forward pass in float64 (test infrastructure only; see oracle/__init__.py).

SURVEY.md §8(c) C1: the concurrent DUET execution reaches exactly the plain forward pass of the
model (PAPER.md:79 — a valid schedule only reorders nodes that satisfy all dependencies), so the
oracle is that plain definition written out, one function per IR operator, in float64, with
weights and inputs taken as their exact stored fp32/bf16 values and no intermediate rounding.

Conventions the paper leaves open are fixed by DESIGN.md "Readings" (LSTM/GRU = PyTorch gate
conventions, BN eps 1e-5, joins as in SURVEY.md §8(a) A11).

Parameters/inputs: NumPy arrays in their stored form (float32; bf16 as uint16 bit patterns;
int32/int64).  A parameter may instead be a callable `rows(*lead_index) -> array` for tables too
large to hold (the c2 tables are 3.3 GB); only the gather ops accept that form.
"""
from __future__ import annotations

import numpy as np

from .ir import Graph, parse, topo_order

BN_EPS = 1e-5


# ---- stored value -> float64 ---------------------------------------------------------------
def to_f64(a, dtype: str) -> np.ndarray:
    a = np.asarray(a)
    if dtype == "bf16":
        if a.dtype != np.uint16:
            raise TypeError("bf16 values must be given as uint16 bit patterns")
        return (a.astype(np.uint32) << 16).view(np.float32).astype(np.float64)
    if dtype == "f32":
        return a.astype(np.float32).astype(np.float64)
    if dtype in ("i32", "i64"):
        return a.astype(np.int64)
    raise ValueError(dtype)


def round_bf16(x) -> np.ndarray:
    """float64 -> nearest bf16 value (via float32, round-to-nearest-even on the upper 16 bits).
    Used only by run(..., round_storage=True): the diagnostic reading of DESIGN.md R-26 in which
    every bf16-declared node output is stored rounded, as the GPU stores it."""
    f = np.asarray(x, dtype=np.float64).astype(np.float32)
    b = f.view(np.uint32)
    b = (b + np.uint32(0x7FFF) + ((b >> np.uint32(16)) & np.uint32(1))) & np.uint32(0xFFFF0000)
    return b.view(np.float32).astype(np.float64)


def sigmoid(x):
    # 1 / (1 + e^-x), written to avoid overflow warnings for large |x|
    out = np.empty_like(x, dtype=np.float64)
    pos = x >= 0
    out[pos] = 1.0 / (1.0 + np.exp(-x[pos]))
    ex = np.exp(x[~pos])
    out[~pos] = ex / (1.0 + ex)
    return out


def gelu(x):
    """GELU(x) = x * Phi(x) = 0.5 x (1 + erf(x / sqrt 2)) (the exact form BERT / MT-DNN use)."""
    from scipy.special import erf
    return 0.5 * x * (1.0 + erf(x / np.sqrt(2.0)))


def act(x, name: str):
    if name in (None, "none"):
        return x
    if name == "relu":
        return np.maximum(x, 0.0)
    if name == "sigmoid":
        return sigmoid(x)
    if name == "tanh":
        return np.tanh(x)
    if name == "gelu":
        return gelu(x)
    raise ValueError(name)


# ---- operators -----------------------------------------------------
def hash_mod(raw, V):
    """A3 feature hashing: id = raw mod V (floor modulo)."""
    return np.mod(np.asarray(raw, dtype=np.int64), int(V))


def _table_rows(T, dtype, *lead):
    if callable(T):
        return to_f64(T(*lead), dtype)
    return to_f64(np.asarray(T)[lead], dtype)


def gather_sum(ids, T, T_dtype, b):
    """A4 wide: y[b] = b0 + sum_f T[f, ids[b, f]]  (T is [F, R])."""
    ids = np.asarray(ids, dtype=np.int64)
    B, F = ids.shape
    f_idx = np.broadcast_to(np.arange(F), (B, F))
    vals = _table_rows(T, T_dtype, f_idx, ids)           # [B, F]
    return (vals.sum(axis=1) + b[0]).reshape(B, 1)


def gather_concat(ids, E, E_dtype):
    """A4 deep: X[b, f*D:(f+1)*D] = E[f, ids[b, f], :]  (E is [F, R, D])."""
    ids = np.asarray(ids, dtype=np.int64)
    B, F = ids.shape
    f_idx = np.broadcast_to(np.arange(F), (B, F))
    rows = _table_rows(E, E_dtype, f_idx, ids)           # [B, F, D]
    return rows.reshape(B, -1)


def embed_seq(tok, E, E_dtype):
    """A4 tokens, time-major: X[t, b, :] = E[tok[b, t], :]  (E is [V, D])."""
    tok = np.asarray(tok, dtype=np.int64)
    rows = _table_rows(E, E_dtype, tok.T)               # [S, B, D]
    return rows


def linear(x, W, b, a="none"):
    """A5: y = act(x W^T + b), W is [N, K]."""
    return act(x @ W.T + b, a)


def mlp(x, layers, a="relu", last_act="none"):
    for i, (W, b) in enumerate(layers):
        x = linear(x, W, b, a if i + 1 < len(layers) else last_act)
    return x


def reduce_sum(x, b):
    return (x.sum(axis=1) + b[0]).reshape(-1, 1)


def lstm(x, Wih, Whh, bih, bhh, seq=False):
    """A6+A7, PyTorch nn.LSTM conventions (gate order i,f,g,o; h0 = c0 = 0); returns h_S, or
    with `seq` every h_t as [S, B, H] (the input of the next layer of a stacked RNN, PAPER.md:89
    "Varying the stacked RNN layers", Fig. 14)."""
    S, B, _ = x.shape
    H = Whh.shape[1]
    h = np.zeros((B, H))
    c = np.zeros((B, H))
    hs = []
    for t in range(S):
        g = x[t] @ Wih.T + bih + h @ Whh.T + bhh
        i, f, gg, o = g[:, :H], g[:, H:2 * H], g[:, 2 * H:3 * H], g[:, 3 * H:]
        i, f, gg, o = sigmoid(i), sigmoid(f), np.tanh(gg), sigmoid(o)
        c = f * c + i * gg
        h = o * np.tanh(c)
        hs.append(h)
    return np.stack(hs) if seq else h


def gru(x, Wih, Whh, bih, bhh, seq=False):
    """A6+A8, PyTorch nn.GRU conventions (r,z,n; b_hn inside r*(.); h0 = 0); returns h_S, or
    with `seq` every h_t as [S, B, H] (stacked layers, as lstm)."""
    S, B, _ = x.shape
    H = Whh.shape[1]
    h = np.zeros((B, H))
    hs = []
    for t in range(S):
        gx = x[t] @ Wih.T + bih
        gh = h @ Whh.T + bhh
        r = sigmoid(gx[:, :H] + gh[:, :H])
        z = sigmoid(gx[:, H:2 * H] + gh[:, H:2 * H])
        n = np.tanh(gx[:, 2 * H:] + r * gh[:, 2 * H:])
        h = (1.0 - z) * n + z * h
        hs.append(h)
    return np.stack(hs) if seq else h


def conv2d(x, W, stride, pad):
    """Plain NHWC convolution, W is [Cout, kh, kw, Cin]: a sum of kh*kw shifted matmuls."""
    N, H, Wd, C = x.shape
    Co, kh, kw, Ci = W.shape
    assert Ci == C
    Ho = (H + 2 * pad - kh) // stride + 1
    Wo = (Wd + 2 * pad - kw) // stride + 1
    xp = np.zeros((N, H + 2 * pad, Wd + 2 * pad, C))
    xp[:, pad:pad + H, pad:pad + Wd, :] = x
    y = np.zeros((N, Ho, Wo, Co))
    for r in range(kh):
        for s in range(kw):
            patch = xp[:, r:r + stride * (Ho - 1) + 1:stride, s:s + stride * (Wo - 1) + 1:stride, :]
            y += patch @ W[:, r, s, :].T
    return y


def batchnorm(y, gamma, beta, mean, var):
    """Inference BN: (y - mu) / sqrt(var + eps) * gamma + beta."""
    return (y - mean) / np.sqrt(var + BN_EPS) * gamma + beta


def conv2d_bn(x, W, gamma, beta, mean, var, stride, pad, a):
    """A9: conv -> BN -> act (the oracle applies BN explicitly; the GPU folds it)."""
    return act(batchnorm(conv2d(x, W, stride, pad), gamma, beta, mean, var), a)


def maxpool(x, k, stride, pad):
    N, H, W, C = x.shape
    Ho = (H + 2 * pad - k) // stride + 1
    Wo = (W + 2 * pad - k) // stride + 1
    xp = np.full((N, H + 2 * pad, W + 2 * pad, C), -np.inf)
    xp[:, pad:pad + H, pad:pad + W, :] = x
    y = np.full((N, Ho, Wo, C), -np.inf)
    for r in range(k):
        for s in range(k):
            y = np.maximum(y, xp[:, r:r + stride * (Ho - 1) + 1:stride,
                                 s:s + stride * (Wo - 1) + 1:stride, :])
    return y


def avgpool(x):
    """Global average pool over H, W: [N, H, W, C] -> [N, C]."""
    return x.mean(axis=(1, 2))


def dot_join(s, a, w, b):
    """A11 c2: y = sigma(wide + w . a + b)."""
    return sigmoid(s[:, 0] + a @ w + b[0]).reshape(-1, 1)


def cosine_join(a, b):
    """A11 c3: cos(a, b) = a.b / (|a| |b|); 0 when a norm is 0."""
    num = (a * b).sum(axis=1)
    den = np.sqrt((a * a).sum(axis=1)) * np.sqrt((b * b).sum(axis=1))
    out = np.where(den > 0, num / np.where(den > 0, den, 1.0), 0.0)
    return out.reshape(-1, 1)


def concat_head(parts, w, b, a="sigmoid"):
    """A11 c4: y = act(w . concat(parts) + b)."""
    x = np.concatenate(parts, axis=1)
    return act(x @ w + b[0], a).reshape(-1, 1)


def sum_join(parts):
    """A11 c1: y = sigma(sum of branch logits)."""
    return sigmoid(sum(p[:, 0] for p in parts)).reshape(-1, 1)


def mean_join(parts):
    """A11 c5: y = sigma(mean of branch logits)."""
    return sigmoid(sum(p[:, 0] for p in parts) / len(parts)).reshape(-1, 1)


# ---- MT-DNN ("shared layer ... lexicon encoder and a multi-layer bidirectional
# Transformer encoder ... task-specific output layers", Fig. 3) ----------
LN_EPS = 1e-12  # BERT's LayerNorm epsilon (MT-DNN's encoder is BERT's)


def layernorm(x, gamma, beta, eps=LN_EPS):
    """Over the last axis: (x - mean) / sqrt(var + eps) * gamma + beta (biased variance)."""
    mu = x.mean(axis=-1, keepdims=True)
    var = ((x - mu) ** 2).mean(axis=-1, keepdims=True)
    return (x - mu) / np.sqrt(var + eps) * gamma + beta


def bert_embed(tok, seg, Wtok, Wpos, Wseg, gamma, beta, eps=LN_EPS):
    """Lexicon encoder: LN(E_tok[tok[b, s]] + E_pos[s] + E_seg[seg[b, s]]), rows b*S + s -> [B*S, H]."""
    tok = np.asarray(tok, dtype=np.int64)
    seg = np.asarray(seg, dtype=np.int64)
    B, S = tok.shape
    x = Wtok[tok] + Wpos[:S][None, :, :] + Wseg[seg]
    return layernorm(x, gamma, beta, eps).reshape(B * S, -1)


def attention(qkv, heads, seq):
    """Bidirectional multi-head self-attention (Vaswani et al.; no mask: fixed length, R-31).
    qkv = [Q | K | V] per row ([B*S, 3H], rows b*S + s; head h = columns h*dh .. of each part);
    out[b, s, h] = softmax(Q_h K_h^T / sqrt(dh)) V_h -> [B*S, H]."""
    M, H3 = qkv.shape
    H = H3 // 3
    dh = H // heads
    B = M // seq
    q = qkv[:, :H].reshape(B, seq, heads, dh).transpose(0, 2, 1, 3)
    k = qkv[:, H:2 * H].reshape(B, seq, heads, dh).transpose(0, 2, 1, 3)
    v = qkv[:, 2 * H:].reshape(B, seq, heads, dh).transpose(0, 2, 1, 3)
    sc = q @ k.transpose(0, 1, 3, 2) / np.sqrt(dh)          # [B, heads, S, S]
    sc = sc - sc.max(axis=-1, keepdims=True)
    p = np.exp(sc)
    p = p / p.sum(axis=-1, keepdims=True)
    return (p @ v).transpose(0, 2, 1, 3).reshape(M, H)


def add_layernorm(a, b, gamma, beta, eps=LN_EPS):
    """Post-LN residual: LN(a + b)."""
    return layernorm(a + b, gamma, beta, eps)


def select_rows(x, stride, offset=0):
    """Rows offset, offset + stride, ... (the [CLS] token of every sequence)."""
    return x[offset::stride]


# ---- graph evaluation -----------------------------------------------------------------------
def run(ir, params: dict, inputs: dict, keep_all: bool = False, round_storage: bool = False) -> dict:
    """Evaluate the graph in topological order.  Returns {output name: float64 array}
    (or every node value if keep_all).  Shapes come from the arrays, not the IR, so a batch
    subset of the inputs evaluates exactly those rows (inference rows are independent).
    round_storage: round every bf16-declared node output to bf16 (the R-26 storage reading; a
    diagnostic that separates activation-storage rounding from kernel error -- the parity bar
    is always against the unrounded pass)."""
    g: Graph = parse(ir) if isinstance(ir, str) else ir
    val = {}

    def P(name):
        dt, _ = g.params[name]
        p = params[name]
        return p if callable(p) else to_f64(p, dt)

    def Pdt(name):
        return g.params[name][0]

    for nid in topo_order(g):
        n = g.nodes[nid]
        A = [val[nm] for k, nm in n.args if k == "%"]
        pn = [nm for k, nm in n.args if k == "@"]
        op, at = n.op, n.attrs
        if op == "input":
            v = to_f64(inputs[n.name], n.dtype)
        elif op == "hash_mod":
            v = hash_mod(A[0], at["V"])
        elif op == "gather_sum":
            v = gather_sum(A[0], params[pn[0]], Pdt(pn[0]), P(pn[1]))
        elif op == "gather_concat":
            v = gather_concat(A[0], params[pn[0]], Pdt(pn[0]))
        elif op == "embed_seq":
            v = embed_seq(A[0], params[pn[0]], Pdt(pn[0]))
        elif op == "linear":
            v = linear(A[0], P(pn[0]), P(pn[1]), at.get("act", "none"))
        elif op == "mlp":
            layers = [(P(pn[i]), P(pn[i + 1])) for i in range(0, len(pn), 2)]
            v = mlp(A[0], layers, at.get("act", "relu"), at.get("last_act", "none"))
        elif op == "reduce_sum":
            v = reduce_sum(A[0], P(pn[0]))
        elif op == "lstm":
            v = lstm(A[0], *(P(p) for p in pn), seq=bool(int(at.get("seq", 0))))
        elif op == "gru":
            v = gru(A[0], *(P(p) for p in pn), seq=bool(int(at.get("seq", 0))))
        elif op == "conv2d_bn":
            v = conv2d_bn(A[0], *(P(p) for p in pn), at["stride"], at["pad"], at.get("act", "none"))
        elif op == "add":
            v = act(A[0] + A[1], at.get("act", "none"))
        elif op == "maxpool":
            v = maxpool(A[0], at["k"], at["stride"], at["pad"])
        elif op == "avgpool":
            v = avgpool(A[0])
        elif op == "dot_join":
            v = dot_join(A[0], A[1], P(pn[0]), P(pn[1]))
        elif op == "cosine_join":
            v = cosine_join(A[0], A[1])
        elif op == "concat_head":
            v = concat_head(A, P(pn[0]), P(pn[1]), at.get("act", "sigmoid"))
        elif op == "sum_join":
            v = sum_join(A)
        elif op == "mean_join":
            v = mean_join(A)
        elif op == "sigmoid":
            v = sigmoid(A[0])
        elif op == "bert_embed":
            v = bert_embed(A[0], A[1], *(P(p) for p in pn))
        elif op == "attention":
            v = attention(A[0], int(at["heads"]), int(at["seq"]))
        elif op == "add_layernorm":
            v = add_layernorm(A[0], A[1], P(pn[0]), P(pn[1]))
        elif op == "select_rows":
            v = select_rows(A[0], int(at["stride"]), int(at.get("offset", 0)))
        else:
            raise ValueError(f"oracle has no operator {op!r}")
        if round_storage and n.dtype == "bf16" and op != "input":
            v = round_bf16(v)
        val[n.name] = v
    if keep_all:
        return val
    return {g.nodes[i].name: val[g.nodes[i].name] for i in g.outputs}
