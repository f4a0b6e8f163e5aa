"""Pins for the float64 forward oracle: hand-computed values, closed
forms, and torch float64 modules (test-only cross-check; the oracle itself is NumPy)."""
import math

import numpy as np
import pytest
import torch

from oracle import forward as F
from oracle.ir import IRError, parse


def f32(a):
    return np.asarray(a, dtype=np.float32)


def bf16_bits(a):
    t = torch.tensor(np.asarray(a, dtype=np.float32)).to(torch.bfloat16)
    return t.view(torch.int16).numpy().view(np.uint16)


# ---- hand-computed 2-layer toy (SURVEY.md C-P "Forward, MLP/sigmoid") -----------------------
TOY = """
param @W1 : {dt}[2,2]
param @b1 : f32[2]
param @W2 : {dt}[1,2]
param @b2 : f32[1]
%x = input() : {dt}[1,2]
%h = linear(%x, @W1, @b1) {{act=relu}} : {dt}[1,2]
%y = linear(%h, @W2, @b2) {{act=sigmoid}} : f32[1,1]
output %y
"""
TOY_Y = 0.029312230751356319  # sigma(-3.5), h = relu([-2.5, 4.5]) = [0, 4.5], z = 2*0 - 4.5 + 1


@pytest.mark.parametrize("dt", ["f32", "bf16"])
def test_toy_mlp_hand_computed(dt):
    enc = f32 if dt == "f32" else bf16_bits
    params = {"W1": enc([[1, 2], [3, -1]]), "b1": f32([0.5, -0.5]), "W2": enc([[2, -1]]),
              "b2": f32([1])}
    out = F.run(TOY.format(dt=dt), params, {"x": enc([[1, -2]])}, keep_all=True)
    np.testing.assert_array_equal(out["h"], [[0.0, 4.5]])
    assert out["y"][0, 0] == pytest.approx(TOY_Y, rel=1e-15)
    assert 1.0 / (1.0 + math.exp(3.5)) == pytest.approx(TOY_Y, rel=1e-15)


# ---- gathers: integer table pattern, exact ----------------------------------------------------
def _pattern_table(F_, R, D):
    f, v, k = np.meshgrid(np.arange(F_), np.arange(R), np.arange(D), indexing="ij")
    return ((7 * v + 3 * k + 11 * f) % 251) - 125


def test_gather_concat_and_sum_pattern():
    F_, R, D, B = 4, 300, 8, 9
    E = _pattern_table(F_, R, D)
    rng = np.random.default_rng(0)
    ids = rng.integers(0, R, size=(B, F_))
    out = F.gather_concat(ids, f32(E), "f32")
    for b in range(B):
        for f in range(F_):
            for k in range(D):
                assert out[b, f * D + k] == ((7 * ids[b, f] + 3 * k + 11 * f) % 251) - 125
    Tw = _pattern_table(F_, R, 1)[:, :, 0]
    ws = F.gather_sum(ids, bf16_bits(Tw), "bf16", np.array([0.5]))
    for b in range(B):
        assert ws[b, 0] == 0.5 + sum(((7 * ids[b, f] + 11 * f) % 251) - 125 for f in range(F_))


def test_hash_mod_floor():
    raw = np.array([[0, 5, 10**12 + 7, 2**31 - 1]], dtype=np.int64)
    np.testing.assert_array_equal(F.hash_mod(raw, 1000), [[0, 5, (10**12 + 7) % 1000, (2**31 - 1) % 1000]])
    assert F.hash_mod(np.array([-3]), 10)[0] == 7


def test_embed_seq_time_major():
    E = np.arange(20, dtype=np.float32).reshape(10, 2)
    tok = np.array([[1, 2, 3], [4, 5, 6]])
    x = F.embed_seq(tok, E, "f32")
    assert x.shape == (3, 2, 2)
    np.testing.assert_array_equal(x[2, 1], E[6])


# ---- LSTM / GRU closed forms (weights 0) and torch float64 ---------------------------------------
def test_lstm_zero_weight_closed_form():
    H, S, B, E = 3, 7, 2, 4
    bih = np.array([0.3, -0.2, 0.1, 0.5, 0.7, 0.2, -0.4, 0.6, -0.1, 0.2, 0.3, -0.3])
    bhh = np.array([0.1] * 12)
    x = np.random.default_rng(1).normal(size=(S, B, E))
    h = F.lstm(x, np.zeros((4 * H, E)), np.zeros((4 * H, H)), bih, bhh)
    bx = bih + bhh
    sg = lambda v: 1 / (1 + np.exp(-v))
    i, f, g, o = sg(bx[:H]), sg(bx[H:2 * H]), np.tanh(bx[2 * H:3 * H]), sg(bx[3 * H:])
    c = i * g * (1 - f ** S) / (1 - f)
    np.testing.assert_allclose(h, np.broadcast_to(o * np.tanh(c), (B, H)), rtol=1e-13)


def test_gru_zero_weight_closed_form():
    H, S, B, E = 3, 5, 2, 4
    bih = np.array([0.3, -0.2, 0.1, 0.5, 0.7, 0.2, -0.4, 0.6, -0.1])
    bhh = np.array([0.2, 0.1, -0.3, 0.05, 0.0, 0.4, 0.3, -0.2, 0.25])
    x = np.random.default_rng(2).normal(size=(S, B, E))
    h = F.gru(x, np.zeros((3 * H, E)), np.zeros((3 * H, H)), bih, bhh)
    sg = lambda v: 1 / (1 + np.exp(-v))
    r = sg(bih[:H] + bhh[:H])
    z = sg(bih[H:2 * H] + bhh[H:2 * H])
    n = np.tanh(bih[2 * H:] + r * bhh[2 * H:])
    np.testing.assert_allclose(h, np.broadcast_to(n * (1 - z ** S), (B, H)), rtol=1e-13)


@pytest.mark.parametrize("kind", ["lstm", "gru"])
def test_rnn_vs_torch_f64(kind):
    S, B, E, H = 6, 5, 7, 9
    torch.manual_seed(0)
    mod = (torch.nn.LSTM if kind == "lstm" else torch.nn.GRU)(E, H).double()
    x = torch.randn(S, B, E, dtype=torch.float64)
    _, st = mod(x)
    want = (st[0] if kind == "lstm" else st)[0].detach().numpy()
    fn = F.lstm if kind == "lstm" else F.gru
    got = fn(x.numpy(), mod.weight_ih_l0.detach().numpy(), mod.weight_hh_l0.detach().numpy(),
             mod.bias_ih_l0.detach().numpy(), mod.bias_hh_l0.detach().numpy())
    np.testing.assert_allclose(got, want, rtol=1e-12, atol=1e-14)


# ---- conv / BN / pooling ----------------------------------------------------------------------
def test_conv_center_tap_identity_and_bn_identity():
    x = np.random.default_rng(3).normal(size=(2, 5, 6, 4))
    W = np.zeros((4, 3, 3, 4))
    for c in range(4):
        W[c, 1, 1, c] = 1.0
    y = F.conv2d_bn(x, W, np.ones(4), np.zeros(4), np.zeros(4), np.full(4, 1 - 1e-5), 1, 1, "none")
    np.testing.assert_allclose(y, x, rtol=1e-12, atol=1e-15)


@pytest.mark.parametrize("stride,pad,k", [(1, 1, 3), (2, 1, 3), (2, 3, 7), (2, 0, 1)])
def test_conv_bn_vs_torch_f64(stride, pad, k):
    rng = np.random.default_rng(4)
    N, H, W_, C, Co = 2, 11, 9, 3, 5
    x = rng.normal(size=(N, H, W_, C))
    Wt = rng.normal(size=(Co, k, k, C))
    g, b, mu, var = rng.uniform(0.5, 1.5, Co), rng.normal(size=Co), rng.normal(size=Co), rng.uniform(0.5, 1.5, Co)
    got = F.conv2d_bn(x, Wt, g, b, mu, var, stride, pad, "relu")
    conv = torch.nn.functional.conv2d(torch.tensor(x).permute(0, 3, 1, 2),
                                      torch.tensor(Wt).permute(0, 3, 1, 2), stride=stride, padding=pad)
    bn = torch.nn.functional.batch_norm(conv, torch.tensor(mu), torch.tensor(var), torch.tensor(g),
                                        torch.tensor(b), training=False, eps=1e-5)
    want = torch.relu(bn).permute(0, 2, 3, 1).numpy()
    np.testing.assert_allclose(got, want, rtol=1e-11, atol=1e-12)


def test_maxpool_avgpool_vs_torch():
    x = np.random.default_rng(5).normal(size=(2, 9, 8, 3))
    got = F.maxpool(x, 3, 2, 1)
    want = torch.nn.functional.max_pool2d(torch.tensor(x).permute(0, 3, 1, 2), 3, 2, 1).permute(0, 2, 3, 1)
    np.testing.assert_array_equal(got, want.numpy())
    np.testing.assert_allclose(F.avgpool(x), x.reshape(2, -1, 3).mean(1), rtol=1e-14)


@pytest.mark.parametrize("depth", [18, 34, 50, 101])
def test_resnet_small_vs_torch_f64(depth):
    """The workload's ResNet-`depth` IR through the oracle == a torch float64 ResNet built here
    from nn.functional conv2d / batch_norm (torchvision BasicBlock for 18/34, Bottleneck with the
    stride on the 3x3 conv for 50/101; Fig. 15's depths)."""
    from paper_conf_ipps_zhanghl21_b200 import workloads as W
    wl = W.build("c4", small=True, dt="f32", resnet=depth)
    params = {k: s.materialize().numpy() for k, s in wl.params.items()}
    img = wl.inputs["image"].materialize().numpy()
    vals = F.run(wl.ir, params, {"image": img, "tok": wl.inputs["tok"].materialize().numpy(),
                                 "raw": wl.inputs["raw"].materialize().numpy()}, keep_all=True)

    def P(n):
        return torch.tensor(params[n], dtype=torch.float64)

    def cbn(x, name, stride, pad, relu):
        y = torch.nn.functional.conv2d(x, P(name + "_W").permute(0, 3, 1, 2), stride=stride, padding=pad)
        y = torch.nn.functional.batch_norm(y, P(name + "_mean"), P(name + "_var"), P(name + "_gamma"),
                                           P(name + "_beta"), training=False, eps=1e-5)
        return torch.relu(y) if relu else y

    blocks = {18: (2, 2, 2, 2), 34: (3, 4, 6, 3), 50: (3, 4, 6, 3), 101: (3, 4, 23, 3)}[depth]
    exp = 1 if depth < 50 else 4
    x = torch.tensor(img, dtype=torch.float64).permute(0, 3, 1, 2)
    x = cbn(x, "cnn_stem", 2, 3, True)
    x = torch.nn.functional.max_pool2d(x, 3, 2, 1)
    cin = 64
    for li, width in enumerate([64, 128, 256, 512]):
        cout = width * exp
        for bi in range(blocks[li]):
            s = 2 if (li > 0 and bi == 0) else 1
            nm = f"cnn_l{li + 1}b{bi}"
            if exp == 1:
                y = cbn(x, nm + "_c1", s, 1, True)
                y = cbn(y, nm + "_c2", 1, 1, False)
            else:
                y = cbn(x, nm + "_c1", 1, 0, True)
                y = cbn(y, nm + "_c2", s, 1, True)
                y = cbn(y, nm + "_c3", 1, 0, False)
            sc = cbn(x, nm + "_ds", s, 0, False) if (s != 1 or cin != cout) else x
            x = torch.relu(y + sc)
            cin = cout
    want = x.mean(dim=(2, 3)).numpy()
    assert want.shape[1] == 512 * exp
    np.testing.assert_allclose(vals["cnn_gap"], want, rtol=1e-10, atol=1e-12)


@pytest.mark.parametrize("layers", [1, 2, 4])
def test_stacked_gru_vs_torch_f64(layers):
    """Stacked RNN (Fig. 14): the workload's `layers`-deep GRU IR (lower layers emit
    their whole sequence, `seq=1`) through the oracle == torch nn.GRU(num_layers=layers) in f64."""
    from paper_conf_ipps_zhanghl21_b200 import workloads as W
    wl = W.build("c4", small=True, dt="f32", rnn_layers=layers)
    params = {k: s.materialize().numpy() for k, s in wl.params.items()}
    ins = {k: s.materialize().numpy() for k, s in wl.inputs.items()}
    vals = F.run(wl.ir, params, ins, keep_all=True)
    E, H = params["tok_E"].shape[1], params["gru_Whh"].shape[1]
    mod = torch.nn.GRU(E, H, num_layers=layers).double()
    names = [f"gru_l{i}" for i in range(layers - 1)] + ["gru"]
    with torch.no_grad():
        for i, nm in enumerate(names):
            for a, b in (("Wih", "weight_ih"), ("Whh", "weight_hh"), ("bih", "bias_ih"), ("bhh", "bias_hh")):
                getattr(mod, f"{b}_l{i}").copy_(torch.tensor(params[f"{nm}_{a}"], dtype=torch.float64))
    x = torch.tensor(vals["tok_x"])
    with torch.no_grad():
        out, hn = mod(x)
    np.testing.assert_allclose(vals["gru"], hn[-1].numpy(), rtol=1e-11, atol=1e-13)
    if layers > 1:  # a lower layer's seq output is torch's per-layer output sequence
        sub = torch.nn.GRU(E, H).double()
        with torch.no_grad():
            for a, b in (("Wih", "weight_ih"), ("Whh", "weight_hh"), ("bih", "bias_ih"), ("bhh", "bias_hh")):
                getattr(sub, f"{b}_l0").copy_(getattr(mod, f"{b}_l0"))
            seq0, _ = sub(x)
        np.testing.assert_allclose(vals["gru_l0"], seq0.numpy(), rtol=1e-11, atol=1e-13)


def test_stacked_lstm_vs_torch_f64():
    S, B, E, H = 5, 4, 6, 7
    torch.manual_seed(3)
    mod = torch.nn.LSTM(E, H, num_layers=3).double()
    x = torch.randn(S, B, E, dtype=torch.float64)
    with torch.no_grad():
        out, (hn, _) = mod(x)
    v = x.numpy()
    for i in range(3):
        w = [getattr(mod, f"{n}_l{i}").detach().numpy() for n in ("weight_ih", "weight_hh", "bias_ih", "bias_hh")]
        v = F.lstm(v, *w, seq=i < 2)
    np.testing.assert_allclose(v, hn[-1].numpy(), rtol=1e-11, atol=1e-13)


# ---- joins --------------------------------------------------------------------------------------
def test_joins_special_cases():
    a = np.random.default_rng(6).normal(size=(4, 8))
    np.testing.assert_allclose(F.cosine_join(a, a)[:, 0], 1.0, rtol=1e-14)
    np.testing.assert_allclose(F.cosine_join(a, -a)[:, 0], -1.0, rtol=1e-14)
    assert F.cosine_join(np.zeros((1, 3)), np.ones((1, 3)))[0, 0] == 0.0
    l = np.full((4, 1), 0.37)
    np.testing.assert_allclose(F.mean_join([l, l, l]), F.sigmoid(l), rtol=1e-15)
    np.testing.assert_allclose(F.sum_join([l, -l]), 0.5, rtol=1e-15)
    s = np.array([[0.25]])
    np.testing.assert_allclose(F.dot_join(s, np.array([[1.0, 2.0]]), np.array([0.5, -1.0]),
                                          np.array([0.25])), F.sigmoid(np.array([[0.25 + 0.5 - 2 + 0.25]])))
    x = F.concat_head([np.array([[1.0]]), np.array([[2.0, 3.0]])], np.array([1.0, 1.0, -1.0]),
                      np.array([0.0]), "none")
    assert x[0, 0] == 0.0
    assert F.sigmoid(np.array([-800.0, 800.0])).tolist() == [0.0, 1.0]


# ---- IR reader ------------------------------------------------------------------------------------
def test_ir_errors():
    with pytest.raises(IRError):
        parse("%a = add(%b, %b) : f32[1]\n%b = add(%a, %a) : f32[1]\n")  # cycle
    with pytest.raises(IRError):
        parse("%a = linear(%x, @W, @b) : f32[1]\n")  # undefined
    with pytest.raises(IRError):
        parse("%a = input() : f16[1]\n")  # bad dtype
    g = parse("# c\n%x = input() : f32[2,3]\n%y = sigmoid(%x) : f32[2,3]\noutput %y\n")
    assert [n.op for n in g.nodes] == ["input", "sigmoid"] and g.outputs == [1]


# ---- MT-DNN operators (Fig. 3) -----------------------------
def test_gelu_identities_and_torch():
    x = np.linspace(-6, 6, 97)
    g = F.gelu(x)
    np.testing.assert_allclose(g - F.gelu(-x), x, rtol=0, atol=1e-14)       # Phi(x) + Phi(-x) = 1
    assert F.gelu(np.array([0.0]))[0] == 0.0
    np.testing.assert_allclose(F.gelu(np.array([1.0])), [0.8413447460685429], rtol=1e-15)  # Phi(1)
    want = torch.nn.functional.gelu(torch.tensor(x, dtype=torch.float64)).numpy()
    np.testing.assert_allclose(g, want, rtol=1e-14, atol=1e-15)


def test_layernorm_vs_torch_and_invariants():
    rng = np.random.default_rng(4)
    x = rng.normal(size=(7, 33)) * 3 + 1
    g, b = rng.uniform(0.5, 1.5, 33), rng.normal(size=33)
    want = torch.nn.functional.layer_norm(torch.tensor(x), (33,), torch.tensor(g), torch.tensor(b), eps=1e-12)
    np.testing.assert_allclose(F.layernorm(x, g, b), want.numpy(), rtol=1e-12, atol=1e-12)
    y = F.layernorm(x, np.ones(33), np.zeros(33))
    np.testing.assert_allclose(y.mean(axis=1), 0, atol=1e-12)
    np.testing.assert_allclose(y.var(axis=1), 1, rtol=1e-10)


def test_attention_vs_torch_sdpa():
    rng = np.random.default_rng(5)
    B, S, heads, dh = 2, 9, 3, 8
    H = heads * dh
    qkv = rng.normal(size=(B * S, 3 * H))
    got = F.attention(qkv, heads, S)
    t = torch.tensor(qkv).reshape(B, S, 3, heads, dh).permute(2, 0, 3, 1, 4)   # [3, B, heads, S, dh]
    want = torch.nn.functional.scaled_dot_product_attention(t[0], t[1], t[2])   # no mask, 1/sqrt(dh)
    np.testing.assert_allclose(got, want.permute(0, 2, 1, 3).reshape(B * S, H).numpy(), rtol=1e-12, atol=1e-13)
    # a single key: attention returns its value row for every query
    one = F.attention(rng.normal(size=(4, 3 * H)), heads, 1)
    assert one.shape == (4, H)


def test_mtdnn_layer_vs_torch_encoder_layer():
    """c6's embedding + first encoder layer through the oracle == torch nn.Embedding / layer_norm +
    nn.TransformerEncoderLayer (post-LN, GELU, eps 1e-12) in float64 with the same weights."""
    from paper_conf_ipps_zhanghl21_b200 import workloads as W
    wl = W.build("c6", small=True, dt="f32")
    prm = {k: s.materialize().numpy() for k, s in wl.params.items()}
    ins = {k: s.materialize().numpy() for k, s in wl.inputs.items()}
    vals = F.run(wl.ir, prm, ins, keep_all=True)
    T = lambda n: torch.tensor(prm[n], dtype=torch.float64)
    tok, seg = torch.tensor(ins["tok"]).long(), torch.tensor(ins["seg"]).long()
    B, S = tok.shape
    H = prm["tok_E"].shape[1]
    e = torch.nn.functional.embedding(tok, T("tok_E")) + T("pos_E")[:S] + torch.nn.functional.embedding(seg, T("seg_E"))
    e = torch.nn.functional.layer_norm(e, (H,), T("emb_g"), T("emb_b"), eps=1e-12)
    np.testing.assert_allclose(vals["emb"], e.reshape(B * S, H).numpy(), rtol=1e-11, atol=1e-11)
    layer = torch.nn.TransformerEncoderLayer(H, 2, prm["L0_ff1_W"].shape[0], dropout=0.0, activation="gelu",
                                             layer_norm_eps=1e-12, batch_first=True, norm_first=False).double()
    with torch.no_grad():
        layer.self_attn.in_proj_weight.copy_(T("L0_qkv_W"))
        layer.self_attn.in_proj_bias.copy_(T("L0_qkv_b"))
        layer.self_attn.out_proj.weight.copy_(T("L0_o_W"))
        layer.self_attn.out_proj.bias.copy_(T("L0_o_b"))
        layer.linear1.weight.copy_(T("L0_ff1_W"))
        layer.linear1.bias.copy_(T("L0_ff1_b"))
        layer.linear2.weight.copy_(T("L0_ff2_W"))
        layer.linear2.bias.copy_(T("L0_ff2_b"))
        for ln in ("ln1", "ln2"):
            getattr(layer, "norm" + ln[-1]).weight.copy_(T(f"L0_{ln}_g"))
            getattr(layer, "norm" + ln[-1]).bias.copy_(T(f"L0_{ln}_b"))
        layer.eval()
        want = layer(e)
    np.testing.assert_allclose(vals["L0_ln2"], want.reshape(B * S, H).numpy(), rtol=1e-10, atol=1e-10)
    # [CLS] rows feed the task heads
    np.testing.assert_allclose(vals["cls"], vals["L1_ln2"][::S])


def test_reduce_sum_closed_form():
    """c1/c2 wide part 'wide = reduce_sum(gathered weights) + b0' (Cheng et al.'s
    wide model): row sums of integer rows.  Row r = [r, r+1, ..., r+F-1] sums to F*r + F(F-1)/2;
    through the IR as well (op dispatch, bias parameter, [B, 1] shape)."""
    B, F_ = 5, 26
    x = np.arange(B)[:, None] + np.arange(F_)[None, :]
    got = F.reduce_sum(x.astype(np.float64), np.array([0.5]))
    assert got.shape == (B, 1)
    assert got[:, 0].tolist() == [F_ * r + F_ * (F_ - 1) / 2 + 0.5 for r in range(B)]
    ir = f"param @b : f32[1]\n%x = input() : f32[{B},{F_}]\n%y = reduce_sum(%x, @b) : f32[{B},1]\noutput %y\n"
    y = F.run(ir, {"b": np.array([-3.0], np.float32)}, {"x": x.astype(np.float32)})["y"]
    assert y[:, 0].tolist() == [F_ * r + 325 - 3 for r in range(B)]


def test_select_rows_closed_form():
    """MT-DNN's [CLS] select (Fig. 3; R-31): rows offset, offset + S, ... of a
    [B*S, H] activation.  With x[i, k] = 1000 i + k the selected row b is 1000 (b S + offset) + k."""
    B, S, H = 3, 7, 4
    x = 1000.0 * np.arange(B * S)[:, None] + np.arange(H)[None, :]
    for off in (0, 2, S - 1):
        got = F.select_rows(x, S, off)
        assert got.shape == (B, H)
        want = [[1000 * (b * S + off) + k for k in range(H)] for b in range(B)]
        assert got.tolist() == want
    ir = (f"%x = input() : f32[{B * S},{H}]\n%c = select_rows(%x) {{stride={S}, offset=1}} : f32[{B},{H}]\n"
          "output %c\n")
    y = F.run(ir, {}, {"x": x.astype(np.float32)})["c"]
    assert y[:, 0].tolist() == [1000 * (b * S + 1) for b in range(B)]


def test_round_bf16_matches_torch():
    """The R-26 storage-rounding helper is round-to-nearest-even to bf16 (torch's conversion)."""
    rng = np.random.default_rng(3)
    x = np.concatenate([rng.standard_normal(1000) * 10.0 ** rng.integers(-6, 6, 1000),
                        [0.0, -0.0, 1 + 2 ** -8, 1 + 3 * 2 ** -8, 65504.0, 3e38]])
    want = torch.tensor(x).to(torch.float32).to(torch.bfloat16).double().numpy()
    np.testing.assert_array_equal(F.round_bf16(x), want)


def test_bf16_storage_error_grows_with_resnet_depth():
    """Why the deep §VI-D variants sit closest to the bf16 bar (Fig. 15; R-26,
    R-28): rounding every bf16 activation, with exact arithmetic otherwise, already moves c4's output
    by an amount that grows with the ResNet depth (more rounded residual-stream stores).  The
    depth-scaled residual gamma (R-28) keeps it below 0.7 x the 2e-2 bar at every depth, leaving
    the kernels a margin."""
    from paper_conf_ipps_zhanghl21_b200 import workloads as W
    from tests.helpers import oracle_arrays, rel_err
    errs = {}
    for depth in (18, 101):
        wl = W.build("c4", small=True, resnet=depth, batch=8)
        P = oracle_arrays({k: v.materialize("cpu") for k, v in wl.params.items()})
        I = oracle_arrays({k: v.materialize("cpu") for k, v in wl.inputs.items()})
        a, b = F.run(wl.ir, P, I)["y"], F.run(wl.ir, P, I, round_storage=True)["y"]
        errs[depth] = rel_err(b, a)
    assert 0 < errs[18] < errs[101] < 0.7 * 2e-2, errs
