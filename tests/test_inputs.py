"""The seeded generator is bit-reproducible: torch int64 arithmetic equals an independent NumPy
uint64 re-implementation, and row extraction equals full materialisation."""
import numpy as np
import torch

from paper_conf_ipps_zhanghl21_b200 import inputs as G
from paper_conf_ipps_zhanghl21_b200 import workloads as W


def _np_mix32(x):
    x = x.astype(np.uint64)
    m = np.uint64(0xFFFFFFFF)
    x ^= x >> np.uint64(16)
    x = (x * np.uint64(0x7FEB352D)) & m
    x ^= x >> np.uint64(15)
    x = (x * np.uint64(0x2C1B3C6D)) & m
    x ^= x >> np.uint64(16)
    x = (x * np.uint64(0x297A2D39)) & m
    x ^= x >> np.uint64(15)
    return x


def test_hash_matches_numpy_uint64():
    idx = np.array([0, 1, 2, 12345, 2**31 - 1, 2**32 - 1, 2**32, 2**33 + 17, 1_664_000_000])
    seed, stream = 424242, 2
    k = (seed * 0x9E37 + stream * 0x85EB + 0x1234567) & 0xFFFFFFFF
    k = _np_mix32(_np_mix32(np.array([k])))[0]
    lo = idx.astype(np.uint64) & np.uint64(0xFFFFFFFF)
    hi = (idx.astype(np.uint64) >> np.uint64(32)) & np.uint64(0xFFFFFFFF)
    want = _np_mix32(_np_mix32(lo ^ k) ^ hi)
    got = G.hash_u32(seed, stream, torch.tensor(idx, dtype=torch.int64)).numpy().astype(np.uint64)
    np.testing.assert_array_equal(got, want)


def test_distributions():
    idx = torch.arange(200000, dtype=torch.int64)
    u = G.uniform(7, idx, 0.5)
    assert float(u.abs().max()) < 0.5 and abs(float(u.mean())) < 0.01
    n = G.normal(7, idx, 1.0)
    assert abs(float(n.mean())) < 0.02 and abs(float(n.std()) - 1.0) < 0.02
    r = G.randint(7, idx, 1000)
    assert int(r.min()) >= 0 and int(r.max()) < 1000


def test_rows_equal_full():
    spec = W.TensorSpec("bf16", (3, 50, 8), ("normal", 1.0), 99)
    full = spec.materialize()
    f = torch.tensor([[0, 2], [1, 1]])
    r = torch.tensor([[5, 49], [0, 7]])
    rows = spec.rows(f, r)
    assert torch.equal(rows, full[f, r])


def test_workloads_parse_and_sizes():
    from oracle.ir import parse
    for name in W.CONFIGS:
        for small in (True, False):
            wl = W.build(name, small=small)
            g = parse(wl.ir)
            assert set(g.params) == set(wl.params)
            for nm, spec in wl.params.items():
                assert g.params[nm] == (spec.dtype, spec.shape)
