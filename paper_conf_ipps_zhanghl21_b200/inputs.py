"""Seeded, counter-based synthetic input generator (shared by the CUDA path and the oracle tests).

This module holds NO arithmetic of the DUET method: it only turns
(seed, element index) into deterministic numbers so that the GPU can materialise a multi-GB
embedding table on the device while the CPU oracle regenerates exactly the rows it needs.

Why counter-based: SURVEY.md §8(d) fixes seeded synthetic inputs, and the c2 tables are
26 x 10^6 x 64 bf16 = 3.3 GB.  Every value is a pure function g(seed, i) built from 32-bit
integer mixing done in int64 torch arithmetic that never overflows (operands < 2^32, multipliers
< 2^31), followed by exactly-representable integer->float steps and ONE correctly-rounded IEEE
operation.  The result is therefore bit-identical on CPU and CUDA (checked by
tests/test_inputs.py and tests/test_gpu_parity.py).

Distributions:
  * uniform(a):   x = a * v,  v = (2u+1-2^24) / 2^24 with u a 23-bit-safe 24-bit hash field
  * normal(std):  Irwin-Hall of four 16-bit fields, x = std * s / 75674.3 (s an exact integer)
  * randint(n):   31-bit hash field mod n (int64)
"""
from __future__ import annotations

import torch

M32 = 0xFFFFFFFF
_C1 = 0x7FEB352D
_C2 = 0x2C1B3C6D
_C3 = 0x297A2D39
_IH_STD = 75674.3  # std of sum of four (2*h16+1-65536) terms: 2*65536/sqrt(3)


def _mix32(x: torch.Tensor) -> torch.Tensor:
    """32-bit avalanche hash on int64 tensors holding values in [0, 2^32)."""
    x = x ^ (x >> 16)
    x = (x * _C1) & M32
    x = x ^ (x >> 15)
    x = (x * _C2) & M32
    x = x ^ (x >> 16)
    x = (x * _C3) & M32
    x = x ^ (x >> 15)
    return x


def _key(seed: int, stream: int) -> int:
    t = torch.tensor([(seed * 0x9E37 + stream * 0x85EB + 0x1234567) & M32], dtype=torch.int64)
    return int(_mix32(_mix32(t))[0])


def hash_u32(seed: int, stream: int, idx: torch.Tensor) -> torch.Tensor:
    """g(seed, stream, i) in [0, 2^32) as int64, elementwise over an int64 index tensor."""
    k = _key(seed, stream)
    lo = idx & M32
    hi = (idx >> 32) & M32
    return _mix32(_mix32(lo ^ k) ^ hi)


def uniform(seed: int, idx: torch.Tensor, scale: float) -> torch.Tensor:
    """float64 values in (-scale, scale)."""
    u = hash_u32(seed, 0, idx) >> 8  # 24 bits
    v = (2 * u + 1 - (1 << 24)).to(torch.float64) * (2.0 ** -24)  # exact, in (-1, 1)
    return v * scale  # one IEEE rounding


def normal(seed: int, idx: torch.Tensor, std: float, mean: float = 0.0) -> torch.Tensor:
    """Approximately N(mean, std^2) float64 (Irwin-Hall, 4 terms)."""
    a = hash_u32(seed, 1, idx)
    b = hash_u32(seed, 2, idx)
    s = ((2 * (a & 0xFFFF) + 1) + (2 * (a >> 16) + 1) + (2 * (b & 0xFFFF) + 1)
         + (2 * (b >> 16) + 1) - 4 * 65536)
    x = s.to(torch.float64) / _IH_STD  # one IEEE rounding
    if std != 1.0:
        x = x * std
    if mean != 0.0:
        x = x + mean
    return x


def randint(seed: int, idx: torch.Tensor, high: int, low: int = 0) -> torch.Tensor:
    """int64 values in [low, high)."""
    h = hash_u32(seed, 3, idx) & 0x7FFFFFFF
    return low + (h % (high - low))


# ------------------------------------------------------------------------------------------
# Tensor-level materialisation from a spec
# ------------------------------------------------------------------------------------------
TORCH_DTYPE = {"f32": torch.float32, "bf16": torch.bfloat16, "i32": torch.int32, "i64": torch.int64}


def _numel(shape) -> int:
    n = 1
    for s in shape:
        n *= int(s)
    return n


def gen_values(init: tuple, seed: int, idx: torch.Tensor) -> torch.Tensor:
    """Values (float64 or int64) of elements `idx` of a tensor with the given init spec."""
    kind = init[0]
    if kind == "uniform":
        return uniform(seed, idx, float(init[1]))
    if kind == "normal":
        mean = float(init[2]) if len(init) > 2 else 0.0
        return normal(seed, idx, float(init[1]), mean)
    if kind == "uniform_range":  # (lo, hi): lo + (hi-lo) * (v+1)/2
        lo, hi = float(init[1]), float(init[2])
        v = uniform(seed, idx, 1.0)
        return lo + (hi - lo) * ((v + 1.0) * 0.5)
    if kind == "randint":
        low = int(init[2]) if len(init) > 2 else 0
        return randint(seed, idx, int(init[1]), low)
    if kind == "const":
        return torch.full(idx.shape, float(init[1]), dtype=torch.float64, device=idx.device)
    if kind == "arange_mod":  # deterministic small-integer pattern used by golden fixtures
        return (idx % int(init[1])).to(torch.float64)
    if kind == "explicit":  # small literal tensors (golden fixtures)
        vals = torch.tensor(init[1], dtype=torch.float64, device=idx.device).reshape(-1)
        return vals[idx]
    raise ValueError(f"unknown init kind {kind!r}")


def cast(values: torch.Tensor, dtype: str) -> torch.Tensor:
    """Round generated float64/int64 values to the stored dtype (f64->f32->bf16, RNE each)."""
    if dtype == "f32":
        return values.to(torch.float32)
    if dtype == "bf16":
        return values.to(torch.float32).to(torch.bfloat16)
    if dtype == "i32":
        return values.to(torch.int32)
    if dtype == "i64":
        return values.to(torch.int64)
    raise ValueError(dtype)


def materialize(dtype: str, shape, init: tuple, seed: int, device="cpu",
                chunk: int = 1 << 26) -> torch.Tensor:
    """Full tensor of `shape`, generated in chunks on `device` (cpu or cuda)."""
    n = _numel(shape)
    out = torch.empty(n, dtype=TORCH_DTYPE[dtype], device=device)
    for s in range(0, n, chunk):
        e = min(n, s + chunk)
        idx = torch.arange(s, e, dtype=torch.int64, device=device)
        out[s:e] = cast(gen_values(init, seed, idx), dtype)
    return out.reshape(tuple(int(x) for x in shape))


def materialize_rows(dtype: str, shape, init: tuple, seed: int, lead_index: tuple) -> torch.Tensor:
    """Rows of a tensor selected by indices on the leading dims, without materialising it.

    `lead_index` is a tuple of equally-shaped int64 tensors indexing the first len(lead_index)
    dims; the result has shape lead_shape + shape[len(lead_index):].  Used by the oracle tests to
    read table rows of multi-GB embedding tables.
    """
    shape = tuple(int(x) for x in shape)
    k = len(lead_index)
    inner = _numel(shape[k:])
    flat = torch.zeros_like(lead_index[0], dtype=torch.int64)
    for d in range(k):
        flat = flat * shape[d] + lead_index[d].to(torch.int64)
    base = flat.reshape(-1, 1) * inner + torch.arange(inner, dtype=torch.int64).reshape(1, -1)
    vals = cast(gen_values(init, seed, base.reshape(-1)), dtype)
    return vals.reshape(tuple(lead_index[0].shape) + shape[k:])
