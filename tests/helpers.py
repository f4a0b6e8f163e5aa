"""Test glue between the CUDA path (through the C ABI) and the oracle: tensor -> NumPy in the
oracle's stored-value convention, and the relative error of SURVEY.md §8(c) C-A #25."""
import numpy as np
import torch

TOL = {"f32": 1e-5, "bf16": 2e-2}


def to_np(t: torch.Tensor) -> np.ndarray:
    t = t.detach().cpu()
    if t.dtype == torch.bfloat16:
        return t.view(torch.int16).numpy().view(np.uint16)
    return t.numpy()


def oracle_arrays(tensors: dict) -> dict:
    return {k: to_np(v) for k, v in tensors.items()}


def rel_err(y, yhat) -> float:
    """max_i |y_i - yhat_i| / max(max_i |yhat_i|, 1e-30)  (yhat = oracle)."""
    y = np.asarray(y, dtype=np.float64)
    yhat = np.asarray(yhat, dtype=np.float64)
    return float(np.max(np.abs(y - yhat)) / max(float(np.max(np.abs(yhat))), 1e-30))


def lazy_rows(spec):
    """Oracle parameter for a big table: callable returning stored values of selected rows."""
    def rows(*lead):
        idx = tuple(torch.as_tensor(np.ascontiguousarray(a), dtype=torch.int64) for a in lead)
        return to_np(spec.rows(*idx))
    return rows
