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


def l2_rel_err(y, yhat) -> float:
    """||y - yhat||_2 / ||yhat||_2 (reported beside the max metric)."""
    y = np.asarray(y, dtype=np.float64)
    yhat = np.asarray(yhat, dtype=np.float64)
    return float(np.linalg.norm((y - yhat).ravel()) / max(float(np.linalg.norm(yhat.ravel())), 1e-30))


def elem_rel_err(y, yhat, floor: float = 1e-3) -> float:
    """Per-element relative error max_i |y_i - yhat_i| / |yhat_i| over the elements with
    |yhat_i| >= floor * max|yhat| (smaller ones are covered by the max metric): errors confined
    to small-magnitude elements, invisible to rel_err, show up here."""
    y = np.asarray(y, dtype=np.float64).ravel()
    yhat = np.asarray(yhat, dtype=np.float64).ravel()
    m = np.abs(yhat) >= floor * max(float(np.max(np.abs(yhat))), 1e-30)
    if not m.any():
        return 0.0
    return float(np.max(np.abs(y[m] - yhat[m]) / np.abs(yhat[m])))


def check(y, yhat, tol: float, what: str = "", elem_tol: float | None = None) -> float:
    """The parity bar: C-A #25's max metric and the L2-relative error both <= tol; the per-element
    relative error (magnitudes >= 1e-3 of the max) is printed and, when elem_tol is given, bounded.
    Returns the max metric."""
    e, l2, el = rel_err(y, yhat), l2_rel_err(y, yhat), elem_rel_err(y, yhat)
    print(f"[parity] {what}: rel err {e:.3e} (l2 {l2:.3e}, per-element {el:.3e}, tol {tol:g})")
    assert e <= tol and l2 <= tol, (what, e, l2, tol)
    if elem_tol is not None:
        assert el <= elem_tol, (what, el, elem_tol)
    return e


def lazy_rows(spec):
    """Oracle parameter for a big table: callable returning stored values of selected rows."""
    def rows(*lead):
        idx = tuple(torch.as_tensor(np.ascontiguousarray(a), dtype=torch.int64) for a in lead)
        return to_np(spec.rows(*idx))
    return rows
