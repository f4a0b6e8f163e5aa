"""Thin ctypes binding of libduet.so (include/duet.h).  Argument marshalling only: every step of
the hot path runs inside the library's sm_100a kernels; PyTorch supplies device memory and
streams.  There is no CPU fallback: if libduet.so is missing this module raises on import.

    g = Graph(ir_text); g.bind_all({name: cuda_tensor, ...})
    p = g.partition("coarse")
    pr = p.profile(slots)                          # PAPER.md:80 (or p.profile_from_table(...))
    s = pr.schedule(mode=GREEDY_CORRECTION)        # PAPER.md:81, Algorithm 1
    s.run(slots, inputs, outputs)
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("DUET_LIB", os.path.join(_HERE, "libduet.so"))
if not os.path.exists(LIB_PATH):
    raise ImportError(f"libduet.so not built ({LIB_PATH}); run `python -m paper_conf_ipps_zhanghl21_b200.build`")
_lib = C.CDLL(LIB_PATH)

MAX_DIMS = 8
HOST = -1
F32, BF16, I32, I64 = 0, 1, 2, 3
GREEDY_CORRECTION, GREEDY_ONLY, SERIAL, FIXED, RANDOM, ROUND_ROBIN, RANDOM_CORRECTION = 0, 1, 2, 3, 4, 5, 6
STATUS = {0: "OK", -1: "EINVAL", -2: "EPARSE", -3: "ECYCLE", -4: "ESHAPE", -5: "EDTYPE", -6: "EUNBOUND",
          -7: "ECUDA", -8: "ENCCL", -9: "ENOMEM", -10: "EUNSUPPORTED", -11: "ESTATE"}


class DuetError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"{STATUS.get(code, code)}: {msg}")
        self.code = code
        self.name = STATUS.get(code, str(code))


class Tensor(C.Structure):
    _fields_ = [("data", C.c_void_p), ("device", C.c_int), ("dtype", C.c_int), ("ndim", C.c_int),
                ("shape", C.c_int64 * MAX_DIMS)]


class Slot(C.Structure):
    _fields_ = [("gpu", C.c_int), ("stream", C.c_void_p)]


class Link(C.Structure):
    _fields_ = [("alpha_ns", C.c_int64), ("ps_per_byte", C.c_int64)]


class CommModel(C.Structure):
    _fields_ = [("same_gpu", Link), ("cross_gpu", Link)]


class PartitionOpts(C.Structure):
    _fields_ = [("granularity", C.c_int), ("batch_shards", C.c_int)]


class ProfileOpts(C.Structure):
    _fields_ = [("warmup", C.c_int), ("samples", C.c_int), ("reps_per_sample", C.c_int),
                ("calibrate_comm", C.c_int)]


class MeasureOpts(C.Structure):
    _fields_ = [("samples", C.c_int), ("warmup", C.c_int), ("measured_ns", C.c_int64), ("evaluations", C.c_int32)]


class SchedOpts(C.Structure):
    _fields_ = [("mode", C.c_int), ("correction_rounds", C.c_int), ("allow_fallback", C.c_int),
                ("fixed_slot_of", C.POINTER(C.c_int32)), ("seed", C.c_uint32)]


_P = C.c_void_p
_sig = {
    "duet_last_error": (C.c_char_p, []),
    "duet_abi_version": (C.c_int, []),
    "duet_graph_load": (C.c_int, [C.c_char_p, C.c_size_t, C.POINTER(_P)]),
    "duet_graph_bind": (C.c_int, [_P, C.c_char_p, C.POINTER(Tensor)]),
    "duet_graph_info": (C.c_int, [_P] + [C.POINTER(C.c_int32)] * 4),
    "duet_graph_destroy": (None, [_P]),
    "duet_partition": (C.c_int, [_P, C.POINTER(PartitionOpts), C.POINTER(_P)]),
    "duet_partition_export": (C.c_int, [_P, C.POINTER(C.c_int32), C.POINTER(C.c_int32), C.POINTER(C.c_uint8),
                                        C.POINTER(C.c_int32), C.POINTER(C.c_int32), C.POINTER(C.c_int64),
                                        C.POINTER(C.c_int32), C.POINTER(C.c_int32), C.POINTER(C.c_int32)]),
    "duet_partition_destroy": (None, [_P]),
    "duet_partition_shards": (C.c_int, [_P, C.POINTER(C.c_int32), C.POINTER(C.c_int32), C.POINTER(C.c_int32)]),
    "duet_profile": (C.c_int, [_P, C.POINTER(Slot), C.c_int, C.POINTER(ProfileOpts), C.POINTER(_P)]),
    "duet_profile_from_table": (C.c_int, [_P, C.c_int, C.POINTER(C.c_int32), C.POINTER(C.c_int64),
                                          C.POINTER(CommModel), C.POINTER(_P)]),
    "duet_profile_export": (C.c_int, [_P, C.POINTER(C.c_int64), C.POINTER(C.c_int32), C.POINTER(CommModel),
                                      C.POINTER(C.c_int32)]),
    "duet_profile_destroy": (None, [_P]),
    "duet_schedule": (C.c_int, [_P, _P, C.POINTER(SchedOpts), C.POINTER(_P)]),
    "duet_schedule_measured": (C.c_int, [_P, _P, C.POINTER(SchedOpts), C.POINTER(Slot), C.c_int,
                                         C.POINTER(MeasureOpts), C.POINTER(_P)]),
    "duet_schedule_export": (C.c_int, [_P, C.POINTER(C.c_int32), C.POINTER(C.c_int32), C.POINTER(C.c_int64),
                                       C.POINTER(C.c_int32)]),
    "duet_schedule_destroy": (None, [_P]),
    "duet_run": (C.c_int, [_P, C.POINTER(Slot), C.c_int, C.POINTER(Tensor), C.c_int, C.POINTER(Tensor), C.c_int]),
    "duet_schedule_launch_count": (C.c_int, [_P, C.POINTER(C.c_int64)]),
    "duet_schedule_set_trace": (C.c_int, [_P, C.c_int]),
    "duet_schedule_trace": (C.c_int, [_P, C.POINTER(C.c_int64), C.POINTER(C.c_int64), C.c_int32]),
    "duet_node_run": (C.c_int, [_P, C.c_char_p, C.POINTER(Tensor), C.c_int, C.POINTER(Tensor), _P]),
}
for _name, (_res, _args) in _sig.items():
    _f = getattr(_lib, _name)
    _f.restype = _res
    _f.argtypes = _args

EXPORTED = sorted(_sig)


def _check(code: int):
    if code != 0:
        raise DuetError(code, _lib.duet_last_error().decode(errors="replace"))


def abi_version() -> int:
    return _lib.duet_abi_version()


def _np_ptr(a: np.ndarray, ct):
    return a.ctypes.data_as(C.POINTER(ct))


# ---- tensors ------------------------------------------------------------------------------------
def _torch_dtype_code(t) -> int:
    import torch
    m = {torch.float32: F32, torch.bfloat16: BF16, torch.int32: I32, torch.int64: I64}
    if t.dtype not in m:
        raise TypeError(f"unsupported dtype {t.dtype}")
    return m[t.dtype]


def as_tensor(t) -> Tensor:
    """duet_tensor view of a contiguous torch tensor (CUDA -> device ordinal, CPU -> DUET_HOST)."""
    if not t.is_contiguous():
        raise ValueError("tensors passed to libduet must be contiguous")
    if t.dim() > MAX_DIMS:
        raise ValueError("too many dims")
    d = Tensor()
    d.data = t.data_ptr()
    d.device = t.device.index if t.is_cuda else HOST
    d.dtype = _torch_dtype_code(t)
    d.ndim = t.dim()
    for i, s in enumerate(t.shape):
        d.shape[i] = int(s)
    return d


def _tensor_array(ts):
    arr = (Tensor * max(1, len(ts)))()
    for i, t in enumerate(ts):
        arr[i] = as_tensor(t)
    return arr


def make_slots(slots) -> "C.Array":
    """slots: list of (gpu, torch.cuda.Stream) or Slot."""
    arr = (Slot * len(slots))()
    for i, s in enumerate(slots):
        if isinstance(s, Slot):
            arr[i] = s
        else:
            gpu, stream = s
            arr[i].gpu = int(gpu)
            arr[i].stream = stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream)
    return arr


# ---- handles ------------------------------------------------------------------------------------
class Graph:
    def __init__(self, ir: str):
        h = _P()
        b = ir.encode()
        _check(_lib.duet_graph_load(b, len(b), C.byref(h)))
        self._h = h
        self._keep = {}

    def __del__(self):
        if getattr(self, "_h", None) and _lib is not None:  # (module globals vanish at interpreter exit)
            _lib.duet_graph_destroy(self._h)
            self._h = None

    def bind(self, name: str, t):
        _check(_lib.duet_graph_bind(self._h, name.encode(), C.byref(as_tensor(t))))
        self._keep[name] = t  # caller-owned memory must outlive the graph

    def bind_all(self, params: dict):
        for k, v in params.items():
            self.bind(k, v)

    def info(self):
        v = [C.c_int32() for _ in range(4)]
        _check(_lib.duet_graph_info(self._h, *[C.byref(x) for x in v]))
        return dict(zip(("n_nodes", "n_inputs", "n_outputs", "n_params"), (x.value for x in v)))

    def partition(self, granularity="coarse", batch_shards=1) -> "Partition":
        o = PartitionOpts({"coarse": 0, "op": 1}.get(granularity, granularity), batch_shards)
        h = _P()
        _check(_lib.duet_partition(self._h, C.byref(o), C.byref(h)))
        return Partition(h, self)

    def node_run(self, name: str, args, out, stream=None):
        arr = _tensor_array(args)
        o = as_tensor(out)
        st = stream.cuda_stream if stream is not None else 0
        _check(_lib.duet_node_run(self._h, name.encode(), arr, len(args), C.byref(o), st))


class Partition:
    def __init__(self, h, graph):
        self._h, self.graph = h, graph

    def __del__(self):
        if getattr(self, "_h", None) and _lib is not None:  # (module globals vanish at interpreter exit)
            _lib.duet_partition_destroy(self._h)
            self._h = None

    def export(self) -> dict:
        n_sg, n_ph, n_e = C.c_int32(), C.c_int32(), C.c_int32()
        _check(_lib.duet_partition_export(self._h, None, None, None, None, None, None, C.byref(n_sg),
                                          C.byref(n_ph), C.byref(n_e)))
        n_nodes = self.graph.info()["n_nodes"]
        node_to_sg = np.zeros(max(1, n_nodes), np.int32)
        sg_phase = np.zeros(max(1, n_sg.value), np.int32)
        kind = np.zeros(max(1, n_ph.value), np.uint8)
        es, ed = np.zeros(max(1, n_e.value), np.int32), np.zeros(max(1, n_e.value), np.int32)
        eb = np.zeros(max(1, n_e.value), np.int64)
        _check(_lib.duet_partition_export(self._h, _np_ptr(node_to_sg, C.c_int32), _np_ptr(sg_phase, C.c_int32),
                                          _np_ptr(kind, C.c_uint8), _np_ptr(es, C.c_int32), _np_ptr(ed, C.c_int32),
                                          _np_ptr(eb, C.c_int64), None, None, None))
        return {
            "n_sg": n_sg.value,
            "node_to_sg": node_to_sg[:n_nodes].tolist(),
            "sg_phase": sg_phase[:n_sg.value].tolist(),
            "phase_kind": kind[:n_ph.value].tolist(),
            "edges": {(int(a), int(b)): int(c) for a, b, c in zip(es[:n_e.value], ed[:n_e.value], eb[:n_e.value])},
        }

    def shards(self) -> dict:
        """Row shards of a batch_shards > 1 partition (duet_partition_shards)."""
        n = C.c_int32()
        _check(_lib.duet_partition_shards(self._h, None, None, C.byref(n)))
        sh, org = np.zeros(max(1, n.value), np.int32), np.zeros(max(1, n.value), np.int32)
        _check(_lib.duet_partition_shards(self._h, _np_ptr(sh, C.c_int32), _np_ptr(org, C.c_int32), None))
        return {"sg_shard": sh[:n.value].tolist(), "sg_origin": org[:n.value].tolist()}

    @property
    def n_sg(self) -> int:
        n = C.c_int32()
        _check(_lib.duet_partition_export(self._h, None, None, None, None, None, None, C.byref(n), None, None))
        return n.value

    def profile_from_table(self, slot_gpu, t_ns, comm=((0, 0), (0, 0))) -> "Profile":
        sg = np.ascontiguousarray(slot_gpu, dtype=np.int32)
        t = np.ascontiguousarray(t_ns, dtype=np.int64).reshape(-1)
        if t.size != self.n_sg * sg.size:
            raise ValueError("t_ns must be [n_sg, n_slots]")
        cm = CommModel(Link(*comm[0]), Link(*comm[1]))
        h = _P()
        _check(_lib.duet_profile_from_table(self._h, int(sg.size), _np_ptr(sg, C.c_int32), _np_ptr(t, C.c_int64),
                                            C.byref(cm), C.byref(h)))
        return Profile(h, self)

    def profile(self, slots, warmup=20, samples=500, reps=20, calibrate_comm=False) -> "Profile":
        arr = make_slots(slots)
        o = ProfileOpts(warmup, samples, reps, int(calibrate_comm))
        h = _P()
        _check(_lib.duet_profile(self._h, arr, len(slots), C.byref(o), C.byref(h)))
        return Profile(h, self)


class Profile:
    def __init__(self, h, part):
        self._h, self.part = h, part

    def __del__(self):
        if getattr(self, "_h", None) and _lib is not None:  # (module globals vanish at interpreter exit)
            _lib.duet_profile_destroy(self._h)
            self._h = None

    def export(self) -> dict:
        n = C.c_int32()
        _check(_lib.duet_profile_export(self._h, None, None, None, C.byref(n)))
        t = np.zeros(self.part.n_sg * n.value, np.int64)
        sg = np.zeros(n.value, np.int32)
        cm = CommModel()
        _check(_lib.duet_profile_export(self._h, _np_ptr(t, C.c_int64), _np_ptr(sg, C.c_int32), C.byref(cm), None))
        return {"t_ns": t.reshape(self.part.n_sg, n.value), "slot_gpu": sg.tolist(),
                "comm": ((cm.same_gpu.alpha_ns, cm.same_gpu.ps_per_byte),
                         (cm.cross_gpu.alpha_ns, cm.cross_gpu.ps_per_byte))}

    def schedule(self, mode=GREEDY_CORRECTION, correction_rounds=1, allow_fallback=True, fixed=None,
                 seed=0) -> "Schedule":
        fx = None
        if fixed is not None:
            fx = np.ascontiguousarray(fixed, dtype=np.int32)
        o = SchedOpts(mode, correction_rounds, int(allow_fallback), _np_ptr(fx, C.c_int32) if fx is not None else None,
                      seed)
        h = _P()
        _check(_lib.duet_schedule(self.part._h, self._h, C.byref(o), C.byref(h)))
        return Schedule(h, self)

    def schedule_measured(self, slots, mode=GREEDY_CORRECTION, correction_rounds=1, allow_fallback=True,
                          seed=0, samples=20, warmup=3) -> "Schedule":
        """Measured-mode Step 3 (duet_schedule_measured): candidates timed on the device over
        `slots`.  The returned Schedule carries .measured_ns and .evaluations."""
        o = SchedOpts(mode, correction_rounds, int(allow_fallback), None, seed)
        mo = MeasureOpts(samples, warmup, 0, 0)
        sa = make_slots(slots)
        h = _P()
        _check(_lib.duet_schedule_measured(self.part._h, self._h, C.byref(o), sa, len(slots), C.byref(mo),
                                           C.byref(h)))
        s = Schedule(h, self)
        s.measured_ns, s.evaluations = mo.measured_ns, mo.evaluations
        return s


class Schedule:
    def __init__(self, h, prof):
        self._h, self.prof = h, prof

    def __del__(self):
        if getattr(self, "_h", None) and _lib is not None:  # (module globals vanish at interpreter exit)
            _lib.duet_schedule_destroy(self._h)
            self._h = None

    def export(self) -> dict:
        n = self.prof.part.n_sg
        slot = np.zeros(max(1, n), np.int32)
        order = np.zeros(max(1, n), np.int32)
        ms, fb = C.c_int64(), C.c_int32()
        _check(_lib.duet_schedule_export(self._h, _np_ptr(slot, C.c_int32), _np_ptr(order, C.c_int32), C.byref(ms),
                                         C.byref(fb)))
        return {"slot_of": slot[:n].tolist(), "order": order[:n].tolist(), "makespan": ms.value,
                "fell_back": fb.value}

    def run(self, slots, inputs, outputs):
        sa = make_slots(slots)
        ia, oa = _tensor_array(inputs), _tensor_array(outputs)
        _check(_lib.duet_run(self._h, sa, len(slots), ia, len(inputs), oa, len(outputs)))

    def set_trace(self, on: bool = True) -> None:
        _check(_lib.duet_schedule_set_trace(self._h, int(on)))

    def trace(self) -> tuple:
        """(start_ns, end_ns) per subgraph of the last traced duet_run, relative to its fork."""
        n = self.prof.part.n_sg
        a, b = np.zeros(n, np.int64), np.zeros(n, np.int64)
        _check(_lib.duet_schedule_trace(self._h, _np_ptr(a, C.c_int64), _np_ptr(b, C.c_int64), n))
        return a, b

    def launch_count(self) -> int:
        n = C.c_int64()
        _check(_lib.duet_schedule_launch_count(self._h, C.byref(n)))
        return n.value
