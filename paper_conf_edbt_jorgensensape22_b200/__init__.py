"""Python binding of the B200-native GPU-FAST-PROCLUS hot path.

Argument marshalling only: every step of PROCLUS (Alg 1-6) runs in
the sm_100a kernels of ``libproclus.so`` behind the C ABI of
``include/proclus.h``.  The functions below carry the C names; ``Proclus``
is a thin convenience wrapper over a handle.  There is no CPU fallback: if
the shared library is missing or cannot be loaded, importing the binding
raises.  Torch is optional and only used for device buffers and streams
(``torch.Tensor`` inputs are passed by data pointer).
"""
from __future__ import annotations

import ctypes as C
import os
from dataclasses import dataclass

import numpy as np

from . import _build

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = _build.LIB

OK, EINVAL, ENOMEM, ECUDA, ENCCL, EINTERNAL = 0, -1, -2, -3, -4, -5
METRIC_L2, METRIC_L1 = 0, 1
# proclus_variant: GPU-FAST-PROCLUS, GPU-PROCLUS (no caches), GPU-FAST*-PROCLUS
VARIANT_FAST, VARIANT_PLAIN, VARIANT_FAST_STAR = 0, 1, 2
K_MAX = 32
D_MAX = 256


class ProclusError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"proclus status {status}: {msg}")
        self.status = status


class proclus_options(C.Structure):
    _fields_ = [("device", C.c_int32), ("metric", C.c_int32), ("max_iter", C.c_int32),
                ("data_on_device", C.c_int32), ("stream", C.c_void_p), ("trace", C.c_int32),
                ("world_size", C.c_int32), ("rank", C.c_int32), ("n_global", C.c_int64),
                ("row_offset", C.c_int64), ("nccl_unique_id", C.c_void_p),
                ("stats", C.c_int32), ("variant", C.c_int32), ("group", C.c_void_p)]


STAT_KINDS = ["pack", "gather", "greedy", "prepare", "locality", "assign", "cost",
              "refine_x", "final", "split_tail"]


class proclus_stats(C.Structure):
    _fields_ = [("launches", C.c_int64 * 10), ("ms", C.c_double * 10),
                ("alg_bytes", C.c_double * 10), ("run_ms", C.c_double),
                ("total_launches", C.c_int64), ("tail_ms", C.c_double * 4),
                ("fallbacks", C.c_int64 * 4)]


class proclus_result(C.Structure):
    _fields_ = [("labels", C.c_void_p), ("medoids", C.c_void_p), ("dims", C.c_void_p),
                ("cost", C.c_double), ("iterations", C.c_int32),
                ("labels_on_device", C.c_int32)]


class proclus_trace(C.Structure):
    _fields_ = [("cap", C.c_int32), ("count", C.c_int32), ("mcur", C.c_void_p),
                ("delta", C.c_void_p), ("nL", C.c_void_p), ("dims", C.c_void_p),
                ("sizes", C.c_void_p), ("cost", C.c_void_p), ("improved", C.c_void_p),
                ("bad", C.c_void_p), ("X", C.c_void_p)]


# every entry point of include/proclus.h: (name, restype, argtypes)
SIGNATURES = [
    ("proclus_options_init", C.c_int, [C.POINTER(proclus_options)]),
    ("proclus_group_create", C.c_int, [C.c_int32, C.POINTER(C.c_void_p)]),
    ("proclus_group_destroy", None, [C.c_void_p]),
    ("proclus_create", C.c_int, [C.c_void_p, C.c_int64, C.c_int32, C.POINTER(C.c_void_p)]),
    ("proclus_create_ex", C.c_int, [C.c_void_p, C.c_int64, C.c_int32,
                                    C.POINTER(proclus_options), C.POINTER(C.c_void_p)]),
    ("proclus_load", C.c_int, [C.c_void_p, C.c_void_p]),
    ("proclus_prefetch", C.c_int, [C.c_void_p, C.c_void_p]),
    ("proclus_run", C.c_int, [C.c_void_p, C.c_int32, C.c_int32, C.c_int32, C.c_int32,
                              C.c_double, C.c_int32, C.c_uint64, C.POINTER(proclus_result)]),
    ("proclus_run_multi", C.c_int, [C.c_void_p, C.c_void_p, C.c_int32, C.c_void_p, C.c_int32,
                                    C.c_int32, C.c_int32, C.c_double, C.c_int32, C.c_uint64,
                                    C.c_int32, C.POINTER(proclus_result)]),
    ("proclus_run_list", C.c_int, [C.c_void_p, C.c_void_p, C.c_void_p, C.c_int32, C.c_int32,
                                   C.c_int32, C.c_int32, C.c_double, C.c_int32, C.c_uint64,
                                   C.c_int32, C.POINTER(proclus_result)]),
    ("proclus_get_trace", C.c_int, [C.c_void_p, C.POINTER(proclus_trace)]),
    ("proclus_get_stats", C.c_int, [C.c_void_p, C.POINTER(proclus_stats)]),
    ("proclus_last_launches", C.c_int64, [C.c_void_p]),
    ("proclus_destroy", None, [C.c_void_p]),
    ("proclus_last_error", C.c_char_p, []),
    ("proclus_abi_version", C.c_int32, []),
    ("proclus_target_sm", C.c_int32, []),
]

_lib = None


def lib():
    """Load libproclus.so (building it first if the sources are newer)."""
    global _lib
    if _lib is None:
        if _build.needs_build():
            _build.build()
        L = C.CDLL(LIB_PATH)
        for name, res, args in SIGNATURES:
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def _check(status: int):
    if status != OK:
        raise ProclusError(status, lib().proclus_last_error().decode())


# ------------------------------------------------------------ C-named calls
def proclus_options_init() -> proclus_options:
    o = proclus_options()
    _check(lib().proclus_options_init(C.byref(o)))
    return o


def proclus_group_create(world: int) -> C.c_void_p:
    g = C.c_void_p()
    _check(lib().proclus_group_create(world, C.byref(g)))
    return g


def proclus_group_destroy(g):
    lib().proclus_group_destroy(g)


def _ptr(a) -> int:
    """Data pointer of a numpy array or torch tensor."""
    if hasattr(a, "data_ptr"):
        return a.data_ptr()
    return a.ctypes.data


def proclus_create_ex(data, n: int, d: int, opt: proclus_options) -> C.c_void_p:
    h = C.c_void_p()
    _check(lib().proclus_create_ex(C.c_void_p(_ptr(data)), n, d, C.byref(opt), C.byref(h)))
    return h


def proclus_create(data, n: int, d: int) -> C.c_void_p:
    h = C.c_void_p()
    _check(lib().proclus_create(C.c_void_p(_ptr(data)), n, d, C.byref(h)))
    return h


def proclus_load(h, data):
    _check(lib().proclus_load(h, C.c_void_p(_ptr(data))))


def proclus_prefetch(h, data):
    _check(lib().proclus_prefetch(h, C.c_void_p(_ptr(data))))


def proclus_run(h, k, l, A, B, minDev, itrPat, seed, res: proclus_result):
    _check(lib().proclus_run(h, k, l, A, B, minDev, itrPat, seed, C.byref(res)))


def proclus_run_multi(h, ks, ls, A, B, minDev, itrPat, seed, reuse_level, outs):
    ks = np.ascontiguousarray(ks, np.int32)
    ls = np.ascontiguousarray(ls, np.int32)
    _check(lib().proclus_run_multi(h, ks.ctypes.data, len(ks), ls.ctypes.data, len(ls),
                                   A, B, minDev, itrPat, seed, reuse_level, outs))


def proclus_run_list(h, ks, ls, k_sample, A, B, minDev, itrPat, seed, reuse_level, outs):
    ks = np.ascontiguousarray(ks, np.int32)
    ls = np.ascontiguousarray(ls, np.int32)
    if ks.shape != ls.shape:
        raise ValueError("ks and ls must have the same length")
    _check(lib().proclus_run_list(h, ks.ctypes.data, ls.ctypes.data, len(ks), k_sample, A, B,
                                  minDev, itrPat, seed, reuse_level, outs))


def proclus_get_trace(h, tr: proclus_trace):
    _check(lib().proclus_get_trace(h, C.byref(tr)))


def proclus_get_stats(h) -> proclus_stats:
    st = proclus_stats()
    _check(lib().proclus_get_stats(h, C.byref(st)))
    return st


def proclus_last_launches(h) -> int:
    return int(lib().proclus_last_launches(h))


def proclus_destroy(h):
    lib().proclus_destroy(h)


def proclus_last_error() -> str:
    return lib().proclus_last_error().decode()


def proclus_abi_version() -> int:
    return int(lib().proclus_abi_version())


def proclus_target_sm() -> int:
    return int(lib().proclus_target_sm())


# ------------------------------------------------------------ wrapper
@dataclass
class Result:
    labels: object          # np.ndarray int32 [n] (or the device tensor given)
    medoids: np.ndarray     # int64 [k]
    dims: np.ndarray        # bool [k, d]
    cost: float
    iterations: int


@dataclass
class Trace:
    mcur: np.ndarray
    delta: np.ndarray
    nL: np.ndarray
    dims: np.ndarray
    sizes: np.ndarray
    cost: np.ndarray
    improved: np.ndarray
    bad: np.ndarray
    X: np.ndarray


class Proclus:
    """A handle: device-resident data plus the FAST caches (Dist, H)."""

    def __init__(self, data, *, metric: int = METRIC_L2, device: int = -1,
                 max_iter: int = 0, trace: bool = False, stream: int | None = None,
                 stats: bool = False, variant: int = VARIANT_FAST,
                 world_size: int = 1, rank: int = 0, n_global: int = 0,
                 row_offset: int = 0, nccl_unique_id: bytes | None = None,
                 group=None):
        on_dev = hasattr(data, "is_cuda") and bool(data.is_cuda)
        if on_dev:
            if data.dtype.__str__() != "torch.float32" or not data.is_contiguous():
                raise ValueError("device data must be a contiguous float32 tensor")
            n, d = data.shape
            self._keep = data
        else:
            data = np.ascontiguousarray(data, dtype=np.float32)
            n, d = data.shape
        self.n, self.d = int(n), int(d)
        o = proclus_options_init()
        o.device = device
        o.metric = metric
        o.max_iter = max_iter
        o.data_on_device = int(on_dev)
        o.stream = stream
        o.trace = int(trace)
        o.stats = int(stats)
        o.variant = int(variant)
        o.world_size = world_size
        o.rank = rank
        o.n_global = n_global
        o.row_offset = row_offset
        self._uid = None
        if nccl_unique_id is not None:
            self._uid = C.create_string_buffer(bytes(nccl_unique_id), 128)
            o.nccl_unique_id = C.cast(self._uid, C.c_void_p)
        if group is not None:
            o.group = group.value if isinstance(group, C.c_void_p) else group
        self.options = o
        self._on_dev = on_dev
        self.h = proclus_create_ex(data, self.n, self.d, o)
        self._k = None
        self._pf = None  # the array of a pending prefetch (kept alive)
        self._loaded = None  # the array of the last (asynchronous) load

    def close(self):
        if getattr(self, "h", None):
            proclus_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    def _device_index(self) -> int:
        return int(self.options.device) if self.options.device >= 0 else _current_device()

    def _checked_data(self, data, copy_ok: bool):
        """The C ABI reads n*d floats from the pointer (host or device per
        the handle): shape, dtype, contiguity and residency are checked here."""
        if self._on_dev:
            if not (hasattr(data, "is_cuda") and data.is_cuda):
                raise ValueError("this handle was created with device data: pass a CUDA tensor")
            if str(data.dtype) != "torch.float32" or not data.is_contiguous():
                raise ValueError("device data must be a contiguous float32 tensor")
            if data.device.index != self._device_index():
                raise ValueError(f"tensor on cuda:{data.device.index}, handle on "
                                 f"cuda:{self._device_index()}")
            if tuple(data.shape) != (self.n, self.d):
                raise ValueError(f"data shape {tuple(data.shape)} != ({self.n}, {self.d})")
            return data
        if hasattr(data, "is_cuda") and data.is_cuda:
            raise ValueError("this handle was created with host data: pass a host array")
        if hasattr(data, "numpy"):
            data = data.numpy()
        arr = np.asarray(data)
        if not copy_ok and (arr.dtype != np.float32 or not arr.flags.c_contiguous):
            raise ValueError("prefetch needs a C-contiguous float32 array (no copy is made)")
        arr = np.ascontiguousarray(arr, dtype=np.float32)
        if arr.shape != (self.n, self.d):
            raise ValueError(f"data shape {arr.shape} != ({self.n}, {self.d})")
        return arr

    def load(self, data):
        data = self._checked_data(data, copy_ok=True)
        proclus_load(self.h, data)
        self._pf = None  # the prefetched buffer is no longer referenced by the library
        self._loaded = data  # the asynchronous copy may still read it until the next run

    def prefetch(self, data):
        """Start the H2D copy of the next dataset (keep `data` unchanged until
        load(data) returns); load(data) then waits for it.  The handle keeps a
        reference to `data` until then."""
        if self._on_dev:
            raise ValueError("prefetch is for handles with host data")
        data = self._checked_data(data, copy_ok=False)
        proclus_prefetch(self.h, data)
        self._pf = data

    def _result_struct(self, k, labels=None):
        on_dev = labels is not None and hasattr(labels, "is_cuda") and bool(labels.is_cuda)
        if labels is not None:
            if on_dev:
                if str(labels.dtype) != "torch.int32" or not labels.is_contiguous():
                    raise ValueError("device labels must be a contiguous int32 tensor")
                if labels.device.index != self._device_index():
                    raise ValueError("labels tensor on another device than the handle")
                if labels.numel() < self.n:
                    raise ValueError(f"labels holds {labels.numel()} < n = {self.n} elements")
            else:
                if (not isinstance(labels, np.ndarray) or labels.dtype != np.int32
                        or not labels.flags.c_contiguous or labels.size < self.n):
                    raise ValueError("host labels must be a C-contiguous int32 ndarray of "
                                     f">= n = {self.n} elements")
        if labels is None:
            labels = np.empty(self.n, np.int32)
        med = np.empty(k, np.int64)
        dims = np.empty((k, self.d), np.uint8)
        r = proclus_result(_ptr(labels), med.ctypes.data, dims.ctypes.data, 0.0, 0, int(on_dev))
        return r, labels, med, dims

    def run(self, k: int, l: int, A: int = 100, B: int = 10, minDev: float = 0.7,
            itrPat: int = 5, seed: int = 1, labels=None) -> Result:
        r, lab, med, dims = self._result_struct(k, labels)
        proclus_run(self.h, k, l, A, B, minDev, itrPat, seed, r)
        self._loaded = None
        self._k = k
        return Result(lab, med, dims.astype(bool), float(r.cost), int(r.iterations))

    def run_multi(self, ks, ls, A=100, B=10, minDev=0.7, itrPat=5, seed=1,
                  reuse_level: int = 2) -> list[Result]:
        outs = (proclus_result * (len(ks) * len(ls)))()
        keep = []
        for a, k in enumerate(ks):
            for b, _ in enumerate(ls):
                r, lab, med, dims = self._result_struct(int(k))
                outs[a * len(ls) + b] = r
                keep.append((lab, med, dims))
        proclus_run_multi(self.h, ks, ls, A, B, minDev, itrPat, seed, reuse_level, outs)
        return [Result(lab, med, dims.astype(bool), float(outs[i].cost), int(outs[i].iterations))
                for i, (lab, med, dims) in enumerate(keep)]

    def run_list(self, settings, k_sample: int, A=100, B=10, minDev=0.7, itrPat=5, seed=1,
                 reuse_level: int = 2) -> list[Result]:
        """Independent settings [(k, l), ...] (settings parallelism): level 2
        draws S and M once for k_sample, so each result equals that
        setting of run_multi over a grid with largest k = k_sample."""
        settings = [(int(k), int(l)) for k, l in settings]
        outs = (proclus_result * len(settings))()
        keep = []
        for i, (k, _) in enumerate(settings):
            r, lab, med, dims = self._result_struct(k)
            outs[i] = r
            keep.append((lab, med, dims))
        proclus_run_list(self.h, [k for k, _ in settings], [l for _, l in settings], k_sample,
                         A, B, minDev, itrPat, seed, reuse_level, outs)
        return [Result(lab, med, dims.astype(bool), float(outs[i].cost), int(outs[i].iterations))
                for i, (lab, med, dims) in enumerate(keep)]

    def trace(self, cap: int = 4096) -> Trace:
        k, d = self._k, self.d
        arrs = dict(mcur=np.zeros((cap, k), np.int32), delta=np.zeros((cap, k)),
                    nL=np.zeros((cap, k), np.int64), dims=np.zeros((cap, k, d), np.uint8),
                    sizes=np.zeros((cap, k), np.int64), cost=np.zeros(cap),
                    improved=np.zeros(cap, np.uint8), bad=np.zeros((cap, k), np.uint8),
                    X=np.zeros((cap, k, d)))
        tr = proclus_trace(cap, 0, *[arrs[f].ctypes.data for f, _ in proclus_trace._fields_[2:]])
        proclus_get_trace(self.h, tr)
        c = tr.count
        t = Trace(**{f: arrs[f][:c].copy() for f in arrs})
        t.improved = t.improved.astype(bool)
        t.bad = t.bad.astype(bool)
        t.dims = t.dims.astype(bool)
        return t

    def stats(self) -> dict:
        st = proclus_get_stats(self.h)
        out = {name: dict(launches=int(st.launches[i]), ms=float(st.ms[i]),
                          alg_bytes=float(st.alg_bytes[i]))
               for i, name in enumerate(STAT_KINDS)}
        out["run_ms"] = float(st.run_ms)
        out["total_launches"] = int(st.total_launches)
        out["tail_ms"] = dict(zip(["locality", "assign", "cost", "refine_x"],
                                  [float(v) for v in st.tail_ms]))
        out["fallbacks"] = dict(zip(["locality", "assign", "final", "-"],
                                    [int(v) for v in st.fallbacks]))
        return out

    @property
    def last_launches(self) -> int:
        return proclus_last_launches(self.h)


def _current_device() -> int:
    import torch

    return int(torch.cuda.current_device())


def proclus(data, k: int, l: int, A: int = 100, B: int = 10, minDev: float = 0.7,
            itrPat: int = 5, seed: int = 1, metric: int = METRIC_L2, **kw) -> Result:
    """One-shot convenience: create a handle, run PROCLUS once, destroy it."""
    with Proclus(data, metric=metric, **kw) as p:
        return p.run(k, l, A, B, minDev, itrPat, seed)
