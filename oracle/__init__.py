"""CPU oracle of PROCLUS -- TEST INFRASTRUCTURE ONLY.

Plain single-threaded fp64 C implementation (``proclus_oracle.c``) of the
method in /root/reference/PAPER.md (Alg 1-6, eqs 1-9), with a thin ctypes
wrapper.  Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``
(``cpu_baseline`` and ``--impl reference``) may import this package.  It
shares no code with the CUDA library in ``paper_conf_edbt_jorgensensape22_b200``.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
from dataclasses import dataclass, field

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "proclus_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

METRIC_L2 = 0
METRIC_L1 = 1


def build(force: bool = False) -> str:
    """Compile the oracle with -O2 -ffp-contract=off (no FMA, no fast-math)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < max(
        os.path.getmtime(_SRC), os.path.getmtime(os.path.join(_HERE, "proclus_oracle.h"))
    ):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(
            ["gcc", "-std=c11", "-O2", "-ffp-contract=off", "-fno-fast-math", "-fPIC",
             "-shared", "-Wall", "-Wno-unused-variable", "-o", tmp, _SRC, "-lm"]
        )
        os.replace(tmp, _LIB)
    return _LIB


class _Params(C.Structure):
    _fields_ = [("k", C.c_int32), ("l", C.c_int32), ("A", C.c_int32), ("B", C.c_int32),
                ("minDev", C.c_double), ("itrPat", C.c_int32), ("seed", C.c_uint64),
                ("metric", C.c_int32), ("max_iter", C.c_int32), ("fast", C.c_int32)]


class _Result(C.Structure):
    _fields_ = [("labels", C.POINTER(C.c_int32)), ("medoids", C.POINTER(C.c_int64)),
                ("dims", C.POINTER(C.c_uint8)), ("cost", C.c_double),
                ("iterations", C.c_int32), ("nS", C.c_int64), ("nM", C.c_int64)]


class _Trace(C.Structure):
    _fields_ = [("cap", C.c_int32), ("count", C.c_int32),
                ("mcur", C.POINTER(C.c_int32)), ("delta", C.POINTER(C.c_double)),
                ("nL", C.POINTER(C.c_int64)), ("dims", C.POINTER(C.c_uint8)),
                ("sizes", C.POINTER(C.c_int64)), ("cost", C.POINTER(C.c_double)),
                ("improved", C.POINTER(C.c_uint8)), ("bad", C.POINTER(C.c_uint8)),
                ("zgap", C.POINTER(C.c_double)), ("costgap", C.POINTER(C.c_double)),
                ("assign_gap", C.POINTER(C.c_double)), ("X", C.POINTER(C.c_double))]


_lib = None


def lib():
    global _lib
    if _lib is None:
        L = C.CDLL(build())
        P = C.POINTER
        L.oracle_splitmix_next.restype = C.c_uint64
        L.oracle_splitmix_next.argtypes = [P(C.c_uint64)]
        L.oracle_uniform.restype = C.c_uint64
        L.oracle_uniform.argtypes = [P(C.c_uint64), C.c_uint64]
        L.oracle_stream_sm.restype = C.c_uint64
        L.oracle_stream_sm.argtypes = [C.c_uint64, C.c_int64]
        L.oracle_stream_it.restype = C.c_uint64
        L.oracle_stream_it.argtypes = [C.c_uint64, C.c_int64, C.c_int64]
        L.oracle_full.restype = C.c_double
        L.oracle_full.argtypes = [C.c_void_p, C.c_void_p, C.c_int32, C.c_int32]
        L.oracle_seg.restype = C.c_double
        L.oracle_seg.argtypes = [C.c_void_p, C.c_void_p, C.c_int32, C.c_void_p]
        L.oracle_sample.argtypes = [C.c_int64, C.c_int64, P(C.c_uint64), C.c_void_p]
        L.oracle_greedy.argtypes = [C.c_void_p, C.c_int32, C.c_void_p, C.c_int64, C.c_int64,
                                    C.c_int64, C.c_int32, C.c_void_p, C.c_void_p]
        L.oracle_delta.argtypes = [C.c_void_p, C.c_int32, C.c_int32, C.c_int32, C.c_void_p]
        L.oracle_locality_X.argtypes = [C.c_void_p, C.c_int64, C.c_int32, C.c_void_p, C.c_int32,
                                        C.c_void_p, C.c_int32, C.c_void_p, C.c_void_p, C.c_void_p]
        L.oracle_find_dimensions.argtypes = [C.c_void_p, C.c_int32, C.c_int32, C.c_int32,
                                             C.c_void_p, C.c_void_p, C.c_void_p]
        L.oracle_assign.argtypes = [C.c_void_p, C.c_int64, C.c_int32, C.c_void_p, C.c_int32,
                                    C.c_void_p, C.c_void_p, C.c_void_p]
        L.oracle_evaluate.restype = C.c_double
        L.oracle_evaluate.argtypes = [C.c_void_p, C.c_int64, C.c_int32, C.c_void_p, C.c_int32,
                                      C.c_void_p, C.c_void_p]
        L.oracle_evaluate_eq9.restype = C.c_double
        L.oracle_evaluate_eq9.argtypes = [C.c_void_p, C.c_int64, C.c_int32, C.c_void_p,
                                          C.c_int32, C.c_void_p]
        L.oracle_bad_medoids.argtypes = [C.c_void_p, C.c_int32, C.c_int64, C.c_double, C.c_void_p]
        L.oracle_cluster_X.argtypes = [C.c_void_p, C.c_int64, C.c_int32, C.c_void_p, C.c_void_p,
                                       C.c_int32, C.c_void_p]
        L.oracle_remove_outliers.argtypes = [C.c_void_p, C.c_int64, C.c_int32, C.c_void_p,
                                             C.c_int32, C.c_void_p, C.c_void_p, C.c_void_p]
        L.oracle_validate.argtypes = [C.c_int64, C.c_int32, C.c_void_p, P(_Params)]
        L.oracle_proclus.argtypes = [C.c_void_p, C.c_int64, C.c_int32, P(_Params), P(_Result),
                                     P(_Trace)]
        L.oracle_proclus_multi.argtypes = [C.c_void_p, C.c_int64, C.c_int32, C.c_void_p,
                                           C.c_int32, C.c_void_p, C.c_int32, P(_Params),
                                           C.c_int32, P(_Result)]
        _lib = L
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data_as(C.c_void_p)


def _f32(data) -> np.ndarray:
    return np.ascontiguousarray(data, dtype=np.float32)


# ---------------------------------------------------------------- RNG
def splitmix_next(state: int) -> tuple[int, int]:
    s = C.c_uint64(state)
    v = lib().oracle_splitmix_next(C.byref(s))
    return int(v), int(s.value)


def uniform(state: int, m: int) -> tuple[int, int]:
    s = C.c_uint64(state)
    v = lib().oracle_uniform(C.byref(s), m)
    return int(v), int(s.value)


def stream_sm(seed: int, k_sm: int) -> int:
    return int(lib().oracle_stream_sm(seed, k_sm))


def stream_it(seed: int, k: int, l: int) -> int:
    return int(lib().oracle_stream_it(seed, k, l))


# ---------------------------------------------------------------- steps
def full(p, q, metric=METRIC_L2) -> float:
    p, q = _f32(p), _f32(q)
    return float(lib().oracle_full(_p(p), _p(q), p.shape[0], metric))


def seg(p, q, dmask) -> float:
    p, q = _f32(p), _f32(q)
    m = np.ascontiguousarray(dmask, dtype=np.uint8)
    return float(lib().oracle_seg(_p(p), _p(q), p.shape[0], _p(m)))


def sample(n: int, nS: int, state: int) -> tuple[np.ndarray, int]:
    S = np.empty(nS, np.int64)
    s = C.c_uint64(state)
    rc = lib().oracle_sample(n, nS, C.byref(s), _p(S))
    assert rc == 0
    return S, int(s.value)


def greedy(data, S, nM: int, q0: int, metric=METRIC_L2):
    data = _f32(data)
    S = np.ascontiguousarray(S, np.int64)
    pos = np.empty(nM, np.int64)
    pd = np.empty(nM, np.float64)
    rc = lib().oracle_greedy(_p(data), data.shape[1], _p(S), S.shape[0], nM, q0, metric,
                             _p(pos), _p(pd))
    assert rc == 0
    return pos, pd


def delta(med, metric=METRIC_L2) -> np.ndarray:
    med = _f32(med)
    out = np.empty(med.shape[0], np.float64)
    lib().oracle_delta(_p(med), med.shape[0], med.shape[1], metric, _p(out))
    return out


def locality_X(data, med, dlt, metric=METRIC_L2):
    data, med = _f32(data), _f32(med)
    n, d = data.shape
    k = med.shape[0]
    dlt = np.ascontiguousarray(dlt, np.float64)
    inL = np.empty((n, k), np.uint8)
    nL = np.empty(k, np.int64)
    X = np.empty((k, d), np.float64)
    lib().oracle_locality_X(_p(data), n, d, _p(med), k, _p(dlt), metric, _p(inL), _p(nL), _p(X))
    return inL.astype(bool), nL, X


def find_dimensions(X, l: int):
    X = np.ascontiguousarray(X, np.float64)
    k, d = X.shape
    m = np.empty((k, d), np.uint8)
    Z = np.empty((k, d), np.float64)
    g = C.c_double(0)
    rc = lib().oracle_find_dimensions(_p(X), k, d, l, _p(m), _p(Z), C.byref(g))
    assert rc == 0
    return m.astype(bool), Z, float(g.value)


def assign(data, med, dmask):
    data, med = _f32(data), _f32(med)
    n, d = data.shape
    k = med.shape[0]
    m = np.ascontiguousarray(dmask, np.uint8)
    lab = np.empty(n, np.int32)
    g = C.c_double(0)
    lib().oracle_assign(_p(data), n, d, _p(med), k, _p(m), _p(lab), C.byref(g))
    return lab, float(g.value)


def evaluate(data, labels, k: int, dmask):
    data = _f32(data)
    n, d = data.shape
    lab = np.ascontiguousarray(labels, np.int32)
    m = np.ascontiguousarray(dmask, np.uint8)
    sizes = np.empty(k, np.int64)
    c = lib().oracle_evaluate(_p(data), n, d, _p(lab), k, _p(m), _p(sizes))
    return float(c), sizes


def evaluate_eq9(data, labels, k: int, dmask) -> float:
    data = _f32(data)
    n, d = data.shape
    lab = np.ascontiguousarray(labels, np.int32)
    m = np.ascontiguousarray(dmask, np.uint8)
    return float(lib().oracle_evaluate_eq9(_p(data), n, d, _p(lab), k, _p(m)))


def bad_medoids(sizes, n: int, minDev: float) -> np.ndarray:
    s = np.ascontiguousarray(sizes, np.int64)
    bad = np.empty(s.shape[0], np.uint8)
    lib().oracle_bad_medoids(_p(s), s.shape[0], n, minDev, _p(bad))
    return bad.astype(bool)


def cluster_X(data, labels, med):
    data, med = _f32(data), _f32(med)
    n, d = data.shape
    k = med.shape[0]
    lab = np.ascontiguousarray(labels, np.int32)
    X = np.empty((k, d), np.float64)
    lib().oracle_cluster_X(_p(data), n, d, _p(lab), _p(med), k, _p(X))
    return X


def remove_outliers(data, med, dmask, labels):
    data, med = _f32(data), _f32(med)
    n, d = data.shape
    k = med.shape[0]
    lab = np.array(labels, dtype=np.int32, copy=True)
    m = np.ascontiguousarray(dmask, np.uint8)
    Dl = np.empty(k, np.float64)
    lib().oracle_remove_outliers(_p(data), n, d, _p(med), k, _p(m), _p(lab), _p(Dl))
    return lab, Dl


# ---------------------------------------------------------------- whole run
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
    zgap: np.ndarray
    costgap: np.ndarray
    assign_gap: np.ndarray
    X: np.ndarray


@dataclass
class Result:
    labels: np.ndarray
    medoids: np.ndarray
    dims: np.ndarray
    cost: float
    iterations: int
    nS: int
    nM: int
    trace: Trace | None = field(default=None, repr=False)


def validate(data, k, l, A=100, B=10, minDev=0.7, itrPat=5, metric=METRIC_L2) -> int:
    data = _f32(data)
    p = _Params(k, l, A, B, minDev, itrPat, 0, metric, 0, 0)
    return int(lib().oracle_validate(data.shape[0], data.shape[1], _p(data), C.byref(p)))


def _alloc_result(n, k, d):
    lab = np.empty(n, np.int32)
    med = np.empty(k, np.int64)
    dims = np.empty((k, d), np.uint8)
    r = _Result(lab.ctypes.data_as(C.POINTER(C.c_int32)), med.ctypes.data_as(C.POINTER(C.c_int64)),
                dims.ctypes.data_as(C.POINTER(C.c_uint8)), 0.0, 0, 0, 0)
    return r, lab, med, dims


def proclus(data, k: int, l: int, A: int = 100, B: int = 10, minDev: float = 0.7,
            itrPat: int = 5, seed: int = 1, metric: int = METRIC_L2, max_iter: int = 0,
            fast: bool = False, trace: bool = False, trace_cap: int = 10000) -> Result:
    """One PROCLUS run (Alg 1). Raises ValueError on EINVAL."""
    data = _f32(data)
    n, d = data.shape
    prm = _Params(k, l, A, B, minDev, itrPat, seed, metric, max_iter, int(fast))
    r, lab, med, dims = _alloc_result(n, k, d)
    tr_obj = None
    trp = None
    if trace:
        cap = trace_cap
        arrs = dict(mcur=np.zeros((cap, k), np.int32), delta=np.zeros((cap, k)),
                    nL=np.zeros((cap, k), np.int64), dims=np.zeros((cap, k, d), np.uint8),
                    sizes=np.zeros((cap, k), np.int64), cost=np.zeros(cap),
                    improved=np.zeros(cap, np.uint8), bad=np.zeros((cap, k), np.uint8),
                    zgap=np.zeros(cap), costgap=np.zeros(cap), assign_gap=np.zeros(cap),
                    X=np.zeros((cap, k, d)))
        ct = {np.int32: C.c_int32, np.int64: C.c_int64, np.uint8: C.c_uint8, np.float64: C.c_double}
        t = _Trace(cap, 0, *[arrs[name].ctypes.data_as(C.POINTER(ct[arrs[name].dtype.type]))
                             for name, _ in _Trace._fields_[2:]])
        trp = C.byref(t)
    rc = lib().oracle_proclus(_p(data), n, d, C.byref(prm), C.byref(r), trp)
    if rc == -1:
        raise ValueError("oracle: invalid arguments")
    if rc != 0:
        raise MemoryError("oracle: allocation failed")
    if trace:
        c = t.count
        tr_obj = Trace(**{name: arrs[name][:c].copy() for name in arrs})
        tr_obj.improved = tr_obj.improved.astype(bool)
        tr_obj.bad = tr_obj.bad.astype(bool)
        tr_obj.dims = tr_obj.dims.astype(bool)
    return Result(lab, med, dims.astype(bool), float(r.cost), int(r.iterations), int(r.nS),
                  int(r.nM), tr_obj)


def proclus_multi(data, ks, ls, A=100, B=10, minDev=0.7, itrPat=5, seed=1,
                  metric=METRIC_L2, reuse_level: int = 2, max_iter: int = 0) -> list[Result]:
    """Multi-parameter runs, k outer, l inner."""
    data = _f32(data)
    n, d = data.shape
    ks = np.ascontiguousarray(ks, np.int32)
    ls = np.ascontiguousarray(ls, np.int32)
    prm = _Params(0, 0, A, B, minDev, itrPat, seed, metric, max_iter, 0)
    outs = (_Result * (len(ks) * len(ls)))()
    keep = []
    for a, k in enumerate(ks):
        for b, _ in enumerate(ls):
            r, lab, med, dims = _alloc_result(n, int(k), d)
            outs[a * len(ls) + b] = r
            keep.append((lab, med, dims))
    rc = lib().oracle_proclus_multi(_p(data), n, d, _p(ks), len(ks), _p(ls), len(ls),
                                    C.byref(prm), reuse_level, outs)
    if rc == -1:
        raise ValueError("oracle: invalid arguments")
    if rc != 0:
        raise MemoryError("oracle: allocation failed")
    res = []
    for i, (lab, med, dims) in enumerate(keep):
        res.append(Result(lab, med, dims.astype(bool), float(outs[i].cost),
                          int(outs[i].iterations), int(outs[i].nS), int(outs[i].nM)))
    return res
