"""REFERENCE ORACLE for nu-LPA -- TEST INFRASTRUCTURE ONLY.

Thin ctypes wrapper around ``oracle/oracle.c`` (plain single-threaded C,
written from PAPER.md; see that file's header for citations and the
readings R1..R11 listed in DESIGN.md), plus NMI, an evaluation metric the
north star uses to compare community structure (not part of the method).

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its
``cpu_baseline`` leg and ``--impl reference``) may import this package.  The
product package ``paper_conf_ipps_sahunk25_b200`` never imports it and shares
no code with it.

Parity status: every function here is pinned by ``tests/test_oracle.py``
(closed forms, brute force on tiny graphs, published karate-club values,
invariants); none is "parity unpinned".
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

EMPTY = -1


def build(force: bool = False) -> str:
    """Compile oracle.c with gcc into oracle/liboracle.so (no CUDA involved)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def _L():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        i64, i32, u64, f64, f32, vp = (ctypes.c_int64, ctypes.c_int32, ctypes.c_uint64,
                                       ctypes.c_double, ctypes.c_float, ctypes.c_void_p)
        lib.oracle_next_pow2.argtypes = [u64]
        lib.oracle_next_pow2.restype = u64
        lib.oracle_hashtable_primes.argtypes = [u64, vp, vp]
        lib.oracle_hashtable_primes.restype = None
        lib.oracle_hashtable_clear.argtypes = [vp, vp, u64]
        lib.oracle_hashtable_clear.restype = None
        lib.oracle_hashtable_accumulate.argtypes = [vp, vp, u64, u64, i32, f32, ctypes.c_int, vp]
        lib.oracle_hashtable_accumulate.restype = ctypes.c_int
        lib.oracle_hashtable_max_key.argtypes = [vp, vp, u64, vp, vp]
        lib.oracle_hashtable_max_key.restype = i32
        lib.oracle_vertex_best.argtypes = [i64, vp, vp, vp, vp, vp, vp]
        lib.oracle_vertex_best.restype = i32
        lib.oracle_lpa_move_async.argtypes = [i64, vp, vp, vp, vp, vp, ctypes.c_int, vp, vp]
        lib.oracle_lpa_move_async.restype = i64
        lib.oracle_lpa_move_sync.argtypes = [i64, vp, vp, vp, vp, vp, vp, vp, ctypes.c_int, vp, vp, vp, vp]
        lib.oracle_lpa_move_sync.restype = i64
        lib.oracle_lpa.argtypes = [i64, vp, vp, vp, vp, f64, ctypes.c_int, ctypes.c_int, ctypes.c_int, vp]
        lib.oracle_lpa.restype = ctypes.c_int
        lib.oracle_modularity.argtypes = [i64, vp, vp, vp, vp]
        lib.oracle_modularity.restype = f64
        lib.oracle_set_tie_rule.argtypes = [ctypes.c_int]
        lib.oracle_set_tie_rule.restype = None
        _lib = lib
    return _lib


def _p(a):
    return None if a is None else a.ctypes.data


TIE_SMALLEST, TIE_SLOT = 0, 1


class _tie:
    """Select the tie order of hashtableMaxKey for one call (R6): 0 smallest
    label (north star), 1 smallest home slot k mod p1 then smallest label."""

    def __init__(self, rule):
        self.rule = int(rule)

    def __enter__(self):
        _L().oracle_set_tie_rule(self.rule)

    def __exit__(self, *exc):
        _L().oracle_set_tie_rule(0)


class CSR:
    """Host CSR graph as the oracle reads it: int64 offsets, int32 indices,
    float32 weights or None (unit weights)."""

    def __init__(self, offsets, indices, weights=None):
        self.offsets = np.ascontiguousarray(np.asarray(offsets), dtype=np.int64)
        self.indices = np.ascontiguousarray(np.asarray(indices), dtype=np.int32)
        self.weights = None if weights is None else np.ascontiguousarray(np.asarray(weights), dtype=np.float32)
        self.N = int(self.offsets.shape[0] - 1)
        self.M = int(self.offsets[-1])
        assert self.indices.shape[0] == self.M
        assert self.weights is None or self.weights.shape[0] == self.M

    @staticmethod
    def from_graph(g) -> "CSR":
        """Accept any object with offsets/indices/weights attributes (numpy or torch CPU)."""
        def np_(x):
            if x is None:
                return None
            return x.numpy() if hasattr(x, "numpy") else np.asarray(x)
        return CSR(np_(g.offsets), np_(g.indices), np_(getattr(g, "weights", None)))


def as_csr(g) -> CSR:
    return g if isinstance(g, CSR) else CSR.from_graph(g)


# --- Algorithm 2 and its helpers -------------------------------------------------

def next_pow2(x: int) -> int:
    return int(_L().oracle_next_pow2(x))


def hashtable_primes(degree: int):
    p1, p2 = ctypes.c_uint64(), ctypes.c_uint64()
    _L().oracle_hashtable_primes(degree, ctypes.byref(p1), ctypes.byref(p2))
    return p1.value, p2.value


class Hashtable:
    """One per-vertex open-addressing table (Algorithm 2)."""

    def __init__(self, degree: int):
        self.p1, self.p2 = hashtable_primes(degree)
        self.Hk = np.full(max(self.p1, 1), EMPTY, dtype=np.int32)
        self.Hv = np.zeros(max(self.p1, 1), dtype=np.float32)
        _L().oracle_hashtable_clear(_p(self.Hk), _p(self.Hv), self.p1)

    def accumulate(self, k: int, v: float, max_retries: int = 16):
        slot = ctypes.c_int64(-1)
        probes = _L().oracle_hashtable_accumulate(_p(self.Hk), _p(self.Hv), self.p1, self.p2,
                                                  int(k), float(v), max_retries, ctypes.byref(slot))
        return probes, slot.value

    def max_key(self, tie_rule: int = 0):
        w1, w2 = ctypes.c_float(), ctypes.c_float()
        with _tie(tie_rule):
            k = _L().oracle_hashtable_max_key(_p(self.Hk), _p(self.Hv), self.p1, ctypes.byref(w1), ctypes.byref(w2))
        return k, w1.value, w2.value


# --- Algorithm 1 ------------------------------------------------------------------

def vertex_best(g, i: int, labels, tie_rule: int = 0):
    g = as_csr(g)
    labels = np.ascontiguousarray(labels, dtype=np.int32)
    w1, w2 = ctypes.c_float(), ctypes.c_float()
    with _tie(tie_rule):
        c = _L().oracle_vertex_best(int(i), _p(g.offsets), _p(g.indices), _p(g.weights), _p(labels),
                                    ctypes.byref(w1), ctypes.byref(w2))
    return int(c), w1.value, w2.value


def lpa_move_async(g, labels, unprocessed, pickless: bool, tie_rule: int = 0):
    """One asynchronous lpaMove; updates labels / unprocessed IN PLACE; returns Delta N."""
    g = as_csr(g)
    assert labels.dtype == np.int32 and labels.flags.c_contiguous
    assert unprocessed.dtype == np.uint8 and unprocessed.flags.c_contiguous
    buf_k = np.empty(2 * g.M + 1, dtype=np.int32)
    buf_v = np.empty(2 * g.M + 1, dtype=np.float32)
    with _tie(tie_rule):
        return int(_L().oracle_lpa_move_async(g.N, _p(g.offsets), _p(g.indices), _p(g.weights),
                                              _p(labels), _p(unprocessed), int(bool(pickless)),
                                              _p(buf_k), _p(buf_v)))


def lpa_move_sync(g, labels, unprocessed, pickless: bool, tie_rule: int = 0):
    """One synchronous (Jacobi) lpaMove.  Returns (dN, new_labels, new_unprocessed, w1, w2)."""
    g = as_csr(g)
    C_old = np.ascontiguousarray(labels, dtype=np.int32)
    U_old = np.ascontiguousarray(unprocessed, dtype=np.uint8)
    C_new = np.empty_like(C_old)
    U_new = np.empty_like(U_old)
    w1 = np.empty(g.N, dtype=np.float32)
    w2 = np.empty(g.N, dtype=np.float32)
    buf_k = np.empty(2 * g.M + 1, dtype=np.int32)
    buf_v = np.empty(2 * g.M + 1, dtype=np.float32)
    with _tie(tie_rule):
        dN = _L().oracle_lpa_move_sync(g.N, _p(g.offsets), _p(g.indices), _p(g.weights), _p(C_old), _p(C_new),
                                       _p(U_old), _p(U_new), int(bool(pickless)), _p(buf_k), _p(buf_v),
                                       _p(w1), _p(w2))
    return int(dN), C_new, U_new, w1, w2


def lpa(g, tolerance: float = 0.05, max_iterations: int = 20, pickless_period: int = 4, sync: bool = False,
        tie_rule: int = 0):
    """Algorithm 1 lpa().  Returns (labels, iterations, dN_per_iteration).
    Defaults are the paper's: tau = 0.05, 20 iterations, PL every 4."""
    g = as_csr(g)
    C = np.empty(g.N, dtype=np.int32)
    dN = np.zeros(max(max_iterations, 1), dtype=np.int64)
    with _tie(tie_rule):
        it = _L().oracle_lpa(g.N, _p(g.offsets), _p(g.indices), _p(g.weights), _p(C), float(tolerance),
                             int(max_iterations), int(pickless_period), int(bool(sync)), _p(dN))
    return C, int(it), dN[:it].copy()


def modularity(g, labels) -> float:
    """Equation 1, float64."""
    g = as_csr(g)
    C = np.ascontiguousarray(labels, dtype=np.int32)
    assert C.shape[0] == g.N and (g.N == 0 or (C.min() >= 0 and C.max() < g.N))
    return float(_L().oracle_modularity(g.N, _p(g.offsets), _p(g.indices), _p(g.weights), _p(C)))


# --- evaluation metric (not part of the method) ----------------------------------

def nmi(a, b) -> float:
    """Normalized mutual information, arithmetic-mean normalisation:
    NMI = 2 I(A;B) / (H(A) + H(B)); 1.0 when both partitions are trivial."""
    a = np.asarray(a).astype(np.int64)
    b = np.asarray(b).astype(np.int64)
    n = a.shape[0]
    if n == 0:
        return 1.0
    _, ai = np.unique(a, return_inverse=True)
    _, bi = np.unique(b, return_inverse=True)
    nb = bi.max() + 1
    pair = ai * nb + bi
    pa =np.bincount(ai).astype(np.float64) / n
    pb = np.bincount(bi).astype(np.float64) / n
    ha = -np.sum(pa * np.log(pa))
    hb = -np.sum(pb * np.log(pb))
    up, cnt = np.unique(pair, return_counts=True)
    pab = cnt.astype(np.float64) / n
    ia_, ib_ = up // nb, up % nb
    mi = np.sum(pab * np.log(pab / (pa[ia_] * pb[ib_])))
    if ha + hb == 0.0:
        return 1.0
    return float(2.0 * mi / (ha + hb))
