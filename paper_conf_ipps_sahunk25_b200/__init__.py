"""paper_conf_ipps_sahunk25_b200 -- B200-native nu-LPA (PAPER.md, Sahu).

Thin ctypes binding of the C ABI in ``include/nulpa.h`` (library
``libnulpa.so`` built in-tree for sm_100a by ``build.py``).  Every function
here only marshals arguments: all steps of the label sweep, the convergence
loop and the modularity run in the CUDA kernels of ``csrc/nulpa.cu``.  There
is no CPU fallback: if the library or a CUDA device is missing, calls raise.

The functions carry the C names (``nulpa_create``, ``nulpa_run``,
``nulpa_sweep``, ``nulpa_labels``, ``nulpa_modularity`` ...); ``Graph`` is a
small convenience wrapper over a handle.
"""
from __future__ import annotations

import ctypes
import os
from typing import Optional

__all__ = [
    "NulpaError", "Params", "Stats", "Graph", "lpa", "load_library", "library_path",
    "nulpa_create", "nulpa_run", "nulpa_sweep", "nulpa_labels", "nulpa_set_labels", "nulpa_flags",
    "nulpa_modularity", "nulpa_modularity_partial", "nulpa_modularity_finish", "nulpa_reset",
    "nulpa_bind_state", "nulpa_get_stats", "nulpa_release_memory", "nulpa_pack_changed", "nulpa_apply_pairs",
    "nulpa_pack_flag_bits", "nulpa_or_flag_bits", "nulpa_destroy", "nulpa_default_params", "nulpa_version",
    "ASYNC", "SYNC", "MEM_HOST", "MEM_DEVICE",
]

_PKG = os.path.dirname(os.path.abspath(__file__))
# NULPA_LIB: load another build of the library (kernel A/B experiments only)
_LIB_PATH = os.environ.get("NULPA_LIB") or os.path.join(_PKG, "libnulpa.so")

ASYNC, SYNC = 0, 1
TIE_SMALLEST = 0            # the only tie rule: smallest label (R6)
MEM_HOST, MEM_DEVICE = 0, 1
BINS = ("thread", "warp", "block", "giant")


class NulpaError(RuntimeError):
    pass


class Params(ctypes.Structure):
    _fields_ = [
        ("tolerance", ctypes.c_double),
        ("max_iterations", ctypes.c_int32),
        ("pickless_period", ctypes.c_int32),
        ("mode", ctypes.c_int32),
        ("switch_degree", ctypes.c_int32),
        ("block_degree", ctypes.c_int32),
        ("giant_degree", ctypes.c_int32),
        ("reset", ctypes.c_int32),
        ("timing", ctypes.c_int32),
        ("tie_rule", ctypes.c_int32),
        ("bin_order", ctypes.c_int32),
        ("wide_degree", ctypes.c_int32),
        ("first_sweep_block", ctypes.c_int32),
        ("sweep_block", ctypes.c_int32),
        ("device_loop", ctypes.c_int32),
    ]


class Stats(ctypes.Structure):
    _fields_ = [
        ("iterations", ctypes.c_int32),
        ("converged", ctypes.c_int32),
        ("changed", ctypes.c_int64 * 64),
        ("vertices_processed", ctypes.c_int64 * 4),
        ("edges_scanned", ctypes.c_int64 * 4),
        ("vertices_changed", ctypes.c_int64 * 4),
        ("changed_edges", ctypes.c_int64 * 4),
        ("kernel_ms", ctypes.c_double * 4),
        ("launches", ctypes.c_int32 * 4),
        ("other_launches", ctypes.c_int32),
        ("bin_vertices", ctypes.c_int64 * 4),
        ("bin_edges", ctypes.c_int64 * 4),
        ("run_ms", ctypes.c_double),
        ("iter_kernel_ms", (ctypes.c_double * 4) * 64),
        ("iter_processed", (ctypes.c_int64 * 4) * 64),
        ("iter_edges", (ctypes.c_int64 * 4) * 64),
        ("iter_changed", (ctypes.c_int64 * 4) * 64),
        ("iter_changed_edges", (ctypes.c_int64 * 4) * 64),
    ]

    def to_dict(self) -> dict:
        it = self.iterations
        return dict(
            iterations=it, converged=bool(self.converged), changed=list(self.changed[:min(it, 64)]),
            vertices_processed=list(self.vertices_processed), edges_scanned=list(self.edges_scanned),
            vertices_changed=list(self.vertices_changed), changed_edges=list(self.changed_edges),
            kernel_ms=list(self.kernel_ms),
            launches=list(self.launches), other_launches=self.other_launches,
            bin_vertices=list(self.bin_vertices), bin_edges=list(self.bin_edges), run_ms=self.run_ms,
            per_iteration=[dict(kernel_ms=list(self.iter_kernel_ms[l]), processed=list(self.iter_processed[l]),
                                edges=list(self.iter_edges[l]), changed=list(self.iter_changed[l]),
                                changed_edges=list(self.iter_changed_edges[l])) for l in range(min(it, 64))],
        )


_lib = None


def library_path() -> str:
    return _LIB_PATH


def load_library():
    """Load the in-tree libnulpa.so (raises if it was not built)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(_LIB_PATH):
        raise NulpaError(f"{_LIB_PATH} is missing: build it with `python -m paper_conf_ipps_sahunk25_b200.build` "
                         "(or __graft_entry__.build()); there is no CPU fallback")
    lib = ctypes.CDLL(_LIB_PATH)
    vp, i32, i64, f64 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_double
    P = ctypes.POINTER
    sig = {
        "nulpa_default_params": (None, [P(Params)]),
        "nulpa_last_error": (ctypes.c_char_p, []),
        "nulpa_version": (ctypes.c_char_p, []),
        "nulpa_create": (ctypes.c_int, [vp, vp, vp, i64, i64, i64, ctypes.c_int, vp, P(vp)]),
        "nulpa_bind_state": (ctypes.c_int, [vp, vp, vp]),
        "nulpa_run": (ctypes.c_int, [vp, P(Params), P(Stats)]),
        "nulpa_sweep": (ctypes.c_int, [vp, ctypes.c_int, P(Params), P(i64)]),
        "nulpa_reset": (ctypes.c_int, [vp]),
        "nulpa_labels": (ctypes.c_int, [vp, vp, ctypes.c_int]),
        "nulpa_set_labels": (ctypes.c_int, [vp, vp, vp, ctypes.c_int]),
        "nulpa_flags": (ctypes.c_int, [vp, vp, ctypes.c_int]),
        "nulpa_modularity": (ctypes.c_int, [vp, vp, ctypes.c_int, P(f64)]),
        "nulpa_modularity_partial": (ctypes.c_int, [vp, vp, P(f64), P(f64), vp]),
        "nulpa_modularity_finish": (ctypes.c_int, [vp, vp, f64, f64, P(f64)]),
        "nulpa_get_stats": (ctypes.c_int, [vp, P(Stats)]),
        "nulpa_state_pointers": (ctypes.c_int, [vp, P(vp), P(vp)]),
        "nulpa_destroy": (ctypes.c_int, [vp]),
        "nulpa_release_memory": (ctypes.c_int, []),
        "nulpa_pack_changed": (ctypes.c_int, [vp, vp, vp, P(i64)]),
        "nulpa_apply_pairs": (ctypes.c_int, [vp, vp, i64]),
        "nulpa_pack_flag_bits": (ctypes.c_int, [vp, vp, ctypes.c_int, i64, vp]),
        "nulpa_or_flag_bits": (ctypes.c_int, [vp, vp, ctypes.c_int, i64]),
    }
    for name, (res, args) in sig.items():
        f = getattr(lib, name)
        f.restype = res
        f.argtypes = args
    _lib = lib
    return lib


def _check(rc: int):
    if rc != 0:
        msg = load_library().nulpa_last_error().decode(errors="replace")
        raise NulpaError(f"nulpa error {rc}: {msg}")


def _ptr(t) -> Optional[int]:
    if t is None:
        return None
    if hasattr(t, "data_ptr"):
        return t.data_ptr()
    return t.ctypes.data  # numpy


def _is_device(t) -> bool:
    return t is not None and hasattr(t, "is_cuda") and t.is_cuda


def _stream_handle(stream=None) -> Optional[int]:
    import torch
    s = stream if stream is not None else torch.cuda.current_stream()
    return s.cuda_stream


def nulpa_version() -> str:
    return load_library().nulpa_version().decode()


def nulpa_default_params(**overrides) -> Params:
    p = Params()
    load_library().nulpa_default_params(ctypes.byref(p))
    for k, v in overrides.items():
        if v is not None:
            setattr(p, k, v)
    return p


def nulpa_create(offsets, indices, weights=None, n_rows=None, n_global=None, row_begin=0, stream=None):
    """Create a handle.  torch CUDA tensors are borrowed (device memkind);
    host tensors / numpy arrays are copied to the device by the library."""
    dev = _is_device(indices) or _is_device(offsets)
    n_rows = int(offsets.shape[0] - 1) if n_rows is None else int(n_rows)
    n_global = n_rows if n_global is None else int(n_global)
    h = ctypes.c_void_p()
    _check(load_library().nulpa_create(_ptr(offsets), _ptr(indices), _ptr(weights), n_rows, n_global,
                                       int(row_begin), MEM_DEVICE if dev else MEM_HOST,
                                       _stream_handle(stream), ctypes.byref(h)))
    return h


def nulpa_run(h, params: Optional[Params] = None) -> Stats:
    st = Stats()
    _check(load_library().nulpa_run(h, ctypes.byref(params) if params is not None else None, ctypes.byref(st)))
    return st


def nulpa_sweep(h, pickless: bool, params: Optional[Params] = None, want_changed: bool = True) -> Optional[int]:
    dn = ctypes.c_int64(-1)
    _check(load_library().nulpa_sweep(h, int(bool(pickless)), ctypes.byref(params) if params is not None else None,
                                      ctypes.byref(dn) if want_changed else None))
    return dn.value if want_changed else None


def nulpa_reset(h):
    _check(load_library().nulpa_reset(h))


def nulpa_labels(h, out):
    _check(load_library().nulpa_labels(h, _ptr(out), MEM_DEVICE if _is_device(out) else MEM_HOST))
    return out


def nulpa_flags(h, out):
    _check(load_library().nulpa_flags(h, _ptr(out), MEM_DEVICE if _is_device(out) else MEM_HOST))
    return out


def nulpa_set_labels(h, labels, flags=None):
    dev = _is_device(labels)
    if flags is not None and _is_device(flags) != dev:
        raise NulpaError("labels and flags must live in the same memory")
    _check(load_library().nulpa_set_labels(h, _ptr(labels), _ptr(flags), MEM_DEVICE if dev else MEM_HOST))


def nulpa_modularity(h, labels=None) -> float:
    q = ctypes.c_double()
    _check(load_library().nulpa_modularity(h, _ptr(labels), MEM_DEVICE if _is_device(labels) else MEM_HOST,
                                           ctypes.byref(q)))
    return q.value


def nulpa_modularity_partial(h, labels_device, Sigma_device):
    s, m = ctypes.c_double(0.0), ctypes.c_double(0.0)
    _check(load_library().nulpa_modularity_partial(h, _ptr(labels_device), ctypes.byref(s), ctypes.byref(m),
                                                   _ptr(Sigma_device)))
    return s.value, m.value


def nulpa_modularity_finish(h, Sigma_device, sigma_intra: float, two_m: float) -> float:
    q = ctypes.c_double()
    _check(load_library().nulpa_modularity_finish(h, _ptr(Sigma_device), float(sigma_intra), float(two_m),
                                                  ctypes.byref(q)))
    return q.value


def nulpa_bind_state(h, labels_device, flags_device):
    _check(load_library().nulpa_bind_state(h, _ptr(labels_device), _ptr(flags_device)))


def nulpa_release_memory():
    """Return pooled device memory of destroyed handles to the driver."""
    _check(load_library().nulpa_release_memory())


def nulpa_pack_changed(h, prev_device, pairs_device) -> int:
    n = ctypes.c_int64(0)
    _check(load_library().nulpa_pack_changed(h, _ptr(prev_device), _ptr(pairs_device), ctypes.byref(n)))
    return n.value


def nulpa_apply_pairs(h, pairs_device, n: int):
    _check(load_library().nulpa_apply_pairs(h, _ptr(pairs_device), int(n)))


def nulpa_pack_flag_bits(h, bounds_device, P: int, words: int, bits_device):
    _check(load_library().nulpa_pack_flag_bits(h, _ptr(bounds_device), int(P), int(words), _ptr(bits_device)))


def nulpa_or_flag_bits(h, bits_device, P: int, words: int):
    _check(load_library().nulpa_or_flag_bits(h, _ptr(bits_device), int(P), int(words)))


def nulpa_get_stats(h) -> Stats:
    st = Stats()
    _check(load_library().nulpa_get_stats(h, ctypes.byref(st)))
    return st


def nulpa_destroy(h):
    if h:
        _check(load_library().nulpa_destroy(h))


class Graph:
    """A graph (or row shard) resident on the GPU with its label state."""

    def __init__(self, offsets, indices, weights=None, *, n_global=None, row_begin=0, stream=None):
        import torch
        if not torch.cuda.is_available():
            raise NulpaError("nu-LPA needs a CUDA device (sm_100a); there is no CPU fallback")
        self._keep = (offsets, indices, weights)   # borrowed device arrays stay alive
        self.n_rows = int(offsets.shape[0] - 1)
        self.n_global = self.n_rows if n_global is None else int(n_global)
        self.row_begin = int(row_begin)
        self.weighted = weights is not None
        self.h = nulpa_create(offsets, indices, weights, self.n_rows, self.n_global, row_begin, stream)

    @classmethod
    def from_synth(cls, g, **kw):
        return cls(g.offsets, g.indices, g.weights, **kw)

    def close(self):
        if getattr(self, "h", None):
            nulpa_destroy(self.h)
            self.h = None
            nulpa_release_memory()          # hand the pooled memory back (torch may need it next)

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def run(self, **kw) -> dict:
        return nulpa_run(self.h, nulpa_default_params(**kw)).to_dict()

    def sweep(self, pickless: bool, **kw) -> int:
        return nulpa_sweep(self.h, pickless, nulpa_default_params(**kw))

    def reset(self):
        nulpa_reset(self.h)

    def labels(self, device: bool = True):
        import torch
        out = torch.empty(self.n_global, dtype=torch.int32, device="cuda" if device else "cpu")
        return nulpa_labels(self.h, out)

    def flags(self, device: bool = True):
        import torch
        out = torch.empty(self.n_global, dtype=torch.uint8, device="cuda" if device else "cpu")
        return nulpa_flags(self.h, out)

    def set_labels(self, labels, flags=None):
        nulpa_set_labels(self.h, labels, flags)

    def modularity(self, labels=None) -> float:
        return nulpa_modularity(self.h, labels)

    def bind_state(self, labels_device, flags_device):
        self._bound = (labels_device, flags_device)
        nulpa_bind_state(self.h, labels_device, flags_device)

    def stats(self) -> dict:
        return nulpa_get_stats(self.h).to_dict()


def lpa(offsets, indices, weights=None, **params):
    """One-call nu-LPA: returns (labels as a CUDA int32 tensor, stats dict)."""
    g = Graph(offsets, indices, weights)
    try:
        st = g.run(**params)
        return g.labels(), st
    finally:
        g.close()
