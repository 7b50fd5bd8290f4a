"""B200-native pointer-based locally dominant weighted matching (Mandulak et al., SC'24).

Thin Python binding over the C ABI declared in ``include/lmatch.h`` (``liblmatch.so``, built
in-tree for sm_100a).  Argument marshalling only: every step of the path runs in the library's
CUDA kernels.  There is NO CPU fallback -- importing this package without the built library
raises, and the library itself refuses to run without a CUDA device.

The functions keep the C names (``lmatch_create``, ``lmatch_run``, ``lmatch_weight``, ...).
Host arrays are numpy arrays; device arrays are torch CUDA tensors (torch is used only for device
memory and streams).  :class:`Matcher` is a small convenience wrapper owning one handle.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

__all__ = [
    "LMatchError", "Opts", "Stats", "Matcher", "lib_path",
    "lmatch_abi_version", "lmatch_create", "lmatch_create_ex", "lmatch_create_device",
    "lmatch_reload", "lmatch_run", "lmatch_run_device", "lmatch_weight", "lmatch_weight_device",
    "lmatch_info", "lmatch_round_log", "lmatch_round_ms", "lmatch_destroy", "lmatch_strerror",
    "lmatch_last_error", "lmatch_sweep_tile",
]

_HERE = os.path.dirname(os.path.abspath(__file__))
# LMATCH_LIB may point at an alternative build of the same library (kernel-tuning variants).
lib_path = os.environ.get("LMATCH_LIB") or os.path.join(_HERE, "liblmatch.so")
if not os.path.exists(lib_path):
    raise ImportError(
        f"{lib_path} is missing: build it with `make` (or __graft_entry__.build()). "
        "There is no CPU fallback for the matching path.")
_lib = ctypes.CDLL(lib_path)

LMATCH_OK, LMATCH_EINVAL, LMATCH_ERANGE, LMATCH_ENOMEM = 0, -1, -2, -3
LMATCH_ECUDA, LMATCH_ENCCL, LMATCH_ESTATE, LMATCH_EROUNDS = -4, -5, -6, -7


class Opts(ctypes.Structure):
    """Mirror of ``lmatch_opts`` (include/lmatch.h)."""
    _fields_ = [
        ("device", ctypes.c_int32), ("use_device", ctypes.c_int32),
        ("validate_level", ctypes.c_int32), ("timing", ctypes.c_int32),
        ("max_rounds", ctypes.c_int64), ("upload_chunk", ctypes.c_int64),
        ("hbm_budget_bytes", ctypes.c_int64), ("stream_chunk", ctypes.c_int64),
        ("round_loop", ctypes.c_int32), ("prune", ctypes.c_int32),
        ("host_cache", ctypes.c_int32), ("batches", ctypes.c_int32),
        ("algorithm", ctypes.c_int32), ("sort_chunk_log2", ctypes.c_int32),
        ("key_cache", ctypes.c_int32), ("residual_mb", ctypes.c_int32),
        ("frontier", ctypes.c_int32), ("reserved", ctypes.c_int32 * 3),
    ]


class Stats(ctypes.Structure):
    """Mirror of ``lmatch_stats`` (include/lmatch.h)."""
    _fields_ = [
        ("rounds", ctypes.c_int64), ("matched_vertices", ctypes.c_int64),
        ("cardinality", ctypes.c_int64), ("weight", ctypes.c_double),
        ("entries_swept", ctypes.c_int64), ("frontier_total", ctypes.c_int64),
        ("ms_total", ctypes.c_double), ("ms_sweep", ctypes.c_double),
        ("ms_rounds", ctypes.c_double), ("ms_round1_rest", ctypes.c_double),
        ("ms_finish", ctypes.c_double), ("sweep_launches", ctypes.c_int64),
        ("kernel_launches", ctypes.c_int64), ("bytes_streamed", ctypes.c_int64),
        ("resident_entries", ctypes.c_int64), ("cache_rows", ctypes.c_int64),
        ("host_entries_read", ctypes.c_int64), ("cache_bytes", ctypes.c_int64),
        ("tail_passes", ctypes.c_int64), ("ms_sort", ctypes.c_double), ("residual_rows", ctypes.c_int64),
    ]

    def as_dict(self) -> dict:
        return {k: getattr(self, k) for k, _ in self._fields_}


_P = ctypes.c_void_p
_I64 = ctypes.c_int64
_GP = ctypes.POINTER(_P)
_sig = {
    "lmatch_abi_version": ([], ctypes.c_int),
    "lmatch_create": ([_P, _P, _P, _I64, _I64, _GP], ctypes.c_int),
    "lmatch_create_ex": ([_P, _P, _P, _I64, _I64, ctypes.POINTER(Opts), _GP], ctypes.c_int),
    "lmatch_create_device": ([_P, _P, _P, _I64, _I64, ctypes.POINTER(Opts), _P, _GP], ctypes.c_int),
    "lmatch_reload": ([_P, _P, _P, _P], ctypes.c_int),
    "lmatch_run": ([_P, _P, ctypes.POINTER(Stats)], ctypes.c_int),
    "lmatch_run_device": ([_P, _P, _P, ctypes.POINTER(Stats)], ctypes.c_int),
    "lmatch_weight": ([_P, _P, ctypes.POINTER(ctypes.c_double)], ctypes.c_int),
    "lmatch_weight_device": ([_P, _P, _P, ctypes.POINTER(ctypes.c_double)], ctypes.c_int),
    "lmatch_info": ([_P, ctypes.POINTER(_I64), ctypes.POINTER(_I64), ctypes.POINTER(_I64),
                     ctypes.POINTER(_I64)], ctypes.c_int),
    "lmatch_round_log": ([_P, _P, _I64, ctypes.POINTER(_I64)], ctypes.c_int),
    "lmatch_round_ms": ([_P, _P, _I64, ctypes.POINTER(_I64), ctypes.POINTER(_I64)], ctypes.c_int),
    "lmatch_push_rounds": ([_P, ctypes.POINTER(_I64)], ctypes.c_int),
    "lmatch_destroy": ([_P], None),
    "lmatch_sweep_tile": ([_P], ctypes.c_int32),
    "lmatch_strerror": ([ctypes.c_int], ctypes.c_char_p),
    "lmatch_last_error": ([], ctypes.c_char_p),
}
for _name, (_args, _res) in _sig.items():
    _f = getattr(_lib, _name)
    _f.argtypes = _args
    _f.restype = _res


class LMatchError(RuntimeError):
    def __init__(self, status: int, where: str):
        self.status = status
        msg = _lib.lmatch_strerror(status).decode()
        detail = _lib.lmatch_last_error().decode()
        super().__init__(f"{where}: {msg} ({status}): {detail}")


def _check(status: int, where: str):
    if status != LMATCH_OK:
        raise LMatchError(status, where)


def _host(a, dtype):
    a = np.ascontiguousarray(a, dtype=dtype)
    return a, a.ctypes.data


def _dev_ptr(t):
    """data_ptr() of a torch CUDA tensor (or an int address)."""
    if isinstance(t, int):
        return t
    if not t.is_cuda or not t.is_contiguous():
        raise ValueError("expected a contiguous CUDA tensor")
    return t.data_ptr()


def _stream_ptr(stream):
    if stream is None:
        return None
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


# ------------------------------------------------------------------------ C-named wrappers
def lmatch_abi_version() -> int:
    return int(_lib.lmatch_abi_version())


def lmatch_sweep_tile(h=None) -> int:
    """Adjacency entries per round-1 sweep tile of handle h (None: the dense configuration's)."""
    return int(_lib.lmatch_sweep_tile(h))


def lmatch_strerror(status: int) -> str:
    return _lib.lmatch_strerror(status).decode()


def lmatch_last_error() -> str:
    return _lib.lmatch_last_error().decode()


def lmatch_create_ex(offsets, col, w, n: int | None = None, m: int | None = None,
                     opts: Opts | None = None) -> int:
    """Host CSR arrays -> handle (int address).  Raises LMatchError on failure."""
    off, p_off = _host(offsets, np.int64)
    c, p_c = _host(col, np.int32)
    ww, p_w = _host(w, np.float32)
    n = off.shape[0] - 1 if n is None else int(n)
    m = c.shape[0] if m is None else int(m)
    h = _P()
    _check(_lib.lmatch_create_ex(p_off, p_c, p_w, n, m,
                                 ctypes.byref(opts) if opts is not None else None,
                                 ctypes.byref(h)), "lmatch_create_ex")
    return h.value


def lmatch_create(offsets, col, w, n: int | None = None, m: int | None = None) -> int:
    return lmatch_create_ex(offsets, col, w, n, m, None)


def lmatch_create_device(d_offsets, d_col, d_w, n: int, m: int, opts: Opts | None = None,
                         stream=None) -> int:
    """Device CSR (torch CUDA tensors int64/int32/float32) -> handle."""
    h = _P()
    _check(_lib.lmatch_create_device(_dev_ptr(d_offsets), _dev_ptr(d_col), _dev_ptr(d_w), int(n),
                                     int(m), ctypes.byref(opts) if opts is not None else None,
                                     _stream_ptr(stream), ctypes.byref(h)), "lmatch_create_device")
    return h.value


def lmatch_reload(h: int, offsets, col, w) -> None:
    _, p_off = _host(offsets, np.int64) if not isinstance(offsets, int) else (None, offsets)
    _, p_c = _host(col, np.int32) if not isinstance(col, int) else (None, col)
    _, p_w = _host(w, np.float32) if not isinstance(w, int) else (None, w)
    _check(_lib.lmatch_reload(h, p_off, p_c, p_w), "lmatch_reload")


def lmatch_run(h: int, mate_out: np.ndarray | int | None = None, n: int | None = None):
    """Run; returns (mate int32 numpy array, Stats).  mate_out may be a preallocated int32
    array or a raw (pinned) host address (then n is required and the array is returned as None)."""
    st = Stats()
    if isinstance(mate_out, int):
        _check(_lib.lmatch_run(h, mate_out, ctypes.byref(st)), "lmatch_run")
        return None, st
    if mate_out is None:
        nn = ctypes.c_int64()
        _check(_lib.lmatch_info(h, ctypes.byref(nn), None, None, None), "lmatch_info")
        mate_out = np.empty(nn.value, dtype=np.int32)
    assert mate_out.dtype == np.int32 and mate_out.flags.c_contiguous
    _check(_lib.lmatch_run(h, mate_out.ctypes.data, ctypes.byref(st)), "lmatch_run")
    return mate_out, st


def lmatch_run_device(h: int, d_mate, stream=None) -> Stats:
    st = Stats()
    _check(_lib.lmatch_run_device(h, _dev_ptr(d_mate), _stream_ptr(stream), ctypes.byref(st)),
           "lmatch_run_device")
    return st


def lmatch_weight(h: int, mate) -> float:
    mm, p = _host(mate, np.int32)
    out = ctypes.c_double()
    _check(_lib.lmatch_weight(h, p, ctypes.byref(out)), "lmatch_weight")
    return float(out.value)


def lmatch_weight_device(h: int, d_mate, stream=None) -> float:
    out = ctypes.c_double()
    _check(_lib.lmatch_weight_device(h, _dev_ptr(d_mate), _stream_ptr(stream), ctypes.byref(out)),
           "lmatch_weight_device")
    return float(out.value)


def lmatch_info(h: int) -> dict:
    n, m, nz, db = _I64(), _I64(), _I64(), _I64()
    _check(_lib.lmatch_info(h, ctypes.byref(n), ctypes.byref(m), ctypes.byref(nz),
                            ctypes.byref(db)), "lmatch_info")
    return dict(n=n.value, m=m.value, nonempty_rows=nz.value, device_bytes=db.value,
                sweep_tile=int(_lib.lmatch_sweep_tile(h)))


def lmatch_round_log(h: int) -> np.ndarray:
    """Per-round (|F_r|, |L_r|, E(F_r)) of the last run, shape (rounds, 3)."""
    nr = _I64()
    _check(_lib.lmatch_round_log(h, None, 0, ctypes.byref(nr)), "lmatch_round_log")
    out = np.zeros((max(nr.value, 1), 3), dtype=np.int64)
    _check(_lib.lmatch_round_log(h, out.ctypes.data, nr.value, ctypes.byref(nr)), "lmatch_round_log")
    return out[: nr.value]


def lmatch_round_ms(h: int):
    """(timing=1) per-round device ms of the host-driven rounds >= 2 of the last run, and the index
    of the entry that covers the persistent-kernel tail (-1 if none)."""
    nr, tf = _I64(), _I64()
    _check(_lib.lmatch_round_ms(h, None, 0, ctypes.byref(nr), ctypes.byref(tf)), "lmatch_round_ms")
    out = np.zeros(max(nr.value, 1), dtype=np.float64)
    _check(_lib.lmatch_round_ms(h, out.ctypes.data, nr.value, ctypes.byref(nr), ctypes.byref(tf)),
           "lmatch_round_ms")
    return out[: nr.value], int(tf.value)


def lmatch_push_rounds(h: int) -> int:
    """Rounds of the last run whose next frontier was pushed (A6 push frontier)."""
    r = _I64()
    _check(_lib.lmatch_push_rounds(h, ctypes.byref(r)), "lmatch_push_rounds")
    return int(r.value)


def lmatch_destroy(h: int | None) -> None:
    _lib.lmatch_destroy(h)


# ------------------------------------------------------------------------------ convenience
class Matcher:
    """Owns one lmatch handle.  ``Matcher(graph)`` uploads host CSR arrays; ``Matcher.from_device``
    wraps torch CUDA tensors.  ``run()`` -> (mate, stats dict)."""

    def __init__(self, offsets=None, col=None, w=None, *, handle: int | None = None,
                 validate_level: int = 1, timing: bool = False, upload_chunk: int = 0,
                 max_rounds: int = 0, hbm_budget_bytes: int = 0, stream_chunk: int = 0,
                 round_loop: int = 0, prune: bool = False, host_cache: bool = True,
                 batches: int = 0, algorithm: str = "ld", sort_chunk_log2: int = 0,
                 key_cache: bool = False, residual_mb: int = 0, frontier: str = "auto"):
        self.h = None
        if handle is not None:
            self.h = handle
        else:
            if hasattr(offsets, "offsets"):  # a graphgen.Graph-like object
                offsets, col, w = offsets.offsets, offsets.col, offsets.w
            self.h = lmatch_create_ex(offsets, col, w,
                                      opts=make_opts(validate_level, timing, upload_chunk,
                                                     max_rounds, hbm_budget_bytes, stream_chunk,
                                                     round_loop, prune, host_cache, batches,
                                                     algorithm, sort_chunk_log2, key_cache,
                                                     residual_mb, frontier))
        self.info = lmatch_info(self.h)

    @classmethod
    def from_device(cls, d_offsets, d_col, d_w, n, m, stream=None, **kw):
        h = lmatch_create_device(d_offsets, d_col, d_w, n, m,
                                 make_opts(kw.get("validate_level", 1), kw.get("timing", False),
                                           0, kw.get("max_rounds", 0),
                                           algorithm=kw.get("algorithm", "ld")), stream)
        return cls(handle=h)

    def run(self, mate_out=None):
        mate, st = lmatch_run(self.h, mate_out)
        return mate, st.as_dict()

    def run_device(self, d_mate, stream=None) -> dict:
        return lmatch_run_device(self.h, d_mate, stream).as_dict()

    def weight(self, mate) -> float:
        return lmatch_weight(self.h, mate)

    def push_rounds(self) -> int:
        return lmatch_push_rounds(self.h)

    def reload(self, offsets, col, w) -> None:
        lmatch_reload(self.h, offsets, col, w)

    def close(self):
        if self.h is not None:
            lmatch_destroy(self.h)
            self.h = None

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def make_opts(validate_level: int = 1, timing: bool = False, upload_chunk: int = 0,
              max_rounds: int = 0, hbm_budget_bytes: int = 0, stream_chunk: int = 0,
              round_loop: int = 0, prune: bool = False, host_cache: bool = True,
              batches: int = 0, algorithm: str = "ld", sort_chunk_log2: int = 0,
              key_cache: bool = False, residual_mb: int = 0, frontier: str = "auto") -> Opts:
    """round_loop (include/lmatch.h): 0 = hybrid (work-sized launches, then one persistent kernel
    for the tail; default), 1 = host-driven launches only, 2 = persistent kernel after round 1,
    3 = CUDA graph {round 1, persistent kernel}."""
    o = Opts()
    o.round_loop = int(round_loop)
    o.prune = int(bool(prune))
    o.host_cache = 0 if host_cache else -1
    o.batches = int(batches)
    o.algorithm = {"ld": 0, "suitor": 1, "hybrid": 2, "sorted": 3}[algorithm]
    o.sort_chunk_log2 = int(sort_chunk_log2)
    o.key_cache = 1 if key_cache else 0
    o.residual_mb = int(residual_mb)
    o.frontier = {"auto": 0, "pull": 1, "push": 2}[frontier]
    o.hbm_budget_bytes = int(hbm_budget_bytes)
    o.stream_chunk = int(stream_chunk)
    o.validate_level = int(validate_level)
    o.timing = int(bool(timing))
    o.upload_chunk = int(upload_chunk)
    o.max_rounds = int(max_rounds)
    return o
