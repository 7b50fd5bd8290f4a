"""Oracle -- TEST INFRASTRUCTURE ONLY.

Plain CPU statement of what the GPU hot path computes (see oracle.cpp's header for the paper
passages each function follows).  Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  The product package
(``paper_conf_sc_mandulakgfhs24_b200``) never imports it and shares no code with it.

Functions take any object with ``offsets`` (int64[n+1]), ``col`` (int32[m]) and ``w``
(float32[m]) numpy arrays, e.g. :class:`graphgen.Graph`.

Parity status: greedy, ld_seq, ld_frontier, certificate and weight are
all pinned by tests/test_oracle.py (closed forms, Def. II.1 brute force, OPT bound, networkx
matching/maximality checks).  Nothing here is "parity unpinned".
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_SRC = os.path.join(_HERE, "oracle.cpp")
_lib = None

OK, EINVAL, ERANGE = 0, -1, -2


def build(force: bool = False) -> str:
    """Compile liboracle.so (g++ -O2 -fopenmp).  Building the checker is not using it."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        cmd = ["g++", "-O2", "-std=c++17", "-fopenmp", "-fPIC", "-shared", _SRC, "-o", _SO + ".tmp"]
        subprocess.check_call(cmd)
        os.replace(_SO + ".tmp", _SO)
    return _SO


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_SO)
        p, i64, i32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int
        lib.oracle_validate.argtypes = [p, p, p, i64, i64, i32, ctypes.c_char_p, i32]
        lib.oracle_validate.restype = i32
        lib.oracle_greedy.argtypes = [p, p, p, i64, p, p]
        lib.oracle_greedy.restype = i32
        lib.oracle_ld_seq.argtypes = [p, p, p, i64, p]
        lib.oracle_ld_seq.restype = i64
        lib.oracle_ld_frontier.argtypes = [p, p, p, i64, p, p, i64]
        lib.oracle_ld_frontier.restype = i64
        lib.oracle_certificate.argtypes = [p, p, p, i64, p, p]
        lib.oracle_certificate.restype = i32
        lib.oracle_weight.argtypes = [p, p, p, i64, p, p]
        lib.oracle_weight.restype = i32
        lib.oracle_threads.argtypes = [i32]
        lib.oracle_threads.restype = i32
        _lib = lib
    return _lib


def _arrs(g):
    off = np.ascontiguousarray(g.offsets, dtype=np.int64)
    col = np.ascontiguousarray(g.col, dtype=np.int32)
    w = np.ascontiguousarray(g.w, dtype=np.float32)
    return off, col, w, off.shape[0] - 1


@dataclass
class GreedyResult:
    mate: np.ndarray
    cardinality: int
    weight: float
    sort_s: float
    scan_s: float
    edges: int


def greedy(g) -> GreedyResult:
    """Sequential greedy = unique maximal locally dominant matching (R1)."""
    off, col, w, n = _arrs(g)
    mate = np.empty(n, dtype=np.int32)
    st = np.zeros(5, dtype=np.float64)
    _load().oracle_greedy(off.ctypes.data, col.ctypes.data, w.ctypes.data, n, mate.ctypes.data,
                          st.ctypes.data)
    return GreedyResult(mate, int(st[0]), float(st[1]), float(st[2]), float(st[3]), int(st[4]))


def ld_seq(g):
    """Algorithm 1 (LD-SEQ) literally; returns (mate, rounds incl. the final empty round)."""
    off, col, w, n = _arrs(g)
    mate = np.empty(n, dtype=np.int32)
    r = _load().oracle_ld_seq(off.ctypes.data, col.ctypes.data, w.ctypes.data, n, mate.ctypes.data)
    return mate, int(r)


def ld_frontier(g, max_rounds: int = 1 << 16):
    """Frontier-driven Alg. 1; returns (mate, pointing phases, per-phase frontier sizes)."""
    off, col, w, n = _arrs(g)
    mate = np.empty(n, dtype=np.int32)
    fs = np.zeros(max_rounds, dtype=np.int64)
    r = _load().oracle_ld_frontier(off.ctypes.data, col.ctypes.data, w.ctypes.data, n,
                                   mate.ctypes.data, fs.ctypes.data, max_rounds)
    return mate, int(r), fs[: min(r, max_rounds)].copy()


def certificate(g, mate) -> tuple[int, tuple[int, int]]:
    """0 iff mate is exactly the unique maximal LD matching; else (code, offending pair)."""
    off, col, w, n = _arrs(g)
    mate = np.ascontiguousarray(mate, dtype=np.int32)
    assert mate.shape[0] == n
    bad = np.full(2, -1, dtype=np.int64)
    code = _load().oracle_certificate(off.ctypes.data, col.ctypes.data, w.ctypes.data, n,
                                      mate.ctypes.data, bad.ctypes.data)
    return int(code), (int(bad[0]), int(bad[1]))


def weight(g, mate) -> float:
    """w(M) in fp64 (Neumaier) for any mate[]; raises if a pair is not an edge."""
    off, col, w, n = _arrs(g)
    mate = np.ascontiguousarray(mate, dtype=np.int32)
    out = ctypes.c_double(0.0)
    rc = _load().oracle_weight(off.ctypes.data, col.ctypes.data, w.ctypes.data, n,
                               mate.ctypes.data, ctypes.addressof(out))
    if rc != 0:
        raise ValueError("mate pairs a non-edge")
    return float(out.value)


def validate(offsets, col, w, n: int, m: int, level: int = 1) -> tuple[int, str]:
    off = np.ascontiguousarray(offsets, dtype=np.int64)
    c = np.ascontiguousarray(col, dtype=np.int32)
    ww = np.ascontiguousarray(w, dtype=np.float32)
    buf = ctypes.create_string_buffer(256)
    rc = _load().oracle_validate(off.ctypes.data, c.ctypes.data, ww.ctypes.data, n, m, level,
                                 buf, 256)
    return int(rc), buf.value.decode()


def threads(t: int = 0) -> int:
    return int(_load().oracle_threads(t))
