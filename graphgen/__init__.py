"""Seeded synthetic graph inputs shared by the oracle tests, the CUDA parity tests and bench.py.

This package holds none of the matching method's arithmetic -- it only produces symmetric CSR
graphs ``(offsets int64[n+1], col int32[m], w float32[m])`` shaped like the paper's workloads
(PAPER.md:179 weights "uniform ... three decimal points from [0,1]"; Table I graph classes,
PAPER.md:187-207).  All randomness is a counter-based hash of (seed, index) implemented in
``graphgen.cpp``; outputs are identical for any thread count.  Recipe: DESIGN.md "Input recipe".
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass, field

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libgraphgen.so")
_SRC = os.path.join(_HERE, "graphgen.cpp")
_HDR = os.path.join(_HERE, "gg_common.h")
_lib = None

WEIGHT_MODES = {"uniform": 0, "paper": 1, "gradient": 2, "ones": 3}


def build(force: bool = False) -> str:
    """Compile libgraphgen.so (g++ -O3 -fopenmp)."""
    stale = not os.path.exists(_SO) or os.path.getmtime(_SO) < max(os.path.getmtime(_SRC),
                                                                    os.path.getmtime(_HDR))
    if force or stale:
        cmd = ["g++", "-O3", "-march=x86-64-v3", "-ffp-contract=off", "-std=c++17", "-fopenmp", "-fPIC", "-shared",
               _SRC, "-o", _SO + ".tmp"]
        subprocess.check_call(cmd)
        os.replace(_SO + ".tmp", _SO)
    return _SO


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_SO)
        i64, i32, u64, f64 = ctypes.c_int64, ctypes.c_int, ctypes.c_uint64, ctypes.c_double
        p = ctypes.c_void_p
        lib.gg_er_csr.argtypes = [i64, f64, u64, p, p, i64]
        lib.gg_er_csr.restype = i64
        lib.gg_er_max_entries.argtypes = [i64, f64]
        lib.gg_er_max_entries.restype = i64
        lib.gg_rmat_csr.argtypes = [i32, i64, u64, f64, f64, f64, p, p, i64]
        lib.gg_rmat_csr.restype = i64
        lib.gg_mesh_csr.argtypes = [i64, i32, u64, p, p, i64]
        lib.gg_mesh_csr.restype = i64
        lib.gg_weights.argtypes = [p, p, i64, u64, i32, i64, p]
        lib.gg_weights.restype = i32
        lib.gg_hash.argtypes = [u64, u64, u64]
        lib.gg_hash.restype = u64
        lib.gg_set_threads.argtypes = [i32]
        lib.gg_set_threads.restype = i32
        _lib = lib
    return _lib


@dataclass
class Graph:
    """Symmetric CSR graph. ``m`` counts directed entries (= offsets[n]); ``m_u`` = m/2."""
    offsets: np.ndarray  # int64[n+1]
    col: np.ndarray      # int32[m]
    w: np.ndarray        # float32[m]
    name: str = "graph"
    meta: dict = field(default_factory=dict)

    @property
    def n(self) -> int:
        return int(self.offsets.shape[0] - 1)

    @property
    def m(self) -> int:
        return int(self.offsets[-1])

    @property
    def m_u(self) -> int:
        return self.m // 2

    def degrees(self) -> np.ndarray:
        return np.diff(self.offsets)


def _ptr(a: np.ndarray) -> int:
    return a.ctypes.data


def _weights(offsets, col, n, seed, weights, side=0) -> np.ndarray:
    lib = _load()
    w = np.empty(col.shape[0], dtype=np.float32)
    mode = WEIGHT_MODES[weights]
    lib.gg_weights(_ptr(offsets), _ptr(col), n, seed, mode, side, _ptr(w))
    return w


def er(n: int, avg_degree: float = 16.0, seed: int = 1, weights: str = "uniform",
       wseed: int | None = None) -> Graph:
    """Erdos-Renyi: n*avg_degree/2 iid uniform pairs; loops dropped; duplicates merged."""
    lib = _load()
    cap = lib.gg_er_max_entries(n, avg_degree)
    offsets = np.empty(n + 1, dtype=np.int64)
    col = np.empty(max(cap, 1), dtype=np.int32)
    m = lib.gg_er_csr(n, avg_degree, seed, _ptr(offsets), _ptr(col), cap)
    assert m >= 0, m
    col = col[:m]
    w = _weights(offsets, col, n, seed if wseed is None else wseed, weights)
    return Graph(offsets, col, w, name=f"er_n{n}_d{avg_degree:g}",
                 meta=dict(kind="er", n=n, avg_degree=avg_degree, seed=seed, weights=weights))


def rmat(scale: int, edgefactor: int = 16, seed: int = 1, a: float = 0.57, b: float = 0.19,
         c: float = 0.19, weights: str = "uniform", wseed: int | None = None) -> Graph:
    """Graph500-style R-MAT (A,B,C,D = .57,.19,.19,.05), random relabel, loops dropped, dedup."""
    lib = _load()
    n = 1 << scale
    cap = 2 * edgefactor * n
    offsets = np.empty(n + 1, dtype=np.int64)
    col = np.empty(cap, dtype=np.int32)
    m = lib.gg_rmat_csr(scale, edgefactor, seed, a, b, c, _ptr(offsets), _ptr(col), cap)
    assert m >= 0, m
    col = col[:m]
    w = _weights(offsets, col, n, seed if wseed is None else wseed, weights)
    return Graph(offsets, col, w, name=f"rmat_s{scale}_ef{edgefactor}",
                 meta=dict(kind="rmat", scale=scale, edgefactor=edgefactor, seed=seed,
                           weights=weights))


def mesh(side: int, keep: float = 1.0, seed: int = 1, weights: str = "uniform",
         wseed: int | None = None) -> Graph:
    """side x side 4-neighbour grid; keep<1 thins edges symmetrically ("road-like")."""
    lib = _load()
    n = side * side
    cap = 4 * n
    offsets = np.empty(n + 1, dtype=np.int64)
    col = np.empty(max(cap, 1), dtype=np.int32)
    m = lib.gg_mesh_csr(side, int(round(keep * 1000)), seed, _ptr(offsets), _ptr(col), cap)
    assert m >= 0, m
    col = col[:m]
    w = _weights(offsets, col, n, seed if wseed is None else wseed, weights, side)
    return Graph(offsets, col, w, name=f"mesh_{side}x{side}" + ("" if keep >= 1 else f"_keep{keep:g}"),
                 meta=dict(kind="mesh", side=side, keep=keep, seed=seed, weights=weights))


def from_edges(n: int, edges, weights=None) -> Graph:
    """Symmetric CSR from an undirected edge list [(u, v[, w]), ...] (hand-made test graphs).

    Both directions are emitted; rows are sorted by neighbour id.  Self-loops are kept if given
    (the method ignores them), so tests can exercise that rule.
    """
    us, vs, ws = [], [], []
    for k, e in enumerate(edges):
        u, v = int(e[0]), int(e[1])
        wt = float(e[2]) if len(e) > 2 else float(weights[k])
        us.append(u); vs.append(v); ws.append(wt)
        if u != v:
            us.append(v); vs.append(u); ws.append(wt)
    us = np.asarray(us, dtype=np.int64)
    vs = np.asarray(vs, dtype=np.int64)
    ws = np.asarray(ws, dtype=np.float32)
    order = np.lexsort((vs, us)) if us.size else np.zeros(0, dtype=np.int64)
    us, vs, ws = us[order], vs[order], ws[order]
    offsets = np.zeros(n + 1, dtype=np.int64)
    if us.size:
        np.add.at(offsets, us + 1, 1)
    offsets = np.cumsum(offsets).astype(np.int64)
    return Graph(offsets, vs.astype(np.int32), ws, name="edges", meta=dict(kind="edges"))


def random_small(n: int, p: float, rng: np.random.Generator, levels: int | None = None) -> Graph:
    """Tiny G(n, p) graph with weights uniform in (0,1]; ``levels`` quantises weights (ties)."""
    edges = []
    for u in range(n):
        for v in range(u + 1, n):
            if rng.random() < p:
                if levels:
                    wt = float(rng.integers(1, levels + 1)) / levels
                else:
                    wt = float(np.float32(1.0 - rng.random()))
                edges.append((u, v, wt))
    return from_edges(n, edges)


def hash2(seed: int, a: int, b: int) -> int:
    return int(_load().gg_hash(seed, a, b))


def set_threads(t: int) -> int:
    return int(_load().gg_set_threads(t))
