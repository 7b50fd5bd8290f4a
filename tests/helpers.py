"""Test-side helpers: golden fixture loader and brute-force checks written straight from the
paper's definitions.  These are independent of oracle/ (no shared code) so that they can pin it.
"""
from __future__ import annotations

import itertools
import os

import numpy as np

import graphgen

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def load_golden(name: str):
    """Returns (graph, expected_mate, expected_phases, expected_weight)."""
    n, edges, mate, phases, weight = None, [], None, None, None
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            tok = line.split()
            if tok[0] == "n":
                n = int(tok[1])
            elif tok[0] == "e":
                edges.append((int(tok[1]), int(tok[2]), float(tok[3])))
            elif tok[0] == "mate":
                mate = np.array([int(t) for t in tok[1:]], dtype=np.int32)
            elif tok[0] == "phases":
                phases = int(tok[1])
            elif tok[0] == "weight":
                weight = float(tok[1])
    return graphgen.from_edges(n, edges), mate, phases, weight


def golden_names():
    return sorted(f for f in os.listdir(GOLDEN) if f.endswith(".txt"))


def edge_list(g):
    """Undirected edges {(u, v): w} with u < v (self-loops dropped), from the CSR."""
    E = {}
    for u in range(g.n):
        for j in range(g.offsets[u], g.offsets[u + 1]):
            v = int(g.col[j])
            if u < v:
                E[(u, v)] = float(g.w[j])
    return E


def strict_key(e, w):
    """Strict total order on edges: (weight, max endpoint, min endpoint) (R1)."""
    u, v = e
    return (w, max(u, v), min(u, v))


def all_matchings(E):
    """Every matching of the edge set E (list of (u,v)), by brute force."""
    edges = list(E)
    out = []

    def rec(i, used, cur):
        if i == len(edges):
            out.append(tuple(cur))
            return
        rec(i + 1, used, cur)
        u, v = edges[i]
        if u not in used and v not in used:
            rec(i + 1, used | {u, v}, cur + [edges[i]])

    rec(0, frozenset(), [])
    return out


def is_maximal(M, E):
    used = {x for e in M for x in e}
    return all(u in used or v in used for (u, v) in E)


def is_locally_dominant(M, E, strict=True):
    """Def. II.1: M is LD if its edges can be inserted in some order such that each edge,
    when added, is (strictly, under the total order; or >= by weight if strict=False) heavier than
    every *available* adjacent edge w.r.t. the matching built so far."""
    for order in itertools.permutations(M):
        cur_used = set()
        ok = True
        for e in order:
            u, v = e
            ke = strict_key(e, E[e])
            for f, wf in E.items():
                if f == e or (u not in f and v not in f):
                    continue
                if f[0] in cur_used or f[1] in cur_used:
                    continue  # not available
                if strict:
                    if not ke > strict_key(f, wf):
                        ok = False
                        break
                else:
                    if not E[e] >= wf:
                        ok = False
                        break
            if not ok:
                break
            cur_used |= {u, v}
        if ok:
            return True
    return False


def mate_from_pairs(n, M):
    mate = np.full(n, -1, dtype=np.int32)
    for u, v in M:
        mate[u] = v
        mate[v] = u
    return mate


def brute_opt(E):
    """Maximum weight matching value by enumeration (tiny graphs only)."""
    best = 0.0
    for M in all_matchings(E):
        best = max(best, sum(E[e] for e in M))
    return best
