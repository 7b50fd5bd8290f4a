"""Pins for the oracle (CPU only, ``-m "not gpu"``).

Each test pins an oracle function to something other than itself:
hand-worked closed forms (tests/golden), the paper's definitions checked by brute force
(Def. II.1, maximality P:42), the 1/2 bound against an independently computed optimum
(Lemma II.1, Cor. II.1 P:80; brute force and networkx's blossom), networkx's own matching /
maximality predicates, and agreement between the paper's two formulations (global-sort greedy,
P:52, and Algorithm 1) on thousands of random tiny graphs with heavy ties.
"""
import math

import networkx as nx
import numpy as np
import pytest

import graphgen
import oracle
from helpers import (all_matchings, brute_opt, edge_list, golden_names, is_locally_dominant,
                     is_maximal, load_golden, mate_from_pairs)


# --------------------------------------------------------------------------- closed forms
@pytest.mark.parametrize("name", golden_names())
def test_golden_closed_forms(name):
    g, mate, phases, weight = load_golden(name)
    r = oracle.greedy(g)
    np.testing.assert_array_equal(r.mate, mate)
    assert math.isclose(r.weight, weight, rel_tol=1e-12)
    m1, _ = oracle.ld_seq(g)
    np.testing.assert_array_equal(m1, mate)
    m2, ph, _ = oracle.ld_frontier(g)
    np.testing.assert_array_equal(m2, mate)
    assert ph == phases
    assert oracle.certificate(g, mate)[0] == 0
    assert math.isclose(oracle.weight(g, mate), weight, rel_tol=1e-12)


@pytest.mark.parametrize("n", list(range(2, 40)))
def test_increasing_path(n):
    """w(i,i+1) = i+1: M* = {(n-2,n-1), (n-4,n-3), ...}; one match per phase, so the
    frontier iteration runs floor(n/2) + (n mod 2) phases and literal Alg. 1 runs floor(n/2)+1
    rounds (its last round adds nothing)."""
    g = graphgen.from_edges(n, [(i, i + 1, float(i + 1)) for i in range(n - 1)])
    expect = np.full(n, -1, dtype=np.int32)
    for hi in range(n - 1, 0, -2):
        expect[hi], expect[hi - 1] = hi - 1, hi
    np.testing.assert_array_equal(oracle.greedy(g).mate, expect)
    m1, r1 = oracle.ld_seq(g)
    np.testing.assert_array_equal(m1, expect)
    assert r1 == n // 2 + 1
    m2, ph, fs = oracle.ld_frontier(g)
    np.testing.assert_array_equal(m2, expect)
    assert ph == n // 2 + (n % 2)
    assert fs[0] == n and all(f == 1 for f in fs[1:])
    assert math.isclose(oracle.greedy(g).weight, sum(range(n - 1, 0, -2)), rel_tol=0)


def test_trivial_cases():
    # m = 0: everything unmatched, zero phases
    g = graphgen.from_edges(5, [])
    assert (oracle.greedy(g).mate == -1).all()
    assert oracle.ld_frontier(g)[1] == 0
    assert oracle.certificate(g, np.full(5, -1, np.int32))[0] == 0
    # disjoint edges: all matched in one phase
    g = graphgen.from_edges(8, [(0, 1, .3), (2, 3, .1), (4, 5, .7), (6, 7, .2)])
    r = oracle.greedy(g)
    np.testing.assert_array_equal(r.mate, [1, 0, 3, 2, 5, 4, 7, 6])
    assert oracle.ld_frontier(g)[1] == 1
    # K_n with distinct weights: hand greedy
    n = 6
    E = [(u, v, float(1 + u * n + v) / 64) for u in range(n) for v in range(u + 1, n)]
    g = graphgen.from_edges(n, E)
    # heaviest (4,5), then (2,3), then (0,1)
    np.testing.assert_array_equal(oracle.greedy(g).mate, [1, 0, 3, 2, 5, 4])


# --------------------------------------------------------------------- definition-level pins
def _random_tiny(rng, nmax=7):
    n = int(rng.integers(2, nmax + 1))
    p = float(rng.choice([0.3, 0.5, 0.8, 1.0]))
    levels = rng.choice([0, 2, 3, 10])
    return graphgen.random_small(n, p, rng, levels=int(levels) if levels else None)


def test_unique_ld_matching_by_definition():
    """Def. II.1 with the strict order: among ALL matchings, exactly one is maximal and
    locally dominant, and it is the oracle's."""
    rng = np.random.default_rng(11)
    for _ in range(300):
        g = _random_tiny(rng)
        E = edge_list(g)
        ld = [M for M in all_matchings(E) if is_maximal(M, E) and is_locally_dominant(M, E)]
        assert len(ld) == 1, (E, ld)
        np.testing.assert_array_equal(oracle.greedy(g).mate, mate_from_pairs(g.n, ld[0]))
        # it is also LD under the paper's literal ">=" rule
        assert is_locally_dominant(ld[0], E, strict=False)


def test_round1_pairs_are_dominant_edges():
    """Fig. 1 / P:46: at M = {} the mutual pairs of the first pointing phase are exactly the
    locally dominant edges (heavier than every adjacent edge)."""
    rng = np.random.default_rng(5)
    for _ in range(200):
        g = _random_tiny(rng, 9)
        E = edge_list(g)
        dom = set()
        for e, we in E.items():
            if all(f == e or (e[0] not in f and e[1] not in f) or
                   (we, max(e), min(e)) > (wf, max(f), min(f)) for f, wf in E.items()):
                dom.add(e)
        # one phase of the frontier iteration == first phase of Alg. 1
        off, col, w = g.offsets, g.col, g.w
        ptr = {}
        for u in range(g.n):
            best = None
            for j in range(off[u], off[u + 1]):
                v = int(col[j])
                if v == u:
                    continue
                k = (float(w[j]), v)
                if best is None or k > best:
                    best = k
            if best is not None:
                ptr[u] = best[1]
        mutual = {(u, v) for u, v in ptr.items() if u < v and ptr.get(v) == u}
        assert mutual == dom


def test_greedy_equals_alg1_many_random():
    """P:52 (global-sort greedy) and Alg. 1, both orders, with heavy ties."""
    rng = np.random.default_rng(7)
    for _ in range(2000):
        g = _random_tiny(rng, 12)
        a = oracle.greedy(g).mate
        b, _ = oracle.ld_seq(g)
        c, _, _ = oracle.ld_frontier(g)
        np.testing.assert_array_equal(a, b)
        np.testing.assert_array_equal(a, c)
        assert oracle.certificate(g, a)[0] == 0


def test_half_approximation_bruteforce():
    """Lemma II.1 / Cor. II.1: w(M) >= OPT/2, OPT by enumeration."""
    rng = np.random.default_rng(3)
    worst = 1.0
    for _ in range(300):
        g = _random_tiny(rng, 10)
        E = edge_list(g)
        opt = brute_opt(E)
        wm = oracle.greedy(g).weight
        if opt > 0:
            worst = min(worst, wm / opt)
            assert wm >= 0.5 * opt - 1e-12
    assert worst < 0.95  # the bound is exercised, not vacuous


def test_half_approximation_networkx_and_predicates():
    """Independent library code: networkx blossom OPT, is_matching, is_maximal_matching."""
    rng = np.random.default_rng(9)
    for trial in range(12):
        if trial % 3 == 0:
            g = graphgen.er(200, 6.0, seed=trial + 1)
        elif trial % 3 == 1:
            g = graphgen.rmat(8, 8, seed=trial + 1)
        else:
            g = graphgen.mesh(14, keep=0.8, seed=trial + 1, weights="paper")
        E = edge_list(g)
        G = nx.Graph()
        G.add_nodes_from(range(g.n))
        for (u, v), w in E.items():
            G.add_edge(u, v, weight=w)
        r = oracle.greedy(g)
        M = {(u, int(v)) for u, v in enumerate(r.mate) if v > u}
        assert nx.is_matching(G, M)
        assert nx.is_maximal_matching(G, M)
        opt = sum(G[u][v]["weight"] for u, v in nx.max_weight_matching(G))
        assert r.weight >= 0.5 * opt - 1e-9
        assert r.weight <= opt + 1e-9
        assert math.isclose(r.weight, sum(E[e] for e in M), rel_tol=1e-12)


# ---------------------------------------------------------------------------- certificate
def test_certificate_rejects_other_maximal_matchings():
    """C(M) holds iff M = M* (R1(iii)): every other maximal matching is rejected."""
    rng = np.random.default_rng(13)
    rejected = 0
    for _ in range(200):
        g = _random_tiny(rng, 8)
        E = edge_list(g)
        star = oracle.greedy(g).mate
        for M in all_matchings(E):
            if not is_maximal(M, E):
                continue
            mate = mate_from_pairs(g.n, M)
            code, _ = oracle.certificate(g, mate)
            if np.array_equal(mate, star):
                assert code == 0
            else:
                assert code == 4
                rejected += 1
    assert rejected > 50


def test_certificate_structural_errors():
    g, mate, _, _ = load_golden("k4.txt")
    bad = mate.copy(); bad[0] = 7
    assert oracle.certificate(g, bad)[0] == 1
    bad = mate.copy(); bad[0] = 0
    assert oracle.certificate(g, bad)[0] == 1
    bad = mate.copy(); bad[0] = 1  # 0->1 but 1->2
    assert oracle.certificate(g, bad)[0] == 2
    g2 = graphgen.from_edges(4, [(0, 1, .5), (2, 3, .5)])
    assert oracle.certificate(g2, np.array([2, 3, 0, 1], np.int32))[0] == 3  # non-edges
    assert oracle.certificate(g2, np.full(4, -1, np.int32))[0] == 4          # not maximal


def test_certificate_accepts_large_greedy():
    g = graphgen.rmat(14, 16, seed=3)
    r = oracle.greedy(g)
    assert oracle.certificate(g, r.mate)[0] == 0
    # flip one matched pair to unmatched -> rejected
    u = int(np.flatnonzero(r.mate >= 0)[0]); v = int(r.mate[u])
    bad = r.mate.copy(); bad[u] = -1; bad[v] = -1
    assert oracle.certificate(g, bad)[0] == 4


# ------------------------------------------------------------------------------- weights
def test_weight_matches_numpy_fp64():
    g = graphgen.er(5000, 12.0, seed=4)
    r = oracle.greedy(g)
    E = edge_list(g)
    ref = math.fsum(E[(u, int(v))] for u, v in enumerate(r.mate) if v > u)
    assert math.isclose(r.weight, ref, rel_tol=1e-13)
    assert math.isclose(oracle.weight(g, r.mate), ref, rel_tol=1e-13)
    assert r.cardinality == int((r.mate >= 0).sum()) // 2


# ---------------------------------------------------------------------------- validation
def test_validate_rules():
    g, _, _, _ = load_golden("k4.txt")
    o, c, w, n, m = g.offsets, g.col, g.w, g.n, g.m
    assert oracle.validate(o, c, w, n, m)[0] == 0
    assert oracle.validate(o, c, w, n, m, level=2)[0] == 0
    o2 = o.copy(); o2[0] = 1
    assert oracle.validate(o2, c, w, n, m)[0] == -1
    o2 = o.copy(); o2[2] = o2[3] + 1
    assert oracle.validate(o2, c, w, n, m)[0] == -1
    assert oracle.validate(o, c, w, n, m + 1)[0] == -1
    c2 = c.copy(); c2[0] = n
    assert oracle.validate(o, c2, w, n, m)[0] == -1
    c2 = c.copy(); c2[0] = -1
    assert oracle.validate(o, c2, w, n, m)[0] == -1
    for bad in (0.0, -0.0, -1.0, float("nan"), float("inf")):
        w2 = w.copy(); w2[3] = bad
        assert oracle.validate(o, c, w2, n, m)[0] == -1, bad
    # asymmetric weight
    w2 = w.copy(); w2[0] = 0.123
    assert oracle.validate(o, c, w2, n, m, level=1)[0] == 0
    assert oracle.validate(o, c, w2, n, m, level=2)[0] == -1
    # duplicate edge with unequal weights (symmetric but ambiguous)
    gd = graphgen.from_edges(2, [(0, 1, .5), (0, 1, .25)])
    assert oracle.validate(gd.offsets, gd.col, gd.w, 2, gd.m, level=2)[0] == -1
    gd = graphgen.from_edges(2, [(0, 1, .5), (0, 1, .5)])
    assert oracle.validate(gd.offsets, gd.col, gd.w, 2, gd.m, level=2)[0] == 0


# ------------------------------------------------------------------------ empirical bands
def test_rmat_round_band():
    """Band, not exact: GAP-kron (Kronecker scale 27) runs 15 iterations; our R-MAT at
    scale 16 should need ~10 pointing phases and clearly fewer than n/2."""
    g = graphgen.rmat(16, 16, seed=1)
    _, ph, fs = oracle.ld_frontier(g)
    assert 6 <= ph <= 20
    assert fs[0] == int((g.degrees() > 0).sum())
    assert all(fs[i + 1] <= fs[i] for i in range(len(fs) - 1)) or ph > 0
