"""GPU checks of the boundary contract (include/lmatch.h) beyond plain parity:

* reload into a handle whose new graph has EMPTY rows where the old one had edges (every
  algorithm and partition handles): no pointer of the old graph may survive;
* the round cap: a cap that stops the iteration with a non-empty frontier returns
  LMATCH_EROUNDS (never OK with a non-maximal matching);
* validate_level 2: a repeated edge with unequal weights is rejected exactly as the oracle's
  validate rejects it (SURVEY 8(b) EINVAL rule; "simple undirected graph");
* algorithm 3 sorts rows in chunks: tiny chunk sizes run the chunking (rows spanning several
  chunk-sized runs, a row longer than a chunk) and stay bit-exact.
"""
import math

import numpy as np
import pytest

import graphgen
import oracle
from helpers import load_golden

pytestmark = pytest.mark.gpu
WTOL = 1e-9


@pytest.fixture(scope="module")
def lm():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_sc_mandulakgfhs24_b200 as p
    return p


def _graph_with_isolated(n=4096, seed=3, every=3):
    """ER-like graph on n vertices where every `every`-th vertex is isolated (an empty row)."""
    rng = np.random.default_rng(seed)
    alive = np.array([v for v in range(n) if v % every], dtype=np.int64)
    edges = set()
    while len(edges) < 4 * n:
        u, v = rng.choice(alive, 2)
        if u != v:
            edges.add((min(u, v), max(u, v)))
    E = [(u, v, float(np.float32(1 - rng.random()))) for (u, v) in sorted(edges)]
    return graphgen.from_edges(n, E)


def _relabel(g, perm):
    """The same graph with vertex v renamed perm[v] (degree multiset preserved)."""
    E = []
    for u in range(g.n):
        for j in range(g.offsets[u], g.offsets[u + 1]):
            v = int(g.col[j])
            if u < v:
                E.append((int(perm[u]), int(perm[v]), float(g.w[j])))
    return graphgen.from_edges(g.n, E)


def _reload_pair(n=4096, parts=(0, 2048, 4096)):
    """Two graphs with equal n and equal per-part entry counts for the bounds `parts`; the second
    renames vertices inside each part, so rows that were non-empty become empty and vice versa."""
    a = _graph_with_isolated(n)
    rng = np.random.default_rng(11)
    perm = np.arange(n)
    for p in range(len(parts) - 1):
        lo, hi = parts[p], parts[p + 1]
        perm[lo:hi] = lo + rng.permutation(hi - lo)
    b = _relabel(a, perm)
    assert a.m == b.m
    for p in range(len(parts) - 1):
        lo, hi = parts[p], parts[p + 1]
        assert a.offsets[hi] - a.offsets[lo] == b.offsets[hi] - b.offsets[lo]
    newly_empty = (np.diff(b.offsets) == 0) & (np.diff(a.offsets) > 0)
    assert newly_empty.sum() > 100
    return a, b


@pytest.mark.parametrize("algorithm", ["ld", "suitor", "hybrid", "sorted"])
def test_reload_rows_become_empty(lm, algorithm):
    """Regression (round-1 verdict): best[] of rows that are empty after a reload must not keep
    the previous graph's pointers (Suitor's first pass and the partition claims read best[] of
    every vertex)."""
    a, b = _reload_pair()
    with lm.Matcher(a, algorithm=algorithm) as M:
        for g in (a, b, a, b):
            M.reload(g.offsets, g.col, g.w)
            mate, st = M.run()
            ref = oracle.greedy(g)
            np.testing.assert_array_equal(mate, ref.mate)
            assert math.isclose(st["weight"], ref.weight, rel_tol=WTOL)


@pytest.mark.parametrize("exchange", ["transport", "p2p"])
def test_partition_reload_rows_become_empty(lm, exchange):
    import paper_conf_sc_mandulakgfhs24_b200.dist as D
    bounds = np.array([0, 2048, 4096], dtype=np.int64)
    a, b = _reload_pair(parts=tuple(bounds))
    parts = []
    for p in range(2):
        lo, lc, lw = D.local_csr(a.offsets, a.col, a.w, int(bounds[p]), int(bounds[p + 1]))
        parts.append(D.LibPart(lo, lc, lw, int(bounds[p]), a.n, bounds, p))
    if exchange == "p2p":
        D.connect_p2p_local(parts)
    try:
        for g in (a, b, a, b):
            for p, part in enumerate(parts):
                part.reload(*D.local_csr(g.offsets, g.col, g.w, int(bounds[p]), int(bounds[p + 1])))
            if exchange == "p2p":
                res = D.run_parts_p2p(parts, D.barrier_events(parts), D.LocalTransport(2))
            else:
                res = D.run_parts(parts, D.LocalTransport(2))
            mate = np.concatenate([m.cpu().numpy() for m in res.mates])
            np.testing.assert_array_equal(mate, oracle.greedy(g).mate)
    finally:
        for part in parts:
            part.close()


@pytest.mark.parametrize("algorithm,round_loop", [("ld", 0), ("ld", 1), ("ld", 2), ("ld", 3),
                                                  ("suitor", 0), ("sorted", 0)])
def test_round_cap_returns_erounds(lm, algorithm, round_loop):
    """A caller-set max_rounds that stops a non-empty frontier is an error (LMATCH_EROUNDS), for
    every algorithm and round-loop mode; the default cap always completes."""
    g = graphgen.mesh(64, seed=1, weights="gradient")  # ~2*side pointing phases
    with lm.Matcher(g, algorithm=algorithm, round_loop=round_loop, max_rounds=3) as M:
        with pytest.raises(lm.LMatchError) as ei:
            M.run()
        assert ei.value.status == lm.LMATCH_EROUNDS
    with lm.Matcher(g, algorithm=algorithm, round_loop=round_loop) as M:
        mate, _ = M.run()
        np.testing.assert_array_equal(mate, oracle.greedy(g).mate)
    # a cap exactly at the phase count Alg. 1 needs is enough
    _, phases, _ = oracle.ld_frontier(g)
    if algorithm == "ld":
        with lm.Matcher(g, round_loop=round_loop, max_rounds=phases) as M:
            mate, st = M.run()
            assert st["rounds"] == phases
            np.testing.assert_array_equal(mate, oracle.greedy(g).mate)


def test_round_cap_out_of_core(lm):
    g = graphgen.mesh(64, seed=1, weights="gradient")
    with lm.Matcher(g, max_rounds=4, hbm_budget_bytes=8 * g.m // 2, stream_chunk=1024) as M:
        with pytest.raises(lm.LMatchError) as ei:
            M.run()
        assert ei.value.status == lm.LMATCH_EROUNDS


def _status(lm, o, c, w, level):
    try:
        lm.Matcher(o, c, w, validate_level=level).close()
        return 0
    except lm.LMatchError as e:
        return e.status


def _with_duplicate(g, u, v, w2):
    """g with the pair (u, v) listed a second time in BOTH rows (so the graph stays symmetric
    as a multiset) with weight w2."""
    E = []
    for a in range(g.n):
        for j in range(g.offsets[a], g.offsets[a + 1]):
            b = int(g.col[j])
            if a < b:
                E.append((a, b, float(g.w[j])))
    E.append((u, v, w2))
    return graphgen.from_edges(g.n, E)


def test_validation_level2_duplicates(lm):
    g, _, _, _ = load_golden("k4.txt")
    u, v = 0, 3
    j = int(np.flatnonzero(g.col[g.offsets[u]:g.offsets[u + 1]] == v)[0]) + int(g.offsets[u])
    w_uv = float(g.w[j])
    # symmetric duplicate with an unequal weight: the multiset hash cannot see it, the exact
    # duplicate check must (and the oracle agrees)
    d = _with_duplicate(g, u, v, 0.25)
    assert oracle.validate(d.offsets, d.col, d.w, d.n, d.m, level=2)[0] == -1
    assert _status(lm, d.offsets, d.col, d.w, 2) == lm.LMATCH_EINVAL
    assert _status(lm, d.offsets, d.col, d.w, 1) == 0
    # a repeated edge with the SAME weight is harmless (same key): accepted, same matching
    e = _with_duplicate(g, u, v, w_uv)
    assert oracle.validate(e.offsets, e.col, e.w, e.n, e.m, level=2)[0] == 0
    assert _status(lm, e.offsets, e.col, e.w, 2) == 0
    with lm.Matcher(e, validate_level=2) as M:
        mate, _ = M.run()
    np.testing.assert_array_equal(mate, oracle.greedy(g).mate)
    # a duplicated self-loop with unequal weights is a repeated (u,u) too
    s = graphgen.from_edges(4, [(0, 1, .5), (2, 3, .5), (1, 1, .3), (1, 1, .4)])
    assert oracle.validate(s.offsets, s.col, s.w, s.n, s.m, level=2)[0] == -1
    assert _status(lm, s.offsets, s.col, s.w, 2) == lm.LMATCH_EINVAL


def test_validation_level2_duplicates_large_and_out_of_core(lm):
    """Rows spread over several duplicate-check chunks (R-MAT s16) and an out-of-core handle
    (rows read through the host part): valid graphs pass, one planted duplicate fails."""
    g = graphgen.rmat(16, 16, seed=7)
    assert _status(lm, g.offsets, g.col, g.w, 2) == 0
    for log2 in (6, 12):  # many duplicate-check chunks (sort_chunk_log2 caps them)
        lm.Matcher(g, validate_level=2, sort_chunk_log2=log2).close()
    deg = np.diff(g.offsets)
    u = int(np.flatnonzero(deg > 3)[-1])  # a late row
    v = int(g.col[g.offsets[u]])
    d = _with_duplicate(g, u, v, 0.5 if float(g.w[g.offsets[u]]) != 0.5 else 0.25)
    assert _status(lm, d.offsets, d.col, d.w, 2) == lm.LMATCH_EINVAL
    with pytest.raises(lm.LMatchError):
        lm.Matcher(d, validate_level=2, sort_chunk_log2=8)
    for x, want in ((g, 0), (d, lm.LMATCH_EINVAL)):
        try:
            lm.Matcher(x, validate_level=2, hbm_budget_bytes=8 * x.m // 3, stream_chunk=4096).close()
            got = 0
        except lm.LMatchError as ex:
            got = ex.status
        assert got == want


@pytest.mark.parametrize("log2", [4, 7, 10])
@pytest.mark.parametrize("maker", [
    lambda: graphgen.rmat(14, 16, seed=3),
    lambda: graphgen.er(5000, 30.0, seed=3, weights="ones"),
    lambda: graphgen.from_edges(3000, [(0, v, float(np.float32(1.0 / (1 + v % 97)))) for v in range(1, 3000)]
                                + [(v, v + 1, 0.5) for v in range(1, 2999)]),
])
def test_sorted_chunked_sort(lm, maker, log2):
    """algorithm 3 with rows sorted in chunks of 2^log2 entries: many chunks, rows longer than a
    chunk (the hub), same result and Alg. 1 phase count as the oracle."""
    g = maker()
    with lm.Matcher(g, algorithm="sorted", sort_chunk_log2=log2) as M:
        mate, st = M.run()
    ref = oracle.greedy(g)
    np.testing.assert_array_equal(mate, ref.mate)
    assert math.isclose(st["weight"], ref.weight, rel_tol=WTOL)
    _, ph, _ = oracle.ld_frontier(g)
    assert st["rounds"] == ph


def test_sort_chunk_option_range(lm):
    g = graphgen.rmat(8, 8, seed=1)
    for bad in (3, 31, -1):
        with pytest.raises(lm.LMatchError) as ei:
            lm.Matcher(g, algorithm="sorted", sort_chunk_log2=bad)
        assert ei.value.status == lm.LMATCH_EINVAL


@pytest.mark.parametrize("round_loop", [0, 1, 2, 3])
@pytest.mark.parametrize("maker", [
    lambda: graphgen.rmat(16, 16, seed=11),
    lambda: graphgen.er(30000, 12.0, seed=4, weights="paper"),
    lambda: graphgen.mesh(200, keep=0.6, seed=5),
    lambda: graphgen.from_edges(5000, [(0, v, float(np.float32(1.0 / (1 + v % 61)))) for v in range(1, 5000)]
                                + [(v, v + 1, float(np.float32(0.3 + (v % 7) / 10))) for v in range(1, 4999)]),
])
def test_key_cache_identity(lm, maker, round_loop):
    """The resident key cache (opts.key_cache; rows' 4 largest keys from the round-1 sweep, tile-
    crossing rows merged) decides most pointers of rounds >= 2 without scanning the row: same
    mate[], same pointing phases as Alg. 1 and as the cache-off path, fewer entries scanned."""
    g = maker()
    ref = oracle.greedy(g)
    _, ph, _ = oracle.ld_frontier(g)
    out = {}
    for kc in (True, False):
        with lm.Matcher(g, key_cache=kc, round_loop=round_loop) as M:
            mate, st = M.run()
            mate2, st2 = M.run()
        np.testing.assert_array_equal(mate, ref.mate)
        np.testing.assert_array_equal(mate2, ref.mate)
        assert st["rounds"] == ph and st2["rounds"] == ph
        assert math.isclose(st["weight"], ref.weight, rel_tol=WTOL)
        out[kc] = st
    if ph > 1:
        assert out[True]["cache_rows"] > 0
        assert out[True]["entries_swept"] <= out[False]["entries_swept"]
    assert out[False]["cache_rows"] == 0


@pytest.mark.parametrize("maker,frac", [
    (lambda: graphgen.rmat(16, 16, seed=5), 0.2),
    (lambda: graphgen.er(1 << 15, 24.0, seed=2, weights="paper"), 0.1),
    (lambda: graphgen.from_edges(4000, [(0, v, float(np.float32(1.0 / (1 + v % 97)))) for v in range(1, 4000)]
                                 + [(v, v + 1, 0.5) for v in range(1, 3999)]), 0.0),
])
def test_out_of_core_residual_rows(lm, maker, frac):
    """NEXT-1 residual rows (opts.residual_mb): host rows that are rescanned are also copied into
    HBM, and later rounds and runs scan that copy.  Bit-identical across repeated runs (the copies
    persist) and a reload (they are dropped), fewer host entries read once rows are resident."""
    g = maker()
    ref = oracle.greedy(g)
    _, ph, _ = oracle.ld_frontier(g)
    chunk = 1024
    budget = int(8 * g.m * frac) + 2 * 8 * chunk
    with lm.Matcher(g, hbm_budget_bytes=budget, stream_chunk=chunk, residual_mb=4) as M:
        stats = []
        for _ in range(3):
            mate, st = M.run()
            np.testing.assert_array_equal(mate, ref.mate)
            assert st["rounds"] == ph
            assert math.isclose(st["weight"], ref.weight, rel_tol=WTOL)
            stats.append(st)
        M.reload(g.offsets, g.col, g.w)
        mate, st = M.run()
        np.testing.assert_array_equal(mate, ref.mate)
    if stats[0]["host_entries_read"] > 0:
        assert stats[2]["residual_rows"] > 0
        assert stats[2]["host_entries_read"] < stats[0]["host_entries_read"]


@pytest.mark.parametrize("round_loop", [0, 2, 3])
@pytest.mark.parametrize("maker", [
    lambda: graphgen.mesh(96, seed=1, weights="gradient"),           # ~2*side phases
    lambda: graphgen.mesh(120, keep=0.6, seed=2, weights="gradient"),
    lambda: graphgen.from_edges(3001, [(i, i + 1, float(i + 1)) for i in range(3000)]),  # 1500 phases
    lambda: graphgen.rmat(15, 16, seed=8),
    lambda: graphgen.from_edges(600, [(i, i + 1, float(i + 1)) for i in range(599)] + [(i, i + 1, float(i + 1)) for i in range(599)]),
])
def test_push_frontier(lm, maker, round_loop):
    """A6 push frontier (opts.frontier): in the persistent-kernel rounds the next frontier is built
    from the rows of the newly matched vertices once the live list is much longer than the
    frontier.  Same mate[] and the same pointing phases as Alg. 1 and as pull-only; many-round
    graphs actually switch to push.  (The last graph lists every edge twice: a pushed vertex is
    claimed once.)"""
    g = maker()
    ref = oracle.greedy(g)
    _, ph, _ = oracle.ld_frontier(g)
    res = {}
    for fr in ("push", "auto", "pull"):
        with lm.Matcher(g, round_loop=round_loop, frontier=fr) as M:
            for _ in range(2):
                mate, st = M.run()
                np.testing.assert_array_equal(mate, ref.mate)
                assert st["rounds"] == ph
                assert math.isclose(st["weight"], ref.weight, rel_tol=WTOL)
            res[fr] = M.push_rounds()
    assert res["pull"] == 0
    if ph > 100:
        assert res["push"] > 0  # (auto waits for a live list of 2^20 vertices)
