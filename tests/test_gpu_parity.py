"""GPU parity: the CUDA path (through the C ABI) vs the oracle, element by element.

Bar: mate[] bit-exact (integer result); lmatch_stats.rounds equal to the
frontier-driven Alg. 1 oracle's pointing phases; w(M) within 1e-9 relative of the oracle's fp64
Neumaier sum (both sum exact fp32 values in fp64; only the summation order differs).
"""
import math

import numpy as np
import pytest

import graphgen
import oracle
from helpers import golden_names, load_golden

pytestmark = pytest.mark.gpu

WTOL = 1e-9


@pytest.fixture(scope="module")
def lm():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_sc_mandulakgfhs24_b200 as p
    return p


def run_gpu(lm, g, **kw):
    with lm.Matcher(g, **kw) as M:
        mate, st = M.run()
        return mate, st


def check_parity(lm, g, rounds=True, **kw):
    mate, st = run_gpu(lm, g, **kw)
    ref = oracle.greedy(g)
    bad = np.flatnonzero(mate != ref.mate)
    assert bad.size == 0, f"{g.name}: {bad.size} mismatches, first {bad[:5]} gpu={mate[bad[:5]]} ref={ref.mate[bad[:5]]}"
    assert st["cardinality"] == ref.cardinality
    assert math.isclose(st["weight"], ref.weight, rel_tol=WTOL, abs_tol=1e-300)
    if rounds:
        _, ph, _ = oracle.ld_frontier(g)
        assert st["rounds"] == ph, (st["rounds"], ph)
    return mate, st


@pytest.mark.parametrize("name", golden_names())
def test_golden(lm, name):
    g, mate, phases, weight = load_golden(name)
    got, st = run_gpu(lm, g)
    np.testing.assert_array_equal(got, mate)
    assert st["rounds"] == phases
    assert math.isclose(st["weight"], weight, rel_tol=1e-12)


def test_empty_and_trivial(lm):
    g = graphgen.from_edges(7, [])
    mate, st = run_gpu(lm, g)
    assert (mate == -1).all() and st["rounds"] == 0 and st["weight"] == 0
    g = graphgen.from_edges(2, [(0, 1, 0.5)])
    mate, st = run_gpu(lm, g)
    assert list(mate) == [1, 0] and st["rounds"] == 1
    g = graphgen.from_edges(3, [(1, 1, 0.5)])  # only a self-loop
    mate, st = run_gpu(lm, g)
    assert (mate == -1).all() and st["rounds"] == 1


def test_random_tiny_many(lm):
    rng = np.random.default_rng(17)
    for _ in range(60):
        n = int(rng.integers(2, 40))
        g = graphgen.random_small(n, float(rng.choice([.1, .3, .7])), rng,
                                  levels=int(rng.choice([0, 2, 5])) or None)
        check_parity(lm, g)


def test_increasing_path_rounds(lm):
    for n in (2, 3, 17, 64, 301):
        g = graphgen.from_edges(n, [(i, i + 1, float(i + 1)) for i in range(n - 1)])
        _, st = check_parity(lm, g)
        assert st["rounds"] == n // 2 + (n % 2)


@pytest.mark.parametrize("maker", [
    lambda: graphgen.er(1 << 16, 16.0, seed=1),                       # config 1 (PR1 ref)
    lambda: graphgen.er(1 << 14, 16.0, seed=2, weights="paper"),      # 3-decimal ties
    lambda: graphgen.er(5000, 30.0, seed=3, weights="ones"),          # ties only
    lambda: graphgen.rmat(12, 16, seed=1),
    lambda: graphgen.rmat(16, 16, seed=1),
    lambda: graphgen.rmat(18, 16, seed=2),
    lambda: graphgen.rmat(15, 16, seed=4, weights="paper"),
    lambda: graphgen.mesh(256, seed=1),                                # uniform mesh
    lambda: graphgen.mesh(300, keep=0.6, seed=1),                      # road-like
    lambda: graphgen.mesh(64, seed=1, weights="gradient"),             # many rounds (~2*side)
    lambda: graphgen.mesh(97, keep=0.6, seed=5, weights="ones"),
])
def test_synthetic_parity(lm, maker):
    check_parity(lm, maker())


def test_hub_rows_span_many_tiles(lm):
    """Rows much longer than a sweep tile (merged with atomicMax across tiles), plus ragged
    tails: a double star with 20k + 7k leaves and a sprinkling of random edges."""
    rng = np.random.default_rng(3)
    edges = [(0, v, float(np.float32(rng.random() * 0.5 + 0.25))) for v in range(2, 20002)]
    edges += [(1, v, float(np.float32(rng.random()))) for v in range(15000, 22001)]
    for _ in range(5000):
        u, v = rng.integers(2, 22001, size=2)
        if u != v:
            edges.append((int(u), int(v), float(np.float32(1 - rng.random()))))
    g = graphgen.from_edges(22001, edges)
    check_parity(lm, g)
    # a single hub with equal weights: the largest leaf id must win
    g = graphgen.from_edges(9001, [(0, v, 1.0) for v in range(1, 9001)])
    mate, _ = check_parity(lm, g)
    assert mate[0] == 9000


def test_chunked_upload_invariance(lm):
    g = graphgen.rmat(14, 16, seed=7)
    a, _ = run_gpu(lm, g)
    b, _ = run_gpu(lm, g, upload_chunk=1000)
    np.testing.assert_array_equal(a, b)
    np.testing.assert_array_equal(a, oracle.greedy(g).mate)


def test_repeat_runs_deterministic(lm):
    g = graphgen.rmat(15, 16, seed=8)
    with lm.Matcher(g) as M:
        a, s1 = M.run()
        b, s2 = M.run()
    np.testing.assert_array_equal(a, b)
    assert s1["weight"] == s2["weight"] and s1["rounds"] == s2["rounds"]


def test_device_api_and_weight(lm):
    import torch
    g = graphgen.rmat(13, 16, seed=9)
    dev = torch.device("cuda")
    d_off = torch.from_numpy(g.offsets).to(dev)
    d_col = torch.from_numpy(g.col).to(dev)
    d_w = torch.from_numpy(g.w).to(dev)
    M = lm.Matcher.from_device(d_off, d_col, d_w, g.n, g.m, stream=torch.cuda.current_stream())
    d_mate = torch.empty(g.n, dtype=torch.int32, device=dev)
    st = M.run_device(d_mate, stream=torch.cuda.current_stream())
    ref = oracle.greedy(g)
    np.testing.assert_array_equal(d_mate.cpu().numpy(), ref.mate)
    assert math.isclose(st["weight"], ref.weight, rel_tol=WTOL)
    # lmatch_weight on arbitrary mates: the oracle's, and an unmatched-everything mate
    assert math.isclose(M.weight(ref.mate), ref.weight, rel_tol=WTOL)
    assert M.weight(np.full(g.n, -1, np.int32)) == 0.0
    assert math.isclose(lm.lmatch_weight_device(M.h, d_mate), ref.weight, rel_tol=WTOL)
    # a different valid matching: drop one pair
    other = ref.mate.copy()
    u = int(np.flatnonzero(other >= 0)[0]); v = int(other[u])
    other[u] = other[v] = -1
    assert math.isclose(M.weight(other), oracle.weight(g, other), rel_tol=WTOL)
    # invalid mates
    bad = ref.mate.copy(); bad[u] = (v + 1) % g.n
    with pytest.raises(lm.LMatchError):
        M.weight(bad)
    M.close()


def test_reload(lm):
    g1 = graphgen.er(4096, 8.0, seed=1)
    g2 = graphgen.er(4096, 8.0, seed=1, wseed=99)  # same structure, new weights
    with lm.Matcher(g1) as M:
        a, _ = M.run()
        M.reload(g2.offsets, g2.col, g2.w)
        b, _ = M.run()
    np.testing.assert_array_equal(a, oracle.greedy(g1).mate)
    np.testing.assert_array_equal(b, oracle.greedy(g2).mate)


def _same_size_graphs(n=6000, k=2600, seed=5):
    """Two graphs with equal n and m but opposite degree mixes: (a) one hub with k leaves plus a
    sparse ring, (b) a ring plus k evenly spread chords (every row short)."""
    rng = np.random.default_rng(seed)
    wt = lambda: float(np.float32(1 - rng.random()))
    ring = [(i, (i + 1) % n, wt()) for i in range(n)]
    hub = [(0, v, wt()) for v in range(2, 2 + k)]
    chords = [(i, (i + n // 2) % n, wt()) for i in range(1, 1 + k)]
    a, b = graphgen.from_edges(n, ring + hub), graphgen.from_edges(n, ring + chords)
    assert a.m == b.m and a.n == b.n
    return a, b


@pytest.mark.parametrize("round_loop", [0, 3])
def test_reload_different_degree_mix(lm, round_loop):
    """Reload with the same n, m but different rows: bin lists and per-row buffers are re-sized
    (grown) and a captured CUDA graph is rebuilt; results match the oracle each time."""
    a, b = _same_size_graphs()
    with lm.Matcher(b, round_loop=round_loop) as M:
        for g in (b, a, b, a):
            M.reload(g.offsets, g.col, g.w)
            mate, st = M.run()
            np.testing.assert_array_equal(mate, oracle.greedy(g).mate)


def test_validation_errors(lm):
    g, _, _, _ = load_golden("k4.txt")
    o, c, w = g.offsets, g.col, g.w

    def status(o, c, w, level=1, n=None, m=None):
        try:
            M = lm.Matcher(o, c, w, validate_level=level) if n is None else None
            if M is None:
                lm.lmatch_destroy(lm.lmatch_create(o, c, w, n, m))
            else:
                M.close()
            return 0
        except lm.LMatchError as e:
            return e.status

    assert status(o, c, w) == 0
    o2 = o.copy(); o2[0] = 1
    assert status(o2, c, w) == lm.LMATCH_EINVAL
    o2 = o.copy(); o2[2] = o2[3] + 1
    assert status(o2, c, w) == lm.LMATCH_EINVAL
    c2 = c.copy(); c2[0] = 4
    assert status(o, c2, w) == lm.LMATCH_EINVAL
    for bad in (0.0, -0.0, -1.0, float("nan"), float("inf")):
        w2 = w.copy(); w2[1] = bad
        assert status(o, c, w2) == lm.LMATCH_EINVAL, bad
    w2 = w.copy(); w2[0] = 0.123
    assert status(o, c, w2, level=1) == 0
    assert status(o, c, w2, level=2) == lm.LMATCH_EINVAL
    assert status(o, c, w, level=2) == 0
    # oracle agrees on every case above
    assert oracle.validate(o, c, w2, 4, g.m, level=2)[0] == -1


@pytest.mark.slow
def test_full_size_rmat24_certificate(lm):
    """configs[1] at full size: R-MAT scale 24, edge factor 16.  mate[] checked exactly with the
    O(m) certificate (C(M) holds iff M is the unique LD matching) and w(M) against the oracle's
    fp64 weight of the same mate[]."""
    g = graphgen.rmat(24, 16, seed=1)
    mate, st = run_gpu(lm, g)
    code, bad = oracle.certificate(g, mate)
    assert code == 0, (code, bad)
    assert math.isclose(st["weight"], oracle.weight(g, mate), rel_tol=WTOL)
    assert st["cardinality"] == int((mate >= 0).sum()) // 2


def _full_size_from_device(maker):
    """A full-size workload generated on the GPU (the generator is bit-identical to the CPU one,
    tests/test_gpu_graphgen.py), run from the device CSR like bench.py, then brought to the host
    for the oracle's O(m) certificate."""
    import torch
    dg = maker(torch.device("cuda"))
    h = dg.offsets.cpu().numpy(), dg.col.cpu().numpy(), dg.w.cpu().numpy()
    return dg, graphgen.Graph(*h)


@pytest.mark.parametrize("name", ["rmat_s26", "mesh_8192", "road_8192"])
def test_full_size_bench_workloads_certificate(lm, name):
    """The workloads bench.py times, at full size and in its launch configuration (device CSR,
    default round loop): R-MAT scale 26 (the headline, 2.1e9 directed entries) and configs[2],
    the 8192 x 8192 mesh and its road-like thinning.  mate[] is checked exactly by the O(m)
    certificate (C(M) holds iff M is the unique LD matching, R1 iii), w(M) against the
    oracle's fp64 weight of the same mate[]."""
    import torch
    import graphgen.gpu as gg
    makers = {"rmat_s26": lambda d: gg.rmat(26, 16, seed=1, device=d),
              "mesh_8192": lambda d: gg.mesh(8192, seed=1, device=d),
              "road_8192": lambda d: gg.mesh(8192, keep=0.6, seed=1, device=d)}
    dg, g = _full_size_from_device(makers[name])
    M = lm.Matcher.from_device(dg.offsets, dg.col, dg.w, dg.n, dg.m,
                               stream=torch.cuda.current_stream())
    del dg
    torch.cuda.empty_cache()
    mate, st = M.run()
    M.close()
    code, bad = oracle.certificate(g, mate)
    assert code == 0, (code, bad)
    assert math.isclose(st["weight"], oracle.weight(g, mate), rel_tol=WTOL)
    assert st["cardinality"] == int((mate >= 0).sum()) // 2


# ------------------------------------------------------------------ A8 out-of-core streaming
@pytest.mark.parametrize("maker,frac,chunk", [
    (lambda: graphgen.rmat(16, 16, seed=5), 0.3, 4096),
    (lambda: graphgen.rmat(14, 16, seed=6), 0.0, 1024),            # nothing resident
    (lambda: graphgen.er(1 << 15, 16.0, seed=2, weights="paper"), 0.5, 8192),
    (lambda: graphgen.mesh(200, keep=0.6, seed=3), 0.2, 2048),
    (lambda: graphgen.mesh(48, seed=1, weights="gradient"), 0.4, 512),
])
def test_out_of_core_streaming(lm, maker, frac, chunk):
    """hbm_budget forces a resident prefix of ~frac*m entries; the rest is streamed through the
    device ring in round 1 and read zero-copy later.  Result must be bit-identical."""
    g = maker()
    budget = int(8 * g.m * frac) + 2 * 8 * chunk
    mate, st = check_parity(lm, g, hbm_budget_bytes=budget, stream_chunk=chunk)
    assert st["resident_entries"] < g.m
    assert st["bytes_streamed"] == 8 * (g.m - st["resident_entries"])
    assert st["sweep_launches"] >= 2


def _hub_graph(seed=3):
    """Hubs of 20k / 7k / 6k leaves (rows far longer than a stream chunk and than the cache
    fill's 4096-entry CTA threshold), ties among hub edges, and random edges between leaves."""
    rng = np.random.default_rng(seed)
    edges = [(0, v, float(np.float32(rng.random() * 0.5 + 0.25))) for v in range(3, 20003)]
    edges += [(1, v, float(np.float32(rng.random()))) for v in range(15000, 22001)]
    edges += [(2, v, 0.5) for v in range(100, 6100)]
    for _ in range(8000):
        u, v = rng.integers(3, 22001, size=2)
        if u != v:
            edges.append((int(u), int(v), float(np.float32(1 - rng.random()))))
    return graphgen.from_edges(22001, edges)


@pytest.mark.parametrize("maker,frac,chunk", [
    (lambda: graphgen.rmat(16, 16, seed=5), 0.3, 4096),
    (lambda: graphgen.rmat(15, 16, seed=7, weights="paper"), 0.0, 1024),   # ties, nothing resident
    (lambda: graphgen.er(1 << 15, 16.0, seed=2), 0.5, 8192),
    (lambda: graphgen.mesh(200, keep=0.6, seed=3), 0.2, 2048),             # degree <= 4: all cached
    (lambda: graphgen.mesh(48, seed=1, weights="gradient"), 0.4, 512),     # many rounds
    (_hub_graph, 0.1, 1024),                                               # hubs span many chunks
    (_hub_graph, 0.0, 4096),
])
def test_out_of_core_host_cache(lm, maker, frac, chunk):
    """NEXT-1 host-row key cache (top-8 keys of every streamed row, filled in round 1): bit-exact
    with the oracle and identical to the cache-off run; the cache must take rows off the
    zero-copy path, and with the cache off every host frontier row is read from host memory."""
    g = maker()
    budget = int(8 * g.m * frac) + 2 * 8 * chunk
    mate, st = check_parity(lm, g, hbm_budget_bytes=budget, stream_chunk=chunk)
    assert st["resident_entries"] < g.m
    assert st["cache_bytes"] > 0
    mate0, st0 = run_gpu(lm, g, hbm_budget_bytes=budget, stream_chunk=chunk, host_cache=False)
    np.testing.assert_array_equal(mate, mate0)
    assert st0["cache_bytes"] == 0 and st0["cache_rows"] == 0
    assert st["rounds"] == st0["rounds"] and st["weight"] == st0["weight"]
    if st["rounds"] > 1:
        assert st["cache_rows"] > 0


@pytest.mark.parametrize("B", [2, 3, 7])
@pytest.mark.parametrize("cache", [True, False])
def test_paper_style_batches(lm, B, cache):
    """NEXT-2 batch knob (Alg. 2 L3-5): the whole adjacency streamed as B batches
    through the 2-slot ring (nothing resident); bit-exact for every B, with and without the
    host-row cache."""
    for g in (graphgen.rmat(15, 16, seed=8), _hub_graph(5)):
        mate, st = check_parity(lm, g, batches=B, host_cache=cache)
        assert st["resident_entries"] == 0
        assert st["bytes_streamed"] == 8 * g.m
        C = max(512, (g.m // B + 511) // 512 * 512)  # batch size, rounded to the sweep tile
        nb = -(-g.m // C)
        assert st["sweep_launches"] == nb, (st["sweep_launches"], nb)


def test_out_of_core_cache_repeat_and_reload(lm):
    """The cache is refilled by every run (and after a reload with other weights)."""
    g = graphgen.rmat(14, 16, seed=21)
    g2 = graphgen.rmat(14, 16, seed=21, weights="paper")
    assert g2.m == g.m and g2.n == g.n
    budget = 8 * g.m // 4 + 2 * 8 * 1024
    with lm.Matcher(g, hbm_budget_bytes=budget, stream_chunk=1024) as M:
        a, _ = M.run()
        b, _ = M.run()
        np.testing.assert_array_equal(a, b)
        np.testing.assert_array_equal(a, oracle.greedy(g).mate)
        M.reload(g2.offsets, g2.col, g2.w)
        c, _ = M.run()
        np.testing.assert_array_equal(c, oracle.greedy(g2).mate)


def test_out_of_core_weight_and_symmetry(lm):
    g = graphgen.rmat(13, 16, seed=9)
    with lm.Matcher(g, hbm_budget_bytes=8 * g.m // 3, stream_chunk=2048, validate_level=2) as M:
        mate, st = M.run()
        assert st["resident_entries"] < g.m
        ref = oracle.greedy(g)
        np.testing.assert_array_equal(mate, ref.mate)
        assert math.isclose(M.weight(ref.mate), ref.weight, rel_tol=WTOL)


# ------------------------------------------------ A3/A5 partitioned mode (P logical parts, 1 GPU)
@pytest.mark.parametrize("P", [1, 2, 3, 4, 8])
@pytest.mark.parametrize("maker", [
    lambda: graphgen.rmat(15, 16, seed=11),
    lambda: graphgen.er(20000, 8.0, seed=12, weights="paper"),
    lambda: graphgen.mesh(150, keep=0.6, seed=13),
    lambda: graphgen.mesh(40, seed=14, weights="gradient"),
])
def test_partitioned_invariance(lm, P, maker):
    """1-D partition + pointer claims + bitmap allgather (LocalTransport on one GPU): mate[] is
    bit-identical to the oracle for every P (Lemma III.1); rounds are unchanged."""
    import paper_conf_sc_mandulakgfhs24_b200.dist as D
    g = maker()
    mate, res = D.match_partitioned_local(g.offsets, g.col, g.w, P)
    ref = oracle.greedy(g)
    np.testing.assert_array_equal(mate, ref.mate)
    assert res.matched == 2 * ref.cardinality
    assert math.isclose(res.weight, ref.weight, rel_tol=WTOL)
    assert res.rounds == oracle.ld_frontier(g)[1]
    if P > 1:
        assert res.exchanged_claims > 0


def test_partitioned_hub_rows(lm):
    import paper_conf_sc_mandulakgfhs24_b200.dist as D
    g = graphgen.from_edges(9001, [(0, v, 1.0) for v in range(1, 9001)] +
                            [(v, v + 1, 0.5) for v in range(100, 8000, 7)])
    mate, res = D.match_partitioned_local(g.offsets, g.col, g.w, 4)
    np.testing.assert_array_equal(mate, oracle.greedy(g).mate)


# --------------------------------------------- round loop: CUDA graph (default) vs host-driven
@pytest.mark.parametrize("maker", [
    lambda: graphgen.rmat(14, 16, seed=21),
    lambda: graphgen.rmat(17, 16, seed=24, weights="paper"),
    lambda: graphgen.mesh(64, seed=22, weights="gradient"),     # ~130 rounds inside the graph
    lambda: graphgen.from_edges(5, []),                         # no work: the WHILE never runs
    lambda: graphgen.from_edges(301, [(i, i + 1, float(i + 1)) for i in range(300)]),
])
def test_round_loop_modes_identical(lm, maker):
    g = maker()
    ref = oracle.greedy(g).mate
    ph = oracle.ld_frontier(g)[1]
    out = [run_gpu(lm, g, round_loop=mode, timing=True) for mode in (0, 1, 2, 3)]
    for mate, st in out:
        np.testing.assert_array_equal(mate, ref)
        assert st["rounds"] == ph
        assert st["weight"] == out[0][1]["weight"]
        assert st["frontier_total"] == out[0][1]["frontier_total"]
        if g.m:
            assert st["ms_sweep"] > 0


def test_graph_replay_and_round_log(lm):
    """The instantiated graph is replayed across runs; the per-round log matches the oracle's
    frontier sizes (Fig. 8 analogue)."""
    g = graphgen.rmat(15, 16, seed=23)
    _, ph, fs = oracle.ld_frontier(g)
    with lm.Matcher(g) as M:
        for _ in range(3):
            mate, st = M.run()
            np.testing.assert_array_equal(mate, oracle.greedy(g).mate)
            log = lm.lmatch_round_log(M.h)
            assert log.shape[0] == st["rounds"] == ph
            np.testing.assert_array_equal(log[:, 0], fs)


# ------------------------------------------------------- self-loops (ignored) at ingest
def _loopy_graph(seed):
    """Random graph whose self-loops carry the LARGEST weights (they would win every row if not
    ignored): short rows (< 32 entries), warp-width rows (32..512) and hub rows crossing many
    512-entry sweep tiles all get a loop."""
    rng = np.random.default_rng(seed)
    n = 6000
    edges = []
    for u in range(n):
        deg = int(rng.choice([1, 3, 40, 300])) if u % 97 else 0
        for v in rng.integers(0, n, size=deg):
            if int(v) != u:
                edges.append((u, int(v), float(np.float32(0.5 * rng.random() + 0.01))))
    for v in range(1, n):  # hub 0 spans many tiles
        if v % 3:
            edges.append((0, v, float(np.float32(0.5 * rng.random() + 0.01))))
    for u in rng.choice(n, size=n // 2, replace=False):
        edges.append((int(u), int(u), 2.0 + float(rng.random())))
    edges.append((0, 0, 9.0))
    return graphgen.from_edges(n, edges)


@pytest.mark.parametrize("mode", ["resident", "streamed", "partitioned"])
def test_self_loops_ignored(lm, mode):
    g = _loopy_graph(21)
    ref = oracle.greedy(g)
    assert ref.cardinality > 0
    if mode == "resident":
        check_parity(lm, g)
        check_parity(lm, g, upload_chunk=777)
    elif mode == "streamed":
        check_parity(lm, g, hbm_budget_bytes=8 * g.m // 3 + 2 * 8 * 1024, stream_chunk=1024)
    else:
        import paper_conf_sc_mandulakgfhs24_b200.dist as D
        for P in (2, 3):
            mate, res = D.match_partitioned_local(g.offsets, g.col, g.w, P)
            np.testing.assert_array_equal(mate, ref.mate)


# ------------------------------------------------- A7 in-place pruning (opt-in)
@pytest.mark.parametrize("maker", [
    lambda: graphgen.rmat(14, 16, seed=31),
    lambda: graphgen.rmat(16, 16, seed=32, weights="paper"),    # 3-decimal ties
    lambda: graphgen.er(1 << 14, 16.0, seed=33),
    lambda: graphgen.er(3000, 40.0, seed=34, weights="ones"),   # ties only; 32-lane rows
    lambda: graphgen.mesh(128, seed=35),
    lambda: graphgen.mesh(200, keep=0.6, seed=36),
    lambda: graphgen.mesh(48, seed=37, weights="gradient"),     # ~100 rounds, persistent kernel
    lambda: _loopy_graph(38),                                   # zeroed self-loop keys are pruned
])
@pytest.mark.parametrize("round_loop", [0, 1, 2, 3])
def test_pruning_parity_and_reentrant(lm, maker, round_loop):
    """Pruning removes only entries whose neighbour is matched (never available again, R3), so
    mate[], the rounds and w(M) equal the oracle's.  The rows stay permutations of themselves,
    so repeated runs on the same handle (whose round-1 sweep reads whole rows again) stay exact,
    and the later rounds scan no more entries than without pruning."""
    g = maker()
    ref = oracle.greedy(g)
    ph = oracle.ld_frontier(g)[1]
    _, base = run_gpu(lm, g, round_loop=round_loop)
    with lm.Matcher(g, prune=True, round_loop=round_loop) as M:
        for _ in range(3):
            mate, st = M.run()
            np.testing.assert_array_equal(mate, ref.mate)
            assert st["rounds"] == ph
            assert math.isclose(st["weight"], ref.weight, rel_tol=WTOL)
            assert st["entries_swept"] <= base["entries_swept"]
            assert st["frontier_total"] == base["frontier_total"]


def test_pruning_keeps_rows_permutations(lm):
    """After pruned runs, a fresh non-pruning run on the SAME handle's adjacency -- reached by
    reading back w(M) of arbitrary mates through lmatch_weight, which looks edges up in the
    handle's rows -- still finds every edge: the multiset of each row is unchanged."""
    g = graphgen.rmat(13, 16, seed=39)
    ref = oracle.greedy(g)
    rng = np.random.default_rng(4)
    with lm.Matcher(g, prune=True) as M:
        for _ in range(2):
            mate, _ = M.run()
            np.testing.assert_array_equal(mate, ref.mate)
        # a different valid matching: every edge lookup must still succeed in the permuted rows
        E = [(u, int(g.col[j])) for u in range(g.n) for j in range(g.offsets[u], g.offsets[u + 1])
             if u < g.col[j]]
        rng.shuffle(E)
        other = np.full(g.n, -1, np.int32)
        for u, v in E[:3000]:
            if other[u] < 0 and other[v] < 0:
                other[u], other[v] = v, u
        assert math.isclose(M.weight(other), oracle.weight(g, other), rel_tol=WTOL)


# ---------------------------------------------------------- NEXT-4: the Suitor algorithm
def check_suitor(lm, g):
    """Suitor under the strict order R1 reaches the same unique matching (mate[] bit-exact,
    w(M) within 1e-9); its pass count is its own, so rounds are not compared."""
    return check_parity(lm, g, rounds=False, algorithm="suitor")


@pytest.mark.parametrize("name", golden_names())
def test_suitor_golden(lm, name):
    g, mate, _, weight = load_golden(name)
    got, st = run_gpu(lm, g, algorithm="suitor")
    np.testing.assert_array_equal(got, mate)
    assert math.isclose(st["weight"], weight, rel_tol=1e-12)


def test_suitor_random_tiny_and_paths(lm):
    rng = np.random.default_rng(23)
    for _ in range(60):
        n = int(rng.integers(2, 40))
        g = graphgen.random_small(n, float(rng.choice([.1, .3, .7])), rng,
                                  levels=int(rng.choice([0, 2, 5])) or None)
        check_suitor(lm, g)
    for n in (2, 3, 17, 301):
        check_suitor(lm, graphgen.from_edges(n, [(i, i + 1, float(i + 1)) for i in range(n - 1)]))
    check_suitor(lm, graphgen.from_edges(7, []))


@pytest.mark.parametrize("maker", [
    lambda: graphgen.er(1 << 16, 16.0, seed=1),
    lambda: graphgen.er(5000, 30.0, seed=3, weights="ones"),
    lambda: graphgen.rmat(16, 16, seed=1),
    lambda: graphgen.rmat(15, 16, seed=4, weights="paper"),
    lambda: graphgen.mesh(256, seed=1),
    lambda: graphgen.mesh(300, keep=0.6, seed=1),
    lambda: graphgen.mesh(128, seed=1, weights="gradient"),
    lambda: _hub_graph(4),
])
def test_suitor_synthetic(lm, maker):
    check_suitor(lm, maker())


def test_suitor_repeat_reload_and_rmat24(lm):
    """Repeated runs and a reload on one Suitor handle; configs[1] at full size against the O(m)
    certificate and the LD path's result."""
    g = graphgen.rmat(14, 16, seed=21)
    g2 = graphgen.rmat(14, 16, seed=21, weights="paper")
    with lm.Matcher(g, algorithm="suitor") as M:
        a, _ = M.run()
        b, _ = M.run()
        np.testing.assert_array_equal(a, b)
        np.testing.assert_array_equal(a, oracle.greedy(g).mate)
        M.reload(g2.offsets, g2.col, g2.w)
        c, _ = M.run()
        np.testing.assert_array_equal(c, oracle.greedy(g2).mate)
    g = graphgen.rmat(24, 16, seed=1)
    mate, st = run_gpu(lm, g, algorithm="suitor")
    code, bad = oracle.certificate(g, mate)
    assert code == 0, (code, bad)
    ref, _ = run_gpu(lm, g)
    np.testing.assert_array_equal(mate, ref)


@pytest.mark.parametrize("round_loop", [0, 1, 2, 3])
def test_hybrid_tail(lm, round_loop):
    """algorithm 2: the LD iteration stops after 32 pointing phases and Suitor finishes on the
    graph without the vertices matched so far.  Many-round graphs take the tail and stay
    bit-exact; graphs that finish within 32 phases are untouched (same phase count as Alg. 1)."""
    for g in (graphgen.mesh(64, seed=1, weights="gradient"),       # ~2*side phases
              graphgen.from_edges(301, [(i, i + 1, float(i + 1)) for i in range(300)]),
              graphgen.mesh(90, keep=0.6, seed=2, weights="gradient")):
        mate, st = check_parity(lm, g, rounds=False, algorithm="hybrid", round_loop=round_loop)
        assert st["tail_passes"] > 0
        assert st["rounds"] == 32
    for g in (graphgen.rmat(16, 16, seed=1), graphgen.mesh(200, seed=3)):
        mate, st = check_parity(lm, g, algorithm="hybrid", round_loop=round_loop)
        assert st["tail_passes"] == 0


# ---------------------------------------------------------- NEXT-3: sorted adjacency + cursor
def check_sorted(lm, g, rounds=True):
    """algorithm 3 computes Alg. 1's pointers (heaviest unmatched neighbour, R1 order) from rows
    sorted once by key, so mate[] is bit-exact and the pointing-phase count is Alg. 1's."""
    return check_parity(lm, g, rounds=rounds, algorithm="sorted")


@pytest.mark.parametrize("name", golden_names())
def test_sorted_golden(lm, name):
    g, mate, _, weight = load_golden(name)
    got, st = run_gpu(lm, g, algorithm="sorted")
    np.testing.assert_array_equal(got, mate)
    assert math.isclose(st["weight"], weight, rel_tol=1e-12)


def test_sorted_random_tiny_and_paths(lm):
    rng = np.random.default_rng(29)
    for _ in range(60):
        n = int(rng.integers(2, 40))
        g = graphgen.random_small(n, float(rng.choice([.1, .3, .7])), rng,
                                  levels=int(rng.choice([0, 2, 5])) or None)
        check_sorted(lm, g)
    for n in (2, 3, 17, 301):
        check_sorted(lm, graphgen.from_edges(n, [(i, i + 1, float(i + 1)) for i in range(n - 1)]))
    check_sorted(lm, graphgen.from_edges(7, []))
    # self-loops (zero keys after ingest) sort to the row end and are never pointed at
    check_sorted(lm, graphgen.from_edges(4, [(0, 0, 9.0), (0, 1, 1.0), (1, 1, 5.0), (2, 3, 2.0)]))


@pytest.mark.parametrize("maker", [
    lambda: graphgen.er(1 << 16, 16.0, seed=1),
    lambda: graphgen.er(5000, 30.0, seed=3, weights="ones"),
    lambda: graphgen.rmat(16, 16, seed=1),
    lambda: graphgen.rmat(15, 16, seed=4, weights="paper"),
    lambda: graphgen.mesh(256, seed=1),
    lambda: graphgen.mesh(300, keep=0.6, seed=1),
    lambda: graphgen.mesh(128, seed=1, weights="gradient"),
    lambda: _hub_graph(4),
    lambda: _loopy_graph(38),
])
def test_sorted_synthetic(lm, maker):
    check_sorted(lm, maker())


def test_sorted_repeat_reload_weight_and_rmat24(lm):
    """The sort runs once per loaded graph (ms_sort > 0 on the first run only, again after a
    reload); lmatch_weight still reads the permuted rows correctly; configs[1] at full size
    against the O(m) certificate and the LD path's result."""
    g = graphgen.rmat(14, 16, seed=21)
    g2 = graphgen.rmat(14, 16, seed=21, weights="paper")
    with lm.Matcher(g, algorithm="sorted", timing=1) as M:
        a, sa = M.run()
        b, sb = M.run()
        np.testing.assert_array_equal(a, b)
        np.testing.assert_array_equal(a, oracle.greedy(g).mate)
        assert sa["ms_sort"] > 0 and sb["ms_sort"] == 0
        assert math.isclose(M.weight(a), oracle.weight(g, a), rel_tol=WTOL)
        M.reload(g2.offsets, g2.col, g2.w)
        c, sc = M.run()
        assert sc["ms_sort"] > 0
        np.testing.assert_array_equal(c, oracle.greedy(g2).mate)
    g = graphgen.rmat(24, 16, seed=1)
    mate, st = run_gpu(lm, g, algorithm="sorted")
    code, bad = oracle.certificate(g, mate)
    assert code == 0, (code, bad)
    ref, sref = run_gpu(lm, g)
    np.testing.assert_array_equal(mate, ref)
    assert st["rounds"] == sref["rounds"]
    assert st["entries_swept"] < sref["entries_swept"]


def test_sorted_rejects_out_of_core(lm):
    """algorithm 3 needs the whole adjacency resident (it sorts it in place): an out-of-core
    handle's run fails loudly with EINVAL instead of falling back."""
    g = graphgen.rmat(12, 16, seed=2)
    with lm.Matcher(g, algorithm="sorted", hbm_budget_bytes=8 * g.m // 2, stream_chunk=1024) as M:
        with pytest.raises(lm.LMatchError):
            M.run()


def test_extreme_weights_key_order(lm):
    """Float subnormal, smallest-normal and near-FLT_MAX weights mixed with ordinary ones, in a
    hub row that spans several sweep tiles, warp-reduced rows and lane-reduced rows: the sweep's
    FP64-pipe key max (kmax64) must order them exactly as the u64 keys."""
    rng = np.random.default_rng(17)
    fi = np.finfo(np.float32)
    pool = np.array([fi.smallest_subnormal, 3 * fi.smallest_subnormal, 1e-40, fi.tiny, 2 * fi.tiny,
                     1e-30, 0.001, 0.5, 0.999, 1.0, 7.0, 1e30, fi.max / 2, fi.max], dtype=np.float32)
    n = 4000
    edges = [(0, v, float(pool[v % len(pool)])) for v in range(1, 1800)]       # hub: > 3 tiles
    for u in range(1800, 2400):                                                 # 40-entry rows
        for d in range(1, 21):
            edges.append((u, 1800 + (u - 1800 + 37 * d) % 600, float(pool[rng.integers(len(pool))])))
    for _ in range(6000):                                                       # short rows
        u, v = rng.integers(2400, n, size=2)
        edges.append((int(u), int(v), float(pool[rng.integers(len(pool))])))
    uniq = {}
    for u, v, w in edges:
        if u != v:
            uniq.setdefault((min(u, v), max(u, v)), w)   # a simple graph: one weight per edge
    g = graphgen.from_edges(n, [(u, v, w) for (u, v), w in uniq.items()])
    check_parity(lm, g)
    check_parity(lm, g, round_loop=1)


@pytest.mark.parametrize("kw", [dict(), dict(round_loop=1), dict(round_loop=2), dict(algorithm="hybrid"),
                                dict(algorithm="suitor")])
def test_crossing_rows_repeat_runs(lm, kw):
    """Tile-crossing rows merge their partial maxima into best[] with atomicMax, and best[] is not
    re-zeroed between runs (LM_XROW_RESET = 0): a run starts from the previous run's final
    pointers, each 0 or a key of the vertex's own row.  Overlapping hubs spanning several tiles
    (their final pointers far below their maxima) and random short rows, every round-loop mode and
    algorithm that runs the sweep: every one of three runs on one handle equals the oracle."""
    rng = np.random.default_rng(21)
    n = 12000
    edges = []
    for h, (lo, hi) in enumerate([(50, 4050), (2000, 7000), (6000, 11990)]):
        for v in range(lo, hi):
            edges.append((h, v, float(np.float32(rng.random() * 0.9 + 0.05))))
    for _ in range(20000):
        u, v = rng.integers(3, n, size=2)
        if u != v:
            edges.append((int(u), int(v), float(np.float32(rng.random()))))
    uniq = {}
    for u, v, w in edges:
        uniq.setdefault((min(u, v), max(u, v)), w)
    g = graphgen.from_edges(n, [(u, v, w) for (u, v), w in uniq.items()])
    ref = oracle.greedy(g)
    with lm.Matcher(g, **kw) as M:
        for _ in range(3):
            mate, st = M.run()
            np.testing.assert_array_equal(mate, ref.mate)
            assert math.isclose(st["weight"], ref.weight, rel_tol=WTOL)
