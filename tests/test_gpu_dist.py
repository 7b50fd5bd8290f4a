"""The library-owned multi-GPU driver (lmatch_partition / lmatch_create_dist / lmatch_run_dist;
include/lmatch.h) on one GPU: P ranks share the device, as threads of one
process (plain device pointers) or as processes (CUDA IPC), with device-side barriers between
the phases.  mate[] must be bit-identical to the oracle's unique matching (Lemma III.1,
P:167-175: the result does not depend on the partition), the pointing-phase count equal to
Alg. 1's, and every rank must report the same global w(M) and |M|.
"""
import math
import os
import subprocess

import numpy as np
import pytest

import graphgen
import oracle

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
WTOL = 1e-9


@pytest.fixture(scope="module")
def D():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_sc_mandulakgfhs24_b200.dist as d
    return d


def check(g, mate, st, rounds=True):
    ref = oracle.greedy(g)
    bad = np.flatnonzero(mate != ref.mate)
    assert bad.size == 0, f"{bad.size} mismatches, first {bad[:5]}"
    assert st.cardinality == ref.cardinality
    assert math.isclose(st.weight, ref.weight, rel_tol=WTOL)
    if rounds:
        _, ph, _ = oracle.ld_frontier(g)
        assert st.rounds == ph, (st.rounds, ph)


@pytest.mark.parametrize("P", [1, 2, 3, 4])
@pytest.mark.parametrize("maker", [
    lambda: graphgen.rmat(14, 16, seed=5),
    lambda: graphgen.er(20000, 8.0, seed=2, weights="paper"),
    lambda: graphgen.mesh(150, keep=0.6, seed=3),
    lambda: graphgen.mesh(48, seed=1, weights="gradient"),
])
def test_dist_threads(D, P, maker):
    g = maker()
    mate, st0, sts = D.match_dist_threads(g.offsets, g.col, g.w, P)
    check(g, mate, st0)
    for st in sts:  # every rank reports the same global result
        assert st.weight == st0.weight and st.cardinality == st0.cardinality
        assert st.rounds == st0.rounds


def test_dist_threads_hubs_and_empty_parts(D):
    """A hub row holding most entries (edge-balanced bounds leave some parts with few or no
    rows) and P larger than the number of 32-vertex blocks."""
    hub = graphgen.from_edges(3000, [(0, v, float(np.float32(1.0 / (1 + v % 89)))) for v in range(1, 3000)]
                              + [(v, v + 1, 0.5) for v in range(1, 2999, 2)])
    for P in (2, 5):
        mate, st, _ = D.match_dist_threads(hub.offsets, hub.col, hub.w, P)
        check(hub, mate, st)
    tiny = graphgen.from_edges(40, [(i, i + 1, float(i + 1)) for i in range(39)])
    mate, st, _ = D.match_dist_threads(tiny.offsets, tiny.col, tiny.w, 3)
    check(tiny, mate, st)
    empty = graphgen.from_edges(70, [])
    mate, st, _ = D.match_dist_threads(empty.offsets, empty.col, empty.w, 2)
    assert (mate == -1).all() and st.cardinality == 0


def test_dist_round_cap(D):
    g = graphgen.mesh(48, seed=1, weights="gradient")
    import paper_conf_sc_mandulakgfhs24_b200 as lm
    with pytest.raises(lm.LMatchError) as ei:
        D.match_dist_threads(g.offsets, g.col, g.w, 2, max_rounds=3)
    assert ei.value.status == lm.LMATCH_EROUNDS


def test_dist_rejects_bad_arguments(D):
    import paper_conf_sc_mandulakgfhs24_b200 as lm
    g = graphgen.rmat(10, 8, seed=1)
    b = D.edge_balanced_bounds(g.offsets, 2)
    lo, lc, lw = D.local_csr(g.offsets, g.col, g.w, int(b[0]), int(b[1]))
    did = D.dist_id_new()
    for kw in (dict(rank=2, world=2), dict(rank=-1, world=2), dict(rank=0, world=3)):
        with pytest.raises(lm.LMatchError) as ei:
            D.DistMatcher(lo, lc, lw, 0, g.n, kw["rank"], kw["world"], b if kw["world"] == 2 else
                          np.array([0, 32, 64, g.n]), did)
        assert ei.value.status == lm.LMATCH_EINVAL
    # a rank of a 2-rank group whose peer never joins: ENCCL after the rendezvous timeout is too
    # long for a test; the single-rank group needs no peer
    M = D.DistMatcher(g.offsets, g.col, g.w, 0, g.n, 0, 1, np.array([0, g.n]), did)
    mate, st = M.run()
    M.close()
    check(g, mate, st)


def _c_program(tmp_path):
    exe = str(tmp_path / "dist_c")
    lib = os.path.join(ROOT, "paper_conf_sc_mandulakgfhs24_b200")
    subprocess.check_call(["gcc", "-O2", "-Wall", "-I", os.path.join(ROOT, "include"),
                           os.path.join(ROOT, "tests", "c", "dist_c.c"), "-L", lib, "-llmatch",
                           "-lpthread", f"-Wl,-rpath,{lib}", "-o", exe])
    return exe


@pytest.mark.parametrize("mode,P", [("fork", 2), ("fork", 3), ("thread", 2), ("thread", 4)])
def test_c_program_end_to_end(D, tmp_path, mode, P):
    """A C caller (tests/c/dist_c.c; gcc against include/lmatch.h) runs a P-rank partitioned
    matching end to end through the C ABI alone: lmatch_partition + lmatch_dist_id_new +
    lmatch_create_dist + lmatch_run_dist (twice) per rank, as child processes (CUDA IPC) or
    threads (plain pointers).  The program itself checks identity with the single-GPU path; here
    the result is checked against the oracle."""
    exe = _c_program(tmp_path)
    pre = str(tmp_path / "g")
    out = subprocess.run([exe, mode, str(P), pre, "20000"], capture_output=True, text=True, timeout=300)
    assert out.returncode == 0, out.stderr + out.stdout
    off = np.fromfile(pre + ".offsets", dtype=np.int64)
    g = graphgen.Graph(off, np.fromfile(pre + ".col", dtype=np.int32), np.fromfile(pre + ".w", dtype=np.float32))
    mate = np.fromfile(pre + ".mate", dtype=np.int32)
    ref = oracle.greedy(g)
    np.testing.assert_array_equal(mate, ref.mate)
    kv = dict(x.split("=") for x in out.stdout.split())
    assert math.isclose(float(kv["weight"]), ref.weight, rel_tol=WTOL)
    assert int(kv["cardinality"]) == ref.cardinality
    _, ph, _ = oracle.ld_frontier(g)
    assert int(kv["rounds"]) == ph


def _proc_main(rank, world, did, path, q):
    import torch
    import paper_conf_sc_mandulakgfhs24_b200.dist as Dm
    g = graphgen.rmat(15, 16, seed=9, weights="paper")
    b = Dm.edge_balanced_bounds(g.offsets, world)
    v0, v1 = int(b[rank]), int(b[rank + 1])
    lo, lc, lw = Dm.local_csr(g.offsets, g.col, g.w, v0, v1)
    dev = torch.device("cuda", 0)
    d = [torch.from_numpy(x).to(dev) for x in (lo, lc, lw)]  # the device-array create
    M = Dm.DistMatcher(d[0], d[1], d[2], v0, g.n, rank, world, b, did, device=dev)
    res = []
    for _ in range(2):
        mate, st = M.run_device()
        res.append((mate.cpu().numpy(), st.weight, st.cardinality, st.rounds))
    M.close()
    np.save(f"{path}_{rank}.npy", res[0][0])
    q.put((rank, [r[1:] for r in res], bool(np.array_equal(res[0][0], res[1][0]))))


@pytest.mark.parametrize("world", [2, 3])
def test_dist_processes_ipc(D, tmp_path, world):
    """world processes on the one GPU, CUDA IPC between them, device arrays for create, two runs
    per handle."""
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    did = D.dist_id_new()
    q = ctx.Queue()
    path = str(tmp_path / "m")
    ps = [ctx.Process(target=_proc_main, args=(r, world, did, path, q)) for r in range(world)]
    for p in ps:
        p.start()
    for p in ps:
        p.join(timeout=600)
        assert p.exitcode == 0
    got = sorted(q.get(timeout=10) for _ in range(world))
    g = graphgen.rmat(15, 16, seed=9, weights="paper")
    mate = np.concatenate([np.load(f"{path}_{r}.npy") for r in range(world)])
    ref = oracle.greedy(g)
    np.testing.assert_array_equal(mate, ref.mate)
    _, ph, _ = oracle.ld_frontier(g)
    for r, runs, same in got:
        assert same
        for w, c, rounds in runs:
            assert math.isclose(w, ref.weight, rel_tol=WTOL) and c == ref.cardinality and rounds == ph
