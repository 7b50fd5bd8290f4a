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


@pytest.mark.parametrize("exchange", ["dist", "p2p"])
def test_bench_self_launch_two_ranks(D, exchange):
    """`python bench.py --gpus 2` without torchrun launches 2 ranks itself (torch.distributed.run
    on 127.0.0.1; gloo control plane; the ranks share this one GPU): each rank generates only its
    rows, the partitioned run's matching equals the oracle's (|M|, w(M)) and rank 0 prints one
    JSON line with n_gpus = 2."""
    import json
    cmd = ["python", os.path.join(ROOT, "bench.py"), "--gpus", "2", "--scale", "14", "--steps", "2",
           "--warmup", "3", "--no-cpu", "--e2e-steps", "1", "--exchange", exchange]
    out = subprocess.run(cmd, capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-3000:]
    lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, out.stdout
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["scaling"] == "strong" and d["value"] > 0
    g = graphgen.rmat(14, 16, seed=1)
    ref = oracle.greedy(g)
    assert d["cardinality"] == ref.cardinality
    assert math.isclose(d["matched_weight"], ref.weight, rel_tol=WTOL)
    _, ph, _ = oracle.ld_frontier(g)
    assert d["rounds"] == ph
    assert d["e2e"]["value"] > 0 and d["gpu_launches"] > 0
    assert len(d["config"]["part_bounds"]) == 3


def _transport_main(rank, world, backend, port, path, q):
    import torch
    import torch.distributed as dist
    import paper_conf_sc_mandulakgfhs24_b200.dist as Dm
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    if backend == "nccl":
        dist.init_process_group("nccl", rank=rank, world_size=world, device_id=dev)
    else:
        dist.init_process_group("gloo", rank=rank, world_size=world)
    g = graphgen.rmat(16, 16, seed=13, weights="paper")
    b = Dm.edge_balanced_bounds(g.offsets, world)
    v0, v1 = int(b[rank]), int(b[rank + 1])
    part = Dm.LibPart(*Dm.local_csr(g.offsets, g.col, g.w, v0, v1), v0, g.n, b, rank, device=dev)
    res = Dm.run_parts([part], Dm.TorchTransport())
    res2 = Dm.run_parts([part], Dm.TorchTransport())  # a second run on the same handles
    np.save(f"{path}_{rank}.npy", res.mates[0].cpu().numpy())
    same = bool(torch.equal(res.mates[0], res2.mates[0]))
    q.put((rank, res.weight, res.matched, res.rounds, same))
    part.close()
    dist.destroy_process_group()


@pytest.mark.parametrize("backend,world", [("nccl", 1), ("gloo", 2), ("gloo", 3)])
def test_torch_transport_with_libparts(D, tmp_path, backend, world):
    """The caller-side exchange (TorchTransport: all_to_all of claims, all_gather of bitmap words,
    all_reduce of frontier sizes) driving REAL partition handles (LibPart) on the GPU: over NCCL
    (one rank -- NCCL refuses two ranks on one GPU) and over gloo (2 and 3 processes on this GPU,
    CUDA tensors staged through host memory).  Same matching as the oracle."""
    import socket
    import torch.multiprocessing as mp
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    path = str(tmp_path / "t")
    ps = [ctx.Process(target=_transport_main, args=(r, world, backend, port, path, q)) for r in range(world)]
    for p in ps:
        p.start()
    for p in ps:
        p.join(timeout=600)
        assert p.exitcode == 0
    got = [q.get(timeout=10) for _ in range(world)]
    g = graphgen.rmat(16, 16, seed=13, weights="paper")
    mate = np.concatenate([np.load(f"{path}_{r}.npy") for r in range(world)])
    ref = oracle.greedy(g)
    np.testing.assert_array_equal(mate, ref.mate)
    _, ph, _ = oracle.ld_frontier(g)
    for r, w, matched, rounds, same in got:
        assert same and rounds == ph and matched == 2 * ref.cardinality
        assert math.isclose(w, ref.weight, rel_tol=WTOL)


@pytest.mark.parametrize("P", [2, 3])
@pytest.mark.parametrize("kw", [dict(hbm_budget_bytes=60000, stream_chunk=1024),
                                dict(hbm_budget_bytes=60000, stream_chunk=1024, host_cache=False),
                                dict(batches=3)])
def test_out_of_core_parts(D, P, kw):
    """NEXT-2 per device: every part streams its own rows from pinned host memory (a budget that
    keeps a prefix resident, or the paper's batch count N_i = 3 with nothing resident), with and
    without the host-row key cache, through the caller-side transport, the Python peer-memory
    round and the library-owned driver.  Same matching as the oracle for every partition."""
    g = graphgen.rmat(15, 16, seed=21)
    ref = oracle.greedy(g)
    _, ph, _ = oracle.ld_frontier(g)
    for exchange in ("transport", "p2p"):
        mate, res = D.match_partitioned_local(g.offsets, g.col, g.w, P, exchange=exchange, **kw)
        np.testing.assert_array_equal(mate, ref.mate)
        assert res.rounds == ph
    mate, st, _ = D.match_dist_threads(g.offsets, g.col, g.w, P, **kw)
    check(g, mate, st)


def test_dist_single_rank_uses_the_device_round_loop(D):
    """A one-rank lmatch_create_dist group exchanges nothing: it sizes the pointer launches from the
    frontier it reads after each compaction and runs the small tail in the persistent kernel, as
    the single-graph path does.  Same result and phases (incl. a many-round graph, whose tail
    switches to the push frontier)."""
    for g in (graphgen.rmat(15, 16, seed=4), graphgen.mesh(64, seed=1, weights="gradient")):
        mate, st, _ = D.match_dist_threads(g.offsets, g.col, g.w, 1)
        check(g, mate, st)


def _lonely_rank(q):
    import paper_conf_sc_mandulakgfhs24_b200 as lm
    import paper_conf_sc_mandulakgfhs24_b200.dist as Dm
    g = graphgen.rmat(10, 8, seed=1)
    b = Dm.edge_balanced_bounds(g.offsets, 2)
    lo, lc, lw = Dm.local_csr(g.offsets, g.col, g.w, int(b[0]), int(b[1]))
    try:
        Dm.DistMatcher(lo, lc, lw, 0, g.n, 0, 2, b, Dm.dist_id_new())
        q.put(0)
    except lm.LMatchError as e:
        q.put(e.status)


def test_dist_missing_peer_times_out(D):
    """Rank 0 of a 2-rank group whose peer never joins gets ENCCL after the rendezvous timeout
    (LMATCH_DIST_TIMEOUT_S=3) instead of hanging, and leaves no segment in /dev/shm."""
    import torch.multiprocessing as mp
    before = set(os.listdir("/dev/shm")) if os.path.isdir("/dev/shm") else set()
    os.environ["LMATCH_DIST_TIMEOUT_S"] = "3"
    try:
        ctx = mp.get_context("spawn")
        q = ctx.Queue()
        p = ctx.Process(target=_lonely_rank, args=(q,))
        p.start()
        p.join(timeout=120)
        assert p.exitcode == 0
        assert q.get(timeout=5) == -5  # LMATCH_ENCCL
    finally:
        del os.environ["LMATCH_DIST_TIMEOUT_S"]
    after = set(os.listdir("/dev/shm")) if os.path.isdir("/dev/shm") else set()
    assert not [x for x in after - before if x.startswith("lmatch-")]
