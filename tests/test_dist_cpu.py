"""N>1 path on CPU: the product driver (paper_conf_sc_mandulakgfhs24_b200.dist.run_parts) with the
numpy partition model, over (a) the in-process LocalTransport and (b) torch.distributed gloo with
world_size 2 and 3 (TorchTransport, the same class the NCCL runs use).  The result must equal the
oracle's unique matching for every partition (Lemma III.1)."""
import math
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import graphgen
import oracle
from dist_model import NumpyP2PPart, NumpyPart

dist_mod = pytest.importorskip("paper_conf_sc_mandulakgfhs24_b200.dist")


def build_parts(g, P):
    b = dist_mod.edge_balanced_bounds(g.offsets, P)
    parts = []
    for p in range(P):
        lo, lc, lw = dist_mod.local_csr(g.offsets, g.col, g.w, int(b[p]), int(b[p + 1]))
        parts.append(NumpyPart(lo, lc, lw, int(b[p]), g.n, b, p))
    return b, parts


def test_edge_balanced_bounds():
    g = graphgen.rmat(12, 16, seed=3)
    for P in (1, 2, 3, 4, 8):
        b = dist_mod.edge_balanced_bounds(g.offsets, P)
        assert b[0] == 0 and b[-1] == g.n and (np.diff(b) >= 0).all()
        assert all(x % 32 == 0 for x in b[:-1])
        per = np.diff(g.offsets[b])
        assert per.max() <= g.m / P + 32 * g.degrees().max() + 1


def _bounds_by_definition(offsets, P, align):
    """The partition rule of include/lmatch.h written out: bound p = the first row whose start
    offset reaches floor(m p / P) (np.searchsorted, side='left'), rounded up to `align`, capped at
    n and kept non-decreasing."""
    n = len(offsets) - 1
    m = int(offsets[-1])
    b = [0]
    for p in range(1, P):
        v = int(np.searchsorted(offsets, (m * p) // P, side="left"))
        b.append(max(b[-1], min(n, -(-v // align) * align)))
    return np.array(b + [n], dtype=np.int64)


def test_partition_in_c_matches_definition():
    """lmatch_partition (the C partitioner, host-only) against the rule written out, on R-MAT,
    a single-hub star (one row holds half the entries), empty graphs and P > n."""
    rng = np.random.default_rng(5)
    hub = graphgen.from_edges(500, [(0, v, 1.0) for v in range(1, 500)])
    cases = [graphgen.rmat(12, 16, seed=3).offsets, graphgen.er(3000, 5.0, seed=2).offsets,
             hub.offsets, np.zeros(1, np.int64), np.zeros(40, np.int64),
             np.concatenate([[0], np.cumsum(rng.integers(0, 50, 777))]).astype(np.int64)]
    for off in cases:
        for P in (1, 2, 3, 7, 64):
            for align in (1, 32, 64):
                got = np.zeros(P + 1, np.int64)
                rc = dist_mod._lib.lmatch_partition(off.ctypes.data, len(off) - 1, P, align,
                                                    got.ctypes.data)
                assert rc == 0
                np.testing.assert_array_equal(got, _bounds_by_definition(off, P, align))
    bad = np.array([1, 2], np.int64)
    got = np.zeros(3, np.int64)
    assert dist_mod._lib.lmatch_partition(bad.ctypes.data, 1, 2, 32, got.ctypes.data) == -1
    assert dist_mod._lib.lmatch_partition(bad.ctypes.data, 1, 0, 32, got.ctypes.data) == -1


def test_dist_id_new_unique():
    ids = {dist_mod.dist_id_new() for _ in range(20)}
    assert len(ids) == 20
    for x in ids:
        assert x.startswith(b"lmatch-") and len(x) == 64


@pytest.mark.parametrize("P", [1, 2, 3, 5])
def test_local_transport_numpy_model(P):

    graphs = [graphgen.rmat(9, 8, seed=P), graphgen.er(600, 5.0, seed=P, weights="paper"),
              graphgen.mesh(20, keep=0.7, seed=P, weights="ones")]
    for g in graphs:
        _, parts = build_parts(g, P)
        res = dist_mod.run_parts(parts, dist_mod.LocalTransport(P))
        mate = np.concatenate([m.numpy() for m in res.mates])
        ref = oracle.greedy(g)
        np.testing.assert_array_equal(mate, ref.mate)
        _, ph, _ = oracle.ld_frontier(g)
        assert res.rounds == ph
        assert math.isclose(res.weight, ref.weight, rel_tol=1e-9)
        assert res.matched == 2 * ref.cardinality


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, spec, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        kind, args = spec
        g = getattr(graphgen, kind)(*args)
        b = dist_mod.edge_balanced_bounds(g.offsets, world)
        lo, lc, lw = dist_mod.local_csr(g.offsets, g.col, g.w, int(b[rank]), int(b[rank + 1]))
        part = NumpyPart(lo, lc, lw, int(b[rank]), g.n, b, rank)
        res = dist_mod.run_parts([part], dist_mod.TorchTransport())
        q.put((rank, res.mates[0].numpy(), res.weight, res.matched, res.rounds))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,spec", [(2, ("rmat", (10, 8, 2))), (3, ("er", (700, 6.0, 3))),
                                        (2, ("mesh", (24, 0.6, 4)))])
def test_gloo_torchtransport(world, spec):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, spec, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    out.sort(key=lambda x: x[0])
    mate = np.concatenate([o[1] for o in out])
    kind, args = spec
    g = getattr(graphgen, kind)(*args)
    ref = oracle.greedy(g)
    np.testing.assert_array_equal(mate, ref.mate)
    for o in out:
        assert math.isclose(o[2], ref.weight, rel_tol=1e-9)
        assert o[3] == 2 * ref.cardinality
        assert o[4] == oracle.ld_frontier(g)[1]


# ------------------------------------------------------------ peer-memory exchange (lmatch_p2p_*)
@pytest.mark.parametrize("P", [1, 2, 3, 5])
def test_p2p_local_numpy_model(P):
    """run_parts_p2p (the peer-memory protocol: claims stored into the owners' inboxes, changed
    bitmap words pushed into every replica, frontier sizes into every slot) with parts in one
    process: the oracle's unique matching and its round count for every P."""
    for g in (graphgen.rmat(9, 8, seed=P), graphgen.mesh(20, keep=0.7, seed=P, weights="ones"),
              graphgen.mesh(12, seed=P, weights="gradient")):
        b = dist_mod.edge_balanced_bounds(g.offsets, P)
        parts = []
        for p in range(P):
            lo, lc, lw = dist_mod.local_csr(g.offsets, g.col, g.w, int(b[p]), int(b[p + 1]))
            parts.append(NumpyP2PPart(lo, lc, lw, int(b[p]), g.n, b, p))
        try:
            for p in parts:
                p.p2p_enable()
            for p in parts:
                for q in parts:
                    if q is not p:
                        p.p2p_attach_local(q.part, q)
            res = dist_mod.run_parts_p2p(parts, dist_mod.barrier_local(parts),
                                         dist_mod.LocalTransport(P))
        finally:
            for p in parts:
                p.close()
        ref = oracle.greedy(g)
        np.testing.assert_array_equal(np.concatenate([m.numpy() for m in res.mates]), ref.mate)
        assert res.rounds == oracle.ld_frontier(g)[1]
        assert math.isclose(res.weight, ref.weight, rel_tol=1e-9)


def _p2p_worker(rank, world, port, spec, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    part = None
    try:
        kind, args = spec
        g = getattr(graphgen, kind)(*args)
        b = dist_mod.edge_balanced_bounds(g.offsets, world)
        lo, lc, lw = dist_mod.local_csr(g.offsets, g.col, g.w, int(b[rank]), int(b[rank + 1]))
        part = NumpyP2PPart(lo, lc, lw, int(b[rank]), g.n, b, rank)
        part.p2p_enable()
        allh = [None] * world
        dist.all_gather_object(allh, (rank, part.p2p_export()))
        for peer, h in allh:
            if peer != rank:
                part.p2p_attach(peer, h)
        res = dist_mod.run_parts_p2p([part], dist_mod.barrier_torch([part]),
                                     dist_mod.TorchTransport())
        q.put((rank, res.mates[0].numpy(), res.weight, res.matched, res.rounds))
        dist.barrier()   # nobody unlinks its window while a peer may still read it
    finally:
        if part is not None:
            part.close()
        dist.destroy_process_group()


@pytest.mark.parametrize("world,spec", [(2, ("rmat", (10, 8, 2))), (3, ("er", (700, 6.0, 3)))])
def test_gloo_p2p(world, spec):
    """The peer-memory driver across processes (shared-memory windows, gloo barriers)."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_p2p_worker, args=(r, world, port, spec, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = [q.get(timeout=180) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    out.sort(key=lambda x: x[0])
    kind, args = spec
    g = getattr(graphgen, kind)(*args)
    ref = oracle.greedy(g)
    np.testing.assert_array_equal(np.concatenate([o[1] for o in out]), ref.mate)
    for o in out:
        assert math.isclose(o[2], ref.weight, rel_tol=1e-9)
        assert o[3] == 2 * ref.cardinality
        assert o[4] == oracle.ld_frontier(g)[1]
