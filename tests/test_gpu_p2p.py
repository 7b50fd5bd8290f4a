"""GPU: the partitioned round with the exchange done by the library's own kernels over peer memory
(include/lmatch.h "Peer-memory exchange"; SURVEY 8(e) B200-native variant).

Claims are stored by the claims kernels straight into the owner's inbox, changed owned bitmap
words are pushed into every replica by the match step, and frontier sizes into every part's slot;
the driver only places barriers.  Two settings on one B200:
  * P logical parts in one process (plain device pointers between the parts' buffers);
  * two processes on the same GPU with CUDA IPC handles (cudaIpcOpenMemHandle), gloo barriers --
    the cross-process path an 8-GPU run uses, minus NVLink.
Bar: mate[] bit-identical to the oracle for every P (Lemma III.1), rounds equal to the
frontier oracle's phases, w(M) within 1e-9 relative.
"""
import math
import os
import socket

import numpy as np
import pytest

import graphgen
import oracle

pytestmark = pytest.mark.gpu

WTOL = 1e-9


@pytest.fixture(scope="module")
def D():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_sc_mandulakgfhs24_b200.dist as dist_mod
    return dist_mod


def _check(g, mate, res):
    ref = oracle.greedy(g)
    np.testing.assert_array_equal(mate, ref.mate)
    assert res.matched == 2 * ref.cardinality
    assert math.isclose(res.weight, ref.weight, rel_tol=WTOL)
    assert res.rounds == oracle.ld_frontier(g)[1]


@pytest.mark.parametrize("P", [1, 2, 3, 4, 8])
@pytest.mark.parametrize("maker", [
    lambda: graphgen.rmat(15, 16, seed=11),
    lambda: graphgen.er(20000, 8.0, seed=12, weights="paper"),
    lambda: graphgen.mesh(150, keep=0.6, seed=13),
    lambda: graphgen.mesh(40, seed=14, weights="gradient"),
])
def test_p2p_local_invariance(D, P, maker):
    """Cross-stream event barriers (default) and host-synchronising barriers."""
    g = maker()
    for ex in ("p2p", "p2p_sync"):
        mate, res = D.match_partitioned_local(g.offsets, g.col, g.w, P, exchange=ex)
        _check(g, mate, res)


@pytest.mark.parametrize("exchange", ["transport", "p2p"])
def test_partitioned_larger_graph(D, exchange):
    """R-MAT scale 20 over 4 and 7 parts (rounds with millions of claims): both exchanges stay
    bit-exact (the in-process transport once raced against the parts' own streams here)."""
    g = graphgen.rmat(20, 16, seed=3)
    for P in (4, 7):
        mate, res = D.match_partitioned_local(g.offsets, g.col, g.w, P, exchange=exchange)
        _check(g, mate, res)


@pytest.mark.parametrize("exchange", ["transport", "p2p"])
def test_partitioned_scale24_repeat_vs_single(D, exchange):
    """R-MAT scale 24 (configs[1]) over 2 parts, three runs on the same parts: every run equals
    the single-GPU result (itself certified exact at this size by test_full_size_rmat24_certificate).
    At this size an unordered stream once made the in-process transport nondeterministic."""
    import torch
    import graphgen.gpu as gg
    import paper_conf_sc_mandulakgfhs24_b200 as lm
    g = gg.rmat(24, 16, seed=1, device=torch.device("cuda"))
    off, col, w = g.offsets.cpu().numpy(), g.col.cpu().numpy(), g.w.cpu().numpy()
    del g
    with lm.Matcher(off, col, w) as M:
        ref, st = M.run()
    b = D.edge_balanced_bounds(off, 2)
    parts = []
    for p in range(2):
        lo, lc, lw = D.local_csr(off, col, w, int(b[p]), int(b[p + 1]))
        parts.append(D.LibPart(lo, lc, lw, int(b[p]), len(off) - 1, b, p))
    if exchange == "p2p":
        D.connect_p2p_local(parts)
        run = lambda: D.run_parts_p2p(parts, D.barrier_local(parts), D.LocalTransport(2))  # noqa: E731
    else:
        run = lambda: D.run_parts(parts, D.LocalTransport(2))  # noqa: E731
    for _ in range(3):
        res = run()
        mate = np.concatenate([m.cpu().numpy() for m in res.mates])
        np.testing.assert_array_equal(mate, ref)
        assert res.rounds == st["rounds"]
        assert math.isclose(res.weight, st["weight"], rel_tol=WTOL)
    for p in parts:
        p.close()


def test_p2p_hub_rows_and_repeat(D):
    """Hub rows cut across parts; two runs on the same connected handles give the same result
    (inbox counts are left at zero by every round, the bitmap shadow is reset per run)."""
    g = graphgen.from_edges(9001, [(0, v, 1.0) for v in range(1, 9001)] +
                            [(v, v + 1, 0.5) for v in range(100, 8000, 7)])
    b = D.edge_balanced_bounds(g.offsets, 4)
    parts = []
    for p in range(4):
        lo, lc, lw = D.local_csr(g.offsets, g.col, g.w, int(b[p]), int(b[p + 1]))
        parts.append(D.LibPart(lo, lc, lw, int(b[p]), g.n, b, p))
    D.connect_p2p_local(parts)
    for _ in range(2):
        res = D.run_parts_p2p(parts, D.barrier_local(parts), D.LocalTransport(4))
        mate = np.concatenate([m.cpu().numpy() for m in res.mates])
        _check(g, mate, res)
    for p in parts:
        p.close()


def test_p2p_misuse(D):
    import paper_conf_sc_mandulakgfhs24_b200 as lm
    g = graphgen.rmat(10, 8, seed=3)
    b = D.edge_balanced_bounds(g.offsets, 2)
    parts = []
    for p in range(2):
        lo, lc, lw = D.local_csr(g.offsets, g.col, g.w, int(b[p]), int(b[p + 1]))
        parts.append(D.LibPart(lo, lc, lw, int(b[p]), g.n, b, p))
    with pytest.raises(lm.LMatchError):       # not enabled
        parts[0].p2p_begin()
    assert D._lib.lmatch_p2p_enable(parts[0].h, 1) == lm.LMATCH_EINVAL   # wrong part index
    parts[0].p2p_enable()
    with pytest.raises(lm.LMatchError):       # peer not attached yet
        parts[0].p2p_begin()
    with pytest.raises(lm.LMatchError):       # the transport calls are refused once enabled
        parts[0].begin()
    for p in parts:
        p.close()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _ipc_worker(rank, world, port, spec, q, events=False):
    import torch
    import torch.distributed as dist
    import paper_conf_sc_mandulakgfhs24_b200.dist as D
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    part = None
    try:
        torch.cuda.set_device(0)
        kind, args = spec
        g = getattr(graphgen, kind)(*args)
        b = D.edge_balanced_bounds(g.offsets, world)
        lo, lc, lw = D.local_csr(g.offsets, g.col, g.w, int(b[rank]), int(b[rank + 1]))
        part = D.LibPart(lo, lc, lw, int(b[rank]), g.n, b, rank)
        D.connect_p2p_torch(part)
        if events:
            D.connect_events_torch(part)
            barrier = D.barrier_torch_events([part])
        else:
            barrier = D.barrier_torch([part])
        out = []
        for _ in range(2):
            res = D.run_parts_p2p([part], barrier, D.TorchTransport())
            out.append((res.mates[0].cpu().numpy(), res.weight, res.matched, res.rounds))
        q.put((rank, out))
        dist.barrier()   # no rank releases its window while a peer may still store into it
    except Exception as e:  # surface the error to the parent
        q.put((rank, repr(e)))
        raise
    finally:
        if part is not None:
            part.close()
        dist.destroy_process_group()


@pytest.mark.parametrize("events", [False, True])
@pytest.mark.parametrize("world,spec", [(2, ("rmat", (14, 16, 5))), (3, ("mesh", (60, 0.6, 2)))])
def test_p2p_ipc_processes(D, world, spec, events):
    """`world` processes on the one GPU, windows and bitmaps opened through CUDA IPC handles
    exchanged with all_gather_object; barriers either drain the stream + gloo barrier, or
    interprocess CUDA events (record, gloo barrier, stream waits: no stream drained); run twice
    on the same connection."""
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_ipc_worker, args=(r, world, port, spec, q, events))
             for r in range(world)]
    for p in procs:
        p.start()
    got = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=120)
    errs = [x for x in got if isinstance(x[1], str)]
    assert not errs, errs
    for p in procs:
        assert p.exitcode == 0
    got.sort(key=lambda x: x[0])
    kind, args = spec
    g = getattr(graphgen, kind)(*args)
    ref = oracle.greedy(g)
    ph = oracle.ld_frontier(g)[1]
    for run in range(2):
        mate = np.concatenate([x[1][run][0] for x in got])
        np.testing.assert_array_equal(mate, ref.mate)
        for x in got:
            assert math.isclose(x[1][run][1], ref.weight, rel_tol=WTOL)
            assert x[1][run][2] == 2 * ref.cardinality
            assert x[1][run][3] == ph
