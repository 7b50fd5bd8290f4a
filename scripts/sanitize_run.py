"""Workload for compute-sanitizer (memcheck / racecheck / synccheck / initcheck): every code path of
the library on small graphs -- all round-loop modes, A7 pruning, the key cache, Suitor, the hybrid,
sorted + cursor (chunked sort), out of core with and without the host-row cache, paper-style
batches, partition handles with the caller-side transport and the in-process peer-memory
exchange, lmatch_weight and validate_level 2.  Every result is checked against the oracle, so a
run that passes the sanitizer also proves the path it exercised.  (The library-owned multi-process
driver is not run here: its device-barrier kernel spins on peers' flags, which the sanitizer's
kernel serialisation would turn into a timeout; its in-process form, threads with event
barriers, is run.)

usage: compute-sanitizer --tool memcheck python scripts/sanitize_run.py [--quick] [--single]
(--single: single-graph handles only)
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import graphgen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_sc_mandulakgfhs24_b200 as lm  # noqa: E402
import paper_conf_sc_mandulakgfhs24_b200.dist as D  # noqa: E402

QUICK = "--quick" in sys.argv  # racecheck: one small graph (it instruments every smem access)
graphs = ([graphgen.rmat(11, 16, seed=1)] if QUICK else
          [graphgen.er(1 << 16, 16.0, seed=1), graphgen.rmat(14, 16, seed=1),
           graphgen.mesh(48, seed=1, weights="gradient")])
runs = 0
for g in graphs:
    ref = oracle.greedy(g).mate
    configs = [dict(round_loop=r) for r in (0, 1, 2, 3)] + [
        dict(prune=True), dict(prune=True, round_loop=2), dict(key_cache=True),
        dict(key_cache=True, round_loop=2), dict(algorithm="suitor"), dict(algorithm="hybrid"),
        dict(algorithm="sorted", sort_chunk_log2=12), dict(validate_level=2),
        dict(hbm_budget_bytes=8 * g.m // 3, stream_chunk=4096),
        dict(hbm_budget_bytes=8 * g.m // 3, stream_chunk=4096, host_cache=False),
        dict(batches=3)]
    for kw in configs:
        print(f"{g.name} {kw}", flush=True)
        with lm.Matcher(g, **kw) as M:
            mate, st = M.run()
            assert np.array_equal(mate, ref), (g.name, kw)
            w = M.weight(mate)
            assert abs(w - st["weight"]) <= 1e-9 * max(1.0, abs(w))
        runs += 1
    if "--single" in sys.argv:
        continue
    for ex in ("transport", "p2p", "p2p_sync"):
        print(f"{g.name} partitioned {ex}", flush=True)
        mate, _ = D.match_partitioned_local(g.offsets, g.col, g.w, 3, exchange=ex)
        assert np.array_equal(mate, ref), (g.name, ex)
        runs += 1
    mate, _ = D.match_partitioned_local(g.offsets, g.col, g.w, 2, exchange="p2p", batches=2)
    assert np.array_equal(mate, ref), (g.name, "p2p batches")
    # the library-owned driver with its ranks as threads (event barriers, no spinning kernel)
    mate, _, _ = D.match_dist_threads(g.offsets, g.col, g.w, 2)
    assert np.array_equal(mate, ref), (g.name, "dist threads")
    runs += 2
print(f"sanitize_run ok: {runs} runs, every mate[] equal to the oracle's")
