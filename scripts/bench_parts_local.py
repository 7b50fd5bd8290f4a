"""P logical partitions of one graph on ONE GPU: the partitioned round driven through the
caller-side transport (LocalTransport: torch copies of the claim segments and bitmap words) vs the
peer-memory exchange (lmatch_p2p_*: the library's kernels store into the other parts' buffers).
Both run every part on the same device, so this measures the exchange and driver overhead per
round, not scaling.  Prints one JSON line per (P, exchange).

    python scripts/bench_parts_local.py --scale 22 --parts 1 2 4 8 --steps 3
"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import graphgen.gpu as gg  # noqa: E402
import paper_conf_sc_mandulakgfhs24_b200.dist as D  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--scale", type=int, default=22)
    ap.add_argument("--parts", type=int, nargs="+", default=[1, 2, 4, 8])
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=2)
    a = ap.parse_args()
    dev = torch.device("cuda", 0)
    g = gg.rmat(a.scale, 16, seed=1, device=dev)
    off = g.offsets.cpu().numpy()
    col = g.col.cpu().numpy()
    w = g.w.cpu().numpy()
    ref = None
    for P in a.parts:
        b = D.edge_balanced_bounds(off, P)
        for ex in ("transport", "p2p", "p2p_events"):
            parts = []
            for p in range(P):
                lo, lc, lw = D.local_csr(off, col, w, int(b[p]), int(b[p + 1]))
                parts.append(D.LibPart(lo, lc, lw, int(b[p]), g.n, b, p, device=dev))
            if ex.startswith("p2p"):
                D.connect_p2p_local(parts)
                bar = D.barrier_events(parts) if ex == "p2p_events" else D.barrier_local(parts)
                run = lambda: D.run_parts_p2p(parts, bar, D.LocalTransport(P))  # noqa: E731
            else:
                run = lambda: D.run_parts(parts, D.LocalTransport(P))  # noqa: E731
            for _ in range(a.warmup):
                res = run()
            torch.cuda.synchronize()
            l0 = D.kernel_launch_count()
            t0 = time.perf_counter()
            for _ in range(a.steps):
                res = run()
            torch.cuda.synchronize()
            dt = (time.perf_counter() - t0) / a.steps
            launches = (D.kernel_launch_count() - l0) // a.steps
            mate = np.concatenate([m.cpu().numpy() for m in res.mates])
            if ref is None:
                ref = mate
            print(json.dumps({"scale": a.scale, "parts": P, "exchange": ex, "ms_per_run": dt * 1e3,
                              "rounds": res.rounds, "ms_per_round": dt * 1e3 / res.rounds,
                              "kernel_launches_per_run": int(launches),
                              "same_mate_as_first": bool(np.array_equal(mate, ref)),
                              "gteps_one_gpu": g.m_u / dt / 1e9}), flush=True)
            for p in parts:
                p.close()


if __name__ == "__main__":
    main()
