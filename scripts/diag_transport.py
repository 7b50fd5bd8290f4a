"""Diagnose the in-process transport path: repeat runs and sizes (builder tooling)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import graphgen.gpu as gg
import paper_conf_sc_mandulakgfhs24_b200 as lm
import paper_conf_sc_mandulakgfhs24_b200.dist as D
dev = torch.device("cuda", 0)
for scale in (20, 22, 24):
    g = gg.rmat(scale, 16, seed=1, device=dev)
    off, col, w = g.offsets.cpu().numpy(), g.col.cpu().numpy(), g.w.cpu().numpy()
    with lm.Matcher(off, col, w) as M:
        ref, st = M.run()
    for P in (2, 4, 8):
        b = D.edge_balanced_bounds(off, P)
        parts = []
        for p in range(P):
            lo, lc, lw = D.local_csr(off, col, w, int(b[p]), int(b[p + 1]))
            parts.append(D.LibPart(lo, lc, lw, int(b[p]), g.n, b, p, device=dev))
        out = []
        for r in range(3):
            res = D.run_parts(parts, D.LocalTransport(P))
            mate = np.concatenate([m.cpu().numpy() for m in res.mates])
            out.append((int((mate != ref).sum()), res.rounds))
        print(scale, P, "ref rounds", st["rounds"], "runs (mismatches, rounds):", out, flush=True)
        for p in parts:
            p.close()
