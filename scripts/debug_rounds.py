"""Debug: GPU mate after k rounds vs a numpy simulation of the frontier iteration (test aid)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import graphgen
import paper_conf_sc_mandulakgfhs24_b200 as lm

def sim(g, kmax):
    n = g.n; o, c, w = g.offsets, g.col, g.w
    wb = w.view(np.uint32).astype(np.uint64)
    key = (wb << np.uint64(32)) | c.astype(np.uint64)
    u = np.repeat(np.arange(n), np.diff(o))
    key[u == c] = 0
    matched = np.zeros(n, bool); best = np.zeros(n, np.uint64)
    need = np.diff(o) > 0
    for r in range(kmax):
        if not need.any(): break
        k2 = key.copy(); k2[matched[c]] = 0
        rowmax = np.zeros(n, np.uint64)
        np.maximum.at(rowmax, u, k2)
        best[need] = rowmax[need]
        ptr = (best & np.uint64(0xffffffff)).astype(np.int64)
        has = best != 0
        mut = has & (best[ptr] & np.uint64(0xffffffff)).astype(np.int64).__eq__(np.arange(n)) & (best[ptr] != 0)
        newm = need & mut
        matched[newm] = True; matched[ptr[newm]] = True
        live = ~matched & has
        need = live & matched[ptr]
    mate = np.where(matched, (best & np.uint64(0xffffffff)).astype(np.int64), -1)
    return mate.astype(np.int32)

for name, g in [("er16", graphgen.er(1 << 16, 16.0, seed=1)), ("rmat14", graphgen.rmat(14, 16, seed=1))]:
    for k in (1, 2, 3, 50):
        with lm.Matcher(g, max_rounds=k) as M:
            mate, st = M.run()
        ref = sim(g, k)
        bad = np.flatnonzero(mate != ref)
        print(name, "rounds", k, st["rounds"], "mismatch", bad.size, bad[:5], mate[bad[:5]], ref[bad[:5]], flush=True)
