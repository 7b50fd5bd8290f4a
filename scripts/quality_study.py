"""Matching quality study (Table II analogue): w(M*) of the unique
locally dominant matching (oracle.greedy, = the GPU result) against the optimum w(OPT) from
networkx's blossom algorithm, on small synthetic graphs of the workload classes (R-MAT, ER, mesh,
road-like) with uniform and 3-decimal "paper" weights.  CPU only; prints one JSON line per graph.

    python scripts/quality_study.py > profiles/r01_quality_vs_opt.jsonl
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import networkx as nx  # noqa: E402
import numpy as np  # noqa: E402

import graphgen  # noqa: E402
import oracle  # noqa: E402


def to_nx(g):
    G = nx.Graph()
    G.add_nodes_from(range(g.n))
    off = g.offsets
    for u in range(g.n):
        for j in range(off[u], off[u + 1]):
            v = int(g.col[j])
            if u < v:
                G.add_edge(u, v, weight=float(g.w[j]))
    return G


def main():
    cases = []
    for w in ("uniform", "paper"):
        cases += [("rmat_s10_ef8", lambda w=w: graphgen.rmat(10, 8, seed=1, weights=w)),
                  ("er_1500_d8", lambda w=w: graphgen.er(1500, 8.0, seed=2, weights=w)),
                  ("mesh_36", lambda w=w: graphgen.mesh(36, seed=3, weights=w)),
                  ("road_40", lambda w=w: graphgen.mesh(40, keep=0.6, seed=4, weights=w))]
        cases[-4:] = [(f"{nm}_{w}", mk) for nm, mk in cases[-4:]]
    for name, mk in cases:
        g = mk()
        ref = oracle.greedy(g)
        t0 = time.time()
        opt = nx.max_weight_matching(to_nx(g))
        t_opt = time.time() - t0
        w_opt = sum(float(g.w[np.flatnonzero(g.col[g.offsets[u]:g.offsets[u + 1]] == v)[0] + g.offsets[u]])
                    for u, v in opt)
        print(json.dumps({"graph": name, "n": g.n, "m_undirected": g.m // 2,
                          "card_ld": ref.cardinality, "card_opt": len(opt),
                          "w_ld": ref.weight, "w_opt": w_opt, "ratio": ref.weight / w_opt,
                          "pct_below_opt": 100 * (1 - ref.weight / w_opt),
                          "blossom_s": round(t_opt, 1)}), flush=True)


if __name__ == "__main__":
    main()
