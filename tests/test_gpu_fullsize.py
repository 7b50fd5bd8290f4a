"""Exactness at the full sizes the bench and BASELINE.json name, beyond 2^32 directed entries.

Every check is the oracle's O(m) certificate (oracle.certificate: C(M) holds iff M is the unique
maximal locally dominant matching, R1 iii; pins: Def. II.1, Lemma III.1
P:167-175) plus w(M) against the oracle's fp64 weight of the same mate[] (1e-9 relative).

* R-MAT scale 28 (configs[3]'s graph, m_d = 8.47e9 > 2^32 directed entries: the round-1 sweep's
  32-bit row-start window wraps), resident on one GPU from the device CSR as bench.py runs it;
* the same graph OUT OF CORE with a 32 GB HBM budget (47% resident, the rest streamed through the
  device ring in round 1 and read zero-copy / through the host-row cache later);
* the sorted-adjacency algorithm (NEXT-3) at R-MAT scale 26 (2.1e9 entries: the row sort runs in
  two chunks);
* the library-owned partitioned driver (lmatch_create_dist / lmatch_run_dist) with P = 2 ranks at
  R-MAT scale 26;
* R-MAT scale 29 (16.99e9 entries, the north_star's ">= 2^33 edges" graph) when
  LMATCH_HUGE=1 (host RAM >= ~150 GB; about 5 minutes).
"""
import math
import os

import numpy as np
import pytest

import graphgen
import oracle

pytestmark = [pytest.mark.gpu, pytest.mark.slow]
WTOL = 1e-9


@pytest.fixture(scope="module")
def lm():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_sc_mandulakgfhs24_b200 as p
    return p


def _certify(g, mate, st):
    code, bad = oracle.certificate(g, mate)
    assert code == 0, (code, bad)
    assert math.isclose(st["weight"], oracle.weight(g, mate), rel_tol=WTOL)
    assert st["cardinality"] == int((mate >= 0).sum()) // 2


def _host_ram_gb():
    return os.sysconf("SC_PAGE_SIZE") * os.sysconf("SC_PHYS_PAGES") / 1e9


def test_rmat_s28_resident_and_out_of_core(lm):
    import torch
    import graphgen.gpu as gg
    if _host_ram_gb() < 100:
        pytest.skip("needs ~80 GB of host RAM for the certificate")
    dg = gg.rmat(28, 16, seed=1, device=torch.device("cuda"))
    assert dg.m > 2 ** 32
    g = graphgen.Graph(dg.offsets.cpu().numpy(), dg.col.cpu().numpy(), dg.w.cpu().numpy())
    M = lm.Matcher.from_device(dg.offsets, dg.col, dg.w, dg.n, dg.m, stream=torch.cuda.current_stream())
    del dg
    torch.cuda.empty_cache()
    mate, st = M.run()
    M.close()
    _certify(g, mate, st)
    # the same graph with 32 GB of the 68 GB adjacency resident: identical mate[]
    with lm.Matcher(g, hbm_budget_bytes=32 * 10 ** 9) as M2:
        mate2, st2 = M2.run()
    assert st2["resident_entries"] < g.m and st2["bytes_streamed"] > 0
    np.testing.assert_array_equal(mate2, mate)
    assert st2["rounds"] == st["rounds"]
    assert math.isclose(st2["weight"], st["weight"], rel_tol=WTOL)


def test_sorted_rmat_s26(lm):
    """NEXT-3 at the bench's size: 2.1e9 entries are sorted in two 2^30-entry chunks (the chunk
    boundary logic), then the cursor rounds; certificate + identity with the LD path."""
    import torch
    import graphgen.gpu as gg
    dg = gg.rmat(26, 16, seed=1, device=torch.device("cuda"))
    g = graphgen.Graph(dg.offsets.cpu().numpy(), dg.col.cpu().numpy(), dg.w.cpu().numpy())
    M = lm.Matcher.from_device(dg.offsets, dg.col, dg.w, dg.n, dg.m, stream=torch.cuda.current_stream(),
                               algorithm="sorted")
    del dg
    torch.cuda.empty_cache()
    mate, st = M.run()
    mate_b, st_b = M.run()  # second run: rows already sorted
    M.close()
    _certify(g, mate, st)
    np.testing.assert_array_equal(mate, mate_b)
    assert st["ms_sort"] >= 0 and st_b["ms_sort"] == 0


def test_dist_two_ranks_rmat_s26(lm):
    """The library-owned partitioned driver at full size: P = 2 ranks (threads on this GPU, plain
    device pointers, device-side barriers), each holding half of R-MAT scale 26."""
    import paper_conf_sc_mandulakgfhs24_b200.dist as D
    g = graphgen.rmat(26, 16, seed=1)
    mate, st, sts = D.match_dist_threads(g.offsets, g.col, g.w, 2)
    _certify(g, mate, {"weight": st.weight, "cardinality": st.cardinality})
    assert all(s.weight == st.weight for s in sts)


@pytest.mark.skipif(os.environ.get("LMATCH_HUGE") != "1", reason="set LMATCH_HUGE=1 (~5 min, ~150 GB host RAM)")
def test_rmat_s29_resident(lm):
    """R-MAT scale 29 (16.99e9 directed entries > 2^33) resident on one GPU: the CSR is assembled
    in pinned host memory (device CSR + packed keys would exceed HBM) as bench.py does."""
    import graphgen.gpu as gg
    if _host_ram_gb() < 150:
        pytest.skip("needs ~150 GB of host RAM")
    import torch
    dg = gg.rmat(29, 16, seed=1, host_out=True)
    assert dg.m > 2 ** 33
    g = graphgen.Graph(dg.offsets.numpy(), dg.col.numpy(), dg.w.numpy())
    torch.cuda.empty_cache()  # the generator's device scratch: the handle needs ~161 GB of HBM
    with lm.Matcher(g) as M:
        mate, st = M.run()
    _certify(g, mate, st)


def test_gradient_mesh_8192_ld_push(lm):
    """configs[2]'s many-round variant at full size on the LD path (SURVEY 8(d) C3 gradient:
    ~2 x 8192 pointing phases): the A6 push frontier keeps every round O(new matches) instead of
    O(live list), so the 16K-round run finishes in about a second; certificate + oracle weight."""
    import torch
    import graphgen.gpu as gg
    dg = gg.mesh(8192, seed=1, weights="gradient", device=torch.device("cuda"))
    g = graphgen.Graph(dg.offsets.cpu().numpy(), dg.col.cpu().numpy(), dg.w.cpu().numpy())
    M = lm.Matcher.from_device(dg.offsets, dg.col, dg.w, dg.n, dg.m, stream=torch.cuda.current_stream())
    del dg
    torch.cuda.empty_cache()
    mate, st = M.run()
    pushed = M.push_rounds()
    M.close()
    assert st["rounds"] > 8000 and pushed > 8000
    _certify(g, mate, st)
