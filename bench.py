#!/usr/bin/env python
"""bench.py -- matching edges/s (GTEPS) and % HBM roofline of the B200 LD-matching path.

One step = one full matching (lmatch_run_device: reset, round-1 sweep, every frontier round,
mate[] + w(M)) of a resident synthetic graph shaped like the paper's workloads (BASELINE.json
configs; recipe in DESIGN.md).  GTEPS = undirected input edges m_u / step time / 1e9.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--workload rmat|er|mesh|road|gradient]
                  [--scale S] [--impl ours|reference]

N > 1 (torchrun, one rank per GPU; `--gpus N` alone self-launches torchrun): strong scaling on
ONE graph, 1-D edge-balanced vertex partition; each rank generates only its rows
and the library-owned driver (lmatch_create_dist / lmatch_run_dist) exchanges claims, changed
matched-bitmap words and frontier sizes through peer memory with device-side barriers
(--exchange p2p|nccl select the Python-driven alternatives).  `--partitioned` runs that path at N=1.

--impl reference: the oracle (sequential greedy = the same unique matching) on the host cores,
on a bounded sample of the workload (a smaller instance of the same generator recipe).
Prints ONE JSON line on rank 0.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

METRIC = "matching edges/s (GTEPS)"
UNIT = "GTEPS"


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=20)
    p.add_argument("--warmup", type=int, default=3)
    p.add_argument("--impl", default="ours", choices=["ours", "reference"])
    p.add_argument("--workload", default="rmat", choices=["rmat", "er", "mesh", "road", "gradient"])
    p.add_argument("--scale", type=int, default=None, help="log2(n) (rmat/er) or log2(n) of mesh")
    p.add_argument("--edgefactor", type=int, default=16)
    p.add_argument("--seed", type=int, default=1)
    p.add_argument("--weights", default=None)
    p.add_argument("--e2e-steps", type=int, default=3)
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--no-cpu", action="store_true")
    p.add_argument("--cpu-scale", type=int, default=None)
    p.add_argument("--gen", default="gpu", choices=["cpu", "gpu"])
    p.add_argument("--hbm-budget-gb", type=float, default=0.0,
                   help="out-of-core (A8): cap the HBM-resident adjacency; the rest is streamed "
                        "from pinned host memory in round 1 and read zero-copy afterwards")
    p.add_argument("--stream-chunk", type=int, default=0, help="entries per streamed chunk (0 = default)")
    p.add_argument("--prune", action="store_true", help="A7 in-place pruning (lmatch_opts.prune)")
    p.add_argument("--batches", type=int, default=0,
                   help="paper-style batch count N_i (lmatch_opts.batches): B > 1 streams the whole "
                        "adjacency from pinned host memory as B batches in round 1")
    p.add_argument("--key-cache", action="store_true",
                   help="resident: the round-1 top-4 key cache (lmatch_opts.key_cache = 1; off by default)")
    p.add_argument("--frontier", default="auto", choices=["auto", "pull", "push"],
                   help="A6 next frontier in the persistent-kernel rounds: auto = pull, switching to "
                        "push on many-round graphs (lmatch_opts.frontier = 0); pull = pull only")
    p.add_argument("--residual-mb", type=int, default=0,
                   help="out of core: MiB of HBM for copies of rescanned host rows (lmatch_opts.residual_mb)")
    p.add_argument("--no-host-cache", action="store_true",
                   help="out-of-core: disable the top-8 host-row key cache (lmatch_opts.host_cache = -1)")
    p.add_argument("--algorithm", default="ld", choices=["ld", "suitor", "hybrid", "sorted"],
                   help="ld = the pointer-based locally dominant iteration (the paper's method); "
                        "suitor = Suitor proposals with atomicMax (NEXT-4, same unique result); "
                        "hybrid = ld, with a Suitor tail after 32 pointing phases; "
                        "sorted = ld over rows sorted once per graph + per-vertex cursors (NEXT-3; "
                        "the sort runs in the first warm-up step and is reported as sort_ms_once)")
    p.add_argument("--exchange", default="dist", choices=["dist", "p2p", "nccl"],
                   help="partitioned path: dist = the library-owned driver (lmatch_create_dist / "
                        "lmatch_run_dist: peer-memory exchange + device-side barriers); p2p = the same "
                        "exchange (lmatch_p2p_*) driven from Python with event barriers; nccl = "
                        "torch.distributed all-to-all + allgather + allreduce (TorchTransport)")
    p.add_argument("--partitioned", action="store_true",
                   help="use the 1-D partitioned path even at N=1 (it is always used for N>1)")
    return p.parse_args()


DEFAULT_SCALE = {"rmat": 26, "er": 26, "mesh": 26, "road": 26, "gradient": 20}


def make_graph_cpu(a, scale, seed):
    import graphgen
    wl = a.workload
    if wl == "rmat":
        return graphgen.rmat(scale, a.edgefactor, seed=seed, weights=a.weights or "uniform")
    if wl == "er":
        return graphgen.er(1 << scale, float(a.edgefactor), seed=seed, weights=a.weights or "uniform")
    side = 1 << (scale // 2)
    if wl == "mesh":
        return graphgen.mesh(side, seed=seed, weights=a.weights or "uniform")
    if wl == "road":
        return graphgen.mesh(side, keep=0.6, seed=seed, weights=a.weights or "uniform")
    return graphgen.mesh(side, seed=seed, weights="gradient")


def host_assembly_needed(a, scale, device) -> bool:
    """True when the generated device CSR (8 B/entry) plus the matcher's packed keys (8 B/entry)
    and per-vertex state would not fit in HBM together (R-MAT s29 on one B200): the generator
    then assembles the CSR in pinned host memory and the handle is created from host arrays."""
    import torch
    if a.workload != "rmat" or a.hbm_budget_gb > 0:
        return False
    n = 1 << scale
    est = 2 * a.edgefactor * n
    hbm = torch.cuda.get_device_properties(device).total_memory
    return 16 * est + 48 * n > 0.85 * hbm


def make_graph_gpu(a, scale, seed, device, host_out=False):
    import graphgen.gpu as gg
    wl = a.workload
    if wl == "rmat":
        return gg.rmat(scale, a.edgefactor, seed=seed, weights=a.weights or "uniform", device=device,
                       host_out=host_out)
    if wl == "er":
        return gg.er(1 << scale, float(a.edgefactor), seed=seed, weights=a.weights or "uniform",
                     device=device)
    side = 1 << (scale // 2)
    if wl == "mesh":
        return gg.mesh(side, seed=seed, weights=a.weights or "uniform", device=device)
    if wl == "road":
        return gg.mesh(side, keep=0.6, seed=seed, weights=a.weights or "uniform", device=device)
    return gg.mesh(side, seed=seed, weights="gradient", device=device)


def workload_config(a, scale, n, m):
    cfg = {"workload": {"rmat": "R-MAT/Graph500 (A,B,C=.57,.19,.19), random relabel",
                        "er": "Erdos-Renyi", "mesh": "2-D 4-neighbour mesh",
                        "road": "road-like mesh (60% of grid edges kept)",
                        "gradient": "2-D mesh, gradient weights (many rounds)"}[a.workload],
           "scale": scale, "n": int(n), "m_directed": int(m), "m_undirected": int(m // 2),
           "weights": a.weights or ("gradient" if a.workload == "gradient" else "uniform fp32 (2^24 levels)"),
           "seed": a.seed}
    if a.workload in ("rmat", "er"):
        cfg["edgefactor"] = a.edgefactor
    if getattr(a, "prune", False):
        cfg["prune"] = True
    if getattr(a, "algorithm", "ld") != "ld":
        cfg["algorithm"] = a.algorithm
    if getattr(a, "frontier", "auto") != "auto":
        cfg["frontier"] = a.frontier
    return cfg


# ----------------------------------------------------------------------------- clocks (NVML)
class ClockSampler:
    REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap",
               0x8: "hw_slowdown", 0x10: "sync_boost", 0x20: "sw_thermal_slowdown",
               0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown",
               0x100: "display_clock_setting"}

    def __init__(self, device_index: int, period_s: float = 0.005):
        self.ok = False
        self.samples, self.reasons = [], 0
        self.period = period_s
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(device_index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception as e:  # pragma: no cover
            self.err = str(e)

    def _loop(self):
        nv = self.nv
        while not self._stop.is_set():
            try:
                self.samples.append(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
                self.reasons |= nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
            except Exception:
                pass
            time.sleep(self.period)

    def __enter__(self):
        if self.ok:
            self._stop = threading.Event()
            self._t = threading.Thread(target=self._loop, daemon=True)
            self._t.start()
        return self

    def __exit__(self, *exc):
        if self.ok:
            self._stop.set()
            self._t.join()

    def summary(self):
        if not self.ok or not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"]}
        names = [v for k, v in self.REASONS.items() if self.reasons & k and v != "gpu_idle"]
        return {"sm_mhz": float(statistics.median(self.samples)), "sm_max_mhz": int(self.max_mhz),
                "reasons": names, "samples": len(self.samples)}


def load_peaks():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        d = json.load(open(path))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs: torch copy_ best of 10)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s; MEASURED_PEAKS.json absent)"


def load_traffic(config_key: str):
    """dram bytes per sweep launch from the committed ncu --set full summary, if it matches."""
    path = os.path.join(ROOT, "profiles", "sweep_traffic.json")
    try:
        d = json.load(open(path))
        e = d.get(config_key)
        return None if e is None else float(e["dram_bytes_per_launch"])
    except Exception:
        return None


def per_round_roofline(round_log, round_ms, tail_from, peak):
    """HBM roofline of every host-driven round >= 2 of the last timed step (and of the persistent
    tail as one entry): algorithmic bytes = 8 B per adjacency entry scanned (E_r) + 64 B per
    frontier vertex (F_r: bin entry 16, pointer write 8, list write 8, match: entry 8 + partner
    pointer 8 + bitmap 16) + 16 B per live vertex the compaction reads and writes (L_r) -- DESIGN.md
    section 7 -- over the round's device time (CUDA events on the launch stream)."""
    out = []
    rows = [list(map(int, r)) for r in round_log[1:]]  # rounds 2, 3, ...
    for i, ms in enumerate(round_ms):
        sel = rows[i:] if i == tail_from else rows[i:i + 1]
        if not sel or ms <= 0:
            continue
        F = sum(r[0] for r in sel)
        L = sum(r[1] for r in sel)
        E = sum(r[2] for r in sel)
        alg = 8 * E + 64 * F + 16 * L
        gbs = alg / (ms / 1e3) / 1e9
        out.append({"round": i + 2, "rounds": len(sel), "ms": round(float(ms), 4), "frontier": F,
                    "live": L, "entries": E, "algorithmic_bytes": alg, "achieved_gbs": round(gbs, 1),
                    "frac": round(gbs / peak, 3),
                    **({"persistent_tail": True} if i == tail_from else {})})
    return out


# ------------------------------------------------------------------------------ cpu baseline
def cpu_baseline(a, sample_scale):
    """The oracle (sequential greedy, single thread) on a bounded sample: a smaller instance of
    the same generator recipe.  Returns a dict in the bench's metric/unit."""
    import oracle
    g = make_graph_cpu(a, sample_scale, a.seed)
    oracle.threads(1)
    r = oracle.greedy(g)
    t = r.sort_s + r.scan_s
    return {"value": g.m_u / t / 1e9, "unit": UNIT, "cores": 1, "kind": "oracle",
            "sample": f"a SMALLER graph than this line's: {a.workload} scale {sample_scale} (n={g.n}, "
                      f"m_u={g.m_u}), same recipe/seed; greedy sort {r.sort_s:.2f}s + scan "
                      f"{r.scan_s:.2f}s, 1 thread, std::sort.  Sort-based GTEPS falls with size "
                      f"(O(m log m)), so at the line's scale the oracle would be somewhat slower",
            "seconds": t}


def cpu_sample_scale(a, baseline: bool = True):
    """cpu_baseline: ~10 s of single-core oracle work; reference-arm steps: ~2 s each."""
    if a.cpu_scale:
        return a.cpu_scale
    if baseline:
        return {"rmat": 22, "er": 22, "mesh": 22, "road": 22, "gradient": 18}[a.workload]
    return {"rmat": 20, "er": 20, "mesh": 20, "road": 20, "gradient": 18}[a.workload]


# ------------------------------------------------------------------------------ reference arm
def run_reference(a, rank, world):
    if rank != 0:
        return 0
    import oracle
    scale = cpu_sample_scale(a, baseline=False)
    g = make_graph_cpu(a, scale, a.seed)
    oracle.threads(1)
    for _ in range(a.warmup):
        oracle.greedy(g)
    t0 = time.perf_counter()
    tt = 0.0
    for _ in range(a.steps):
        r = oracle.greedy(g)
        tt += r.sort_s + r.scan_s
    wall = time.perf_counter() - t0
    val = g.m_u * a.steps / tt / 1e9
    line = {"impl": "reference", "metric": METRIC, "value": val, "unit": UNIT, "n_gpus": world,
            "steps": a.steps, "warmup": a.warmup, "ms_per_step": tt / a.steps * 1e3,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f32-compare",
            "data": "synthetic",
            "config": workload_config(a, scale, g.n, g.m) | {"sample_of_scale": a.scale or DEFAULT_SCALE[a.workload]},
            "cpu_baseline": {"value": val, "unit": UNIT, "cores": 1, "kind": "oracle",
                             "sample": f"{a.workload} scale {scale} instance of the workload recipe"},
            "e2e": {"value": val, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
            "wall_s": wall}
    print(json.dumps(line), flush=True)
    return 0


# ------------------------------------------------------------------- partitioned arm (N >= 1)
def gen_rank_rows(a, scale, rank, world, dev):
    """This rank's rows of the workload graph: the CSR offsets of the whole graph
    (pass 1 of the row-range generator), the edge-balanced bounds from the library's partitioner
    (lmatch_partition), then only the rank's rows [v0, v1) (pass 2).  Each rank holds its
    own rows only, so graphs larger than one GPU's HBM can be partitioned.  Meshes are cheap to
    generate whole and are sliced."""
    import torch
    import graphgen.gpu as gg
    import paper_conf_sc_mandulakgfhs24_b200.dist as D
    if a.workload in ("rmat", "er"):
        if a.workload == "rmat":
            offs = gg.rmat_offsets(scale, a.edgefactor, seed=a.seed, device=dev)
        else:
            offs = gg.er_offsets(1 << scale, float(a.edgefactor), seed=a.seed, device=dev)
        offs_h = offs.cpu().numpy()
        bounds = D.edge_balanced_bounds(offs_h, world)
        v0, v1 = int(bounds[rank]), int(bounds[rank + 1])
        m_loc = int(offs_h[v1] - offs_h[v0])
        # the rank's device CSR (8 B/entry) next to the matcher's packed keys (8 B/entry) and
        # per-vertex state must fit in HBM; else the rows are assembled in pinned host memory
        host_out = 16 * m_loc + 48 * (v1 - v0) > 0.85 * torch.cuda.get_device_properties(dev).total_memory
        if a.workload == "rmat":
            dg = gg.rmat_rows(scale, v0, v1, offs, a.edgefactor, seed=a.seed, weights=a.weights or "uniform",
                              device=dev, host_out=host_out)
        else:
            dg = gg.er_rows(1 << scale, v0, v1, offs, float(a.edgefactor), seed=a.seed,
                            weights=a.weights or "uniform", device=dev)
        del offs
        n, m = len(offs_h) - 1, int(offs_h[-1])
        return dg.offsets, dg.col, dg.w, v0, v1, bounds, n, m, offs_h
    g = make_graph_gpu(a, scale, a.seed, dev)
    offs_h = g.offsets.cpu().numpy()
    bounds = D.edge_balanced_bounds(offs_h, world)
    v0, v1 = int(bounds[rank]), int(bounds[rank + 1])
    s0, s1 = int(offs_h[v0]), int(offs_h[v1])
    lo = (g.offsets[v0:v1 + 1] - s0).contiguous()
    lc, lw = g.col[s0:s1].contiguous(), g.w[s0:s1].contiguous()
    del g
    torch.cuda.empty_cache()
    return lo, lc, lw, v0, v1, bounds, len(offs_h) - 1, int(offs_h[-1]), offs_h


def run_partitioned(a, rank, world, local, dev):
    """One graph, 1-D vertex partition over the N ranks: each rank owns an
    edge-balanced row range.  --exchange dist (default): the library-owned driver
    (lmatch_create_dist / lmatch_run_dist: claims, changed bitmap words and frontier sizes stored
    into the peers' memory by the library's kernels, device-side barriers, no host barrier);
    p2p: the same exchange driven from Python with host/event barriers (dist.run_parts_p2p);
    nccl: claims all-to-all + bitmap allgather + frontier allreduce through torch.distributed
    (TorchTransport).  Strong scaling: the graph is the same for every N."""
    import torch
    import torch.distributed as dist
    import paper_conf_sc_mandulakgfhs24_b200 as lm
    import paper_conf_sc_mandulakgfhs24_b200.dist as D

    scale = a.scale or DEFAULT_SCALE[a.workload]
    t0 = time.time()
    lo, lc, lw, v0, v1, bounds, n, m, offs_h = gen_rank_rows(a, scale, rank, world, dev)
    m_u = m // 2
    host = None
    if not lo.is_cuda:  # assembled in pinned host memory: create from host arrays
        lo, lc, lw = lo.numpy(), lc.numpy(), lw.numpy()
    if not a.no_e2e:
        host = tuple(x.cpu().numpy() if hasattr(x, "is_cuda") else x for x in (lo, lc, lw))
    n_nz_loc = int(np.count_nonzero(np.diff(offs_h[v0:v1 + 1])))
    del offs_h
    gen_s = time.time() - t0
    tr = None
    if a.exchange == "dist":
        obj = [D.dist_id_new() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        part = D.DistMatcher(lo, lc, lw, v0, n, rank, world, bounds, obj[0], device=dev, timing=True)
        d_mate = torch.empty(max(v1 - v0, 1), dtype=torch.int32, device=dev)
        stats_box = {}

        def run():
            mate, st = part.run_device(d_mate)
            stats_box["st"] = st
            return st

        def sweep_ms():
            return stats_box["st"].ms_sweep

        def launches_of():
            return stats_box["st"].kernel_launches
    else:
        part = D.LibPart(lo, lc, lw, v0, n, bounds, rank, device=dev, timing=True)
        tr = D.TorchTransport()
        if a.exchange == "p2p":
            D.connect_p2p_torch(part)
            D.connect_events_torch(part)
            barrier = D.barrier_torch_events([part], dist.new_group(backend="gloo"))
            run = lambda: D.run_parts_p2p([part], barrier, tr)  # noqa: E731
        else:
            run = lambda: D.run_parts([part], tr)  # noqa: E731

        def sweep_ms():
            return part.info()[1]

        launches_of = None
    stream = part.stream  # the stream every library kernel of this part is launched on
    del lo, lc, lw
    torch.cuda.empty_cache()

    def allmax(x):
        t = torch.tensor([float(x)], dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    def allgather(vals):
        t = torch.tensor([float(v) for v in vals], dtype=torch.float64)
        out = [torch.empty_like(t) for _ in range(world)]
        dist.all_gather(out, t)
        return [x.tolist() for x in out]

    for _ in range(a.warmup):
        res = run()
    torch.cuda.synchronize(dev)
    dist.barrier()
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    sw, launches = [], 0
    with ClockSampler(dev.index) as clk:
        torch.cuda.synchronize(dev)
        l0 = D.kernel_launch_count()
        ev0.record(stream)
        for _ in range(a.steps):
            res = run()
            sw.append(sweep_ms())
            if launches_of:
                launches += launches_of()
        ev1.record(stream)
        torch.cuda.synchronize(dev)
        if not launches_of:
            launches = D.kernel_launch_count() - l0
    ms = allmax(ev0.elapsed_time(ev1))
    ms_per_step = ms / a.steps
    value = m_u * a.steps / (ms / 1e3) / 1e9
    if a.exchange == "dist":
        rounds, card, weight = res.rounds, res.cardinality, res.weight
    else:
        rounds, card, weight = res.rounds, res.matched // 2, res.weight

    e2e = None
    if host is not None and a.e2e_steps > 0:
        cud = torch.cuda.cudart()
        for arr in host:
            if arr.nbytes:
                cud.cudaHostRegister(arr.ctypes.data, arr.nbytes, 0)
        mate_h = torch.empty(max(v1 - v0, 1), dtype=torch.int32, pin_memory=True)
        dist.barrier()
        t1 = time.perf_counter()
        for _ in range(a.e2e_steps):
            part.reload(*host)
            if a.exchange == "dist":
                mate_h[: v1 - v0].copy_(part.run_device(d_mate)[0])
            else:
                mate_h[: v1 - v0].copy_(run().mates[0])
        el = allmax(time.perf_counter() - t1)
        for arr in host:
            if arr.nbytes:
                cud.cudaHostUnregister(arr.ctypes.data)
        hb = sum(allgather([sum(x.nbytes for x in host)])[r][0] for r in range(world))
        e2e = {"value": m_u * a.e2e_steps / el / 1e9, "unit": UNIT,
               "h2d_bytes_per_step": int(hb), "d2h_bytes_per_step": int(4 * n),
               "steps": a.e2e_steps, "ms_per_step": el / a.e2e_steps * 1e3,
               "includes": "lmatch_reload of every rank's local CSR (H2D + pack + validate + index) "
                           "+ partitioned run + owned mate[] slices D2H"}

    # roofline of the dominant kernel: the slowest rank's round-1 sweep over ITS owned rows
    # (its own entries and non-empty rows; DESIGN.md section 7 bytes per entry / per row)
    mine = [float(np.mean(sw)), float(part.m_local), float(n_nz_loc)]
    allr = allgather(mine)
    worst = max(allr, key=lambda x: x[0])
    peak, peak_src = load_peaks()
    mine_tile = lm.lmatch_sweep_tile(getattr(part, "h", None))
    tile_w = int(allgather([mine_tile])[allr.index(worst)][0])
    ntiles_w = (worst[1] + tile_w - 1) // tile_w
    sweep_bytes = 8 * worst[1] + 16 * worst[2] + 4 * (ntiles_w + 1)
    achieved = sweep_bytes / (worst[0] / 1e3) / 1e9 if worst[0] > 0 else None
    roofline = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                "frac": (achieved / peak) if achieved else None, "traffic": None,
                "kernel": "k_sweep over the slowest rank's owned rows",
                "algorithmic_bytes_per_launch": int(sweep_bytes),
                "launch_ms": worst[0], "share_of_step": worst[0] / ms_per_step,
                "peak_source": peak_src}
    ms_all = [x[0] for x in allr]
    ent_all = [x[1] for x in allr]
    imbalance = {"entries_max_over_mean": max(ent_all) / max(np.mean(ent_all), 1.0),
                 "sweep_ms_max_over_mean": max(ms_all) / max(np.mean(ms_all), 1e-9),
                 "entries_per_rank": [int(x) for x in ent_all]}
    launches_all = sum(x[0] for x in allgather([launches]))
    if rank == 0:
        desc = {"dist": "the library-owned driver (lmatch_create_dist / lmatch_run_dist): claims, changed "
                        "bitmap words and frontier sizes stored into the peers' memory by the library's "
                        "kernels (CUDA IPC), device-side barriers between phases",
                "p2p": "claims / changed bitmap words / frontier sizes stored into the peers' memory by "
                       "the library's kernels (CUDA IPC, lmatch_p2p_*), interprocess-event barriers "
                       "driven from Python",
                "nccl": "claims all-to-all + bitmap allgather + frontier allreduce per round (NCCL)"}[a.exchange]
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": a.steps,
                "warmup": a.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
                "scaling": "strong", "vs_baseline": None, "dtype": "u64", "data": "synthetic",
                "config": workload_config(a, scale, n, m) | {
                    "parallelism": f"1-D edge-balanced vertex partition over {world} rank(s): " + desc,
                    "exchange": a.exchange,
                    "devices": torch.cuda.device_count(),
                    "l2": f"inputs larger than L2 (adjacency {8 * m / 1e9:.1f} GB total); no flush",
                    "gen_s": round(gen_s, 1), "part_bounds": [int(x) for x in bounds],
                    "generation": "per rank: whole-graph offsets, then only the rank's rows"},
                "roofline": roofline, "cpu_baseline": None, "e2e": e2e,
                "gpu_launches": int(launches_all), "clocks": clk.summary(), "rounds": int(rounds),
                "cardinality": int(card), "matched_weight": weight,
                "mmeps": card * a.steps / (ms / 1e3) / 1e6,
                "imbalance": imbalance}
        print(json.dumps(line), flush=True)
    part.close()
    dist.destroy_process_group()
    return 0


def self_launch(a):
    """`bench.py --gpus N` without torchrun: launch N ranks of this script through
    torch.distributed.run on 127.0.0.1 (ranks share GPUs round-robin when fewer are visible)."""
    import socket
    import subprocess
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={a.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


# -------------------------------------------------------------------------------- our arm
def main():
    a = parse()
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", str(a.gpus)))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if a.impl == "reference":
        return run_reference(a, rank, world)

    if a.gpus > 1 and "WORLD_SIZE" not in os.environ:
        return self_launch(a)
    import torch
    import torch.distributed as dist
    if not torch.cuda.is_available():
        raise SystemExit("bench.py needs a CUDA device (no CPU fallback)")
    if world > 1 or a.partitioned:
        dev = torch.device("cuda", local % torch.cuda.device_count())
        torch.cuda.set_device(dev)
        if "MASTER_ADDR" not in os.environ:  # single-process partitioned run
            os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT="29531", RANK="0", WORLD_SIZE="1")
        if a.exchange == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:  # the library moves the data; torch.distributed is only the control plane
            dist.init_process_group("gloo")
        return run_partitioned(a, rank, world, local, dev)
    torch.cuda.set_device(local)
    import paper_conf_sc_mandulakgfhs24_b200 as lm

    scale = a.scale or DEFAULT_SCALE[a.workload]
    seed = a.seed
    dev = torch.device("cuda", local)
    stream = torch.cuda.current_stream(dev)
    t0 = time.time()
    if a.gen == "cpu":
        g = make_graph_cpu(a, scale, seed)
        d_off = torch.from_numpy(g.offsets).to(dev)
        d_col = torch.from_numpy(g.col).to(dev)
        d_w = torch.from_numpy(g.w).to(dev)
        n, m, m_u = g.n, g.m, g.m_u
    else:
        host_out = host_assembly_needed(a, scale, dev)
        dg = make_graph_gpu(a, scale, seed, dev, host_out=host_out)
        n, m, m_u = dg.n, dg.m, dg.m_u
        if host_out:
            import graphgen
            g = graphgen.Graph(dg.offsets.numpy(), dg.col.numpy(), dg.w.numpy())
            d_off = d_col = d_w = None
        else:
            d_off, d_col, d_w = dg.offsets, dg.col, dg.w
            g = None
    gen_s = time.time() - t0
    torch.cuda.empty_cache()

    # handle built from the device CSR (or, when both do not fit in HBM, from the pinned host
    # CSR); create is untimed: P:179 excludes I/O, allocation, CSR construction and the transfer
    opts = lm.make_opts(validate_level=1, timing=1,
                        hbm_budget_bytes=int(a.hbm_budget_gb * 1e9), stream_chunk=a.stream_chunk,
                        prune=a.prune, host_cache=not a.no_host_cache,
                        batches=a.batches, algorithm=a.algorithm, key_cache=a.key_cache, residual_mb=a.residual_mb,
                        frontier=a.frontier)
    pinned_host = d_off is None
    if pinned_host:
        h = lm.lmatch_create_ex(g.offsets, g.col, g.w, n, m, opts)
    else:
        h = lm.lmatch_create_device(d_off, d_col, d_w, n, m, opts, stream)
    if g is None and not a.no_e2e:  # host copies for the end-to-end leg
        import graphgen
        g = graphgen.Graph(d_off.cpu().numpy(), d_col.cpu().numpy(), d_w.cpu().numpy())
    del d_off, d_col, d_w
    dg = None
    torch.cuda.empty_cache()
    d_mate = torch.empty(n, dtype=torch.int32, device=dev)

    sort_ms_once = None
    for i in range(a.warmup):
        stw = lm.lmatch_run_device(h, d_mate, stream)
        if i == 0 and a.algorithm == "sorted":
            sort_ms_once = stw.ms_sort
    torch.cuda.synchronize(dev)
    if world > 1:
        dist.barrier()
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    sweep_ms, launches, rounds, step_ms = [], 0, [], []
    with ClockSampler(local) as clk:
        torch.cuda.synchronize(dev)
        ev0.record(stream)
        for _ in range(a.steps):
            st = lm.lmatch_run_device(h, d_mate, stream)
            sweep_ms.append(st.ms_sweep)
            step_ms.append(st.ms_total)
            launches += st.kernel_launches
            rounds.append(st.rounds)
        ev1.record(stream)
        torch.cuda.synchronize(dev)
    ms = ev0.elapsed_time(ev1)
    if world > 1:
        t = torch.tensor([ms], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
        tot = torch.tensor([m_u], dtype=torch.float64, device=dev)
        dist.all_reduce(tot)
        total_mu = float(tot.item())
    else:
        total_mu = float(m_u)
    ms_per_step = ms / a.steps
    value = total_mu * a.steps / (ms / 1e3) / 1e9
    last = st.as_dict()

    # roofline of the dominant kernel: the round-1 sweep (one launch per step)
    info = lm.lmatch_info(h)
    n_nz = info["nonempty_rows"]
    tile = info.get("sweep_tile", 512)
    ntiles = (m + tile - 1) // tile
    sweep_bytes = 8 * m + 16 * n_nz + 4 * (ntiles + 1)  # keys + (start lo32, id, best) per row + tile index
    sweep_avg_ms = float(np.mean(sweep_ms))
    peak, peak_src = load_peaks()
    achieved = sweep_bytes / (sweep_avg_ms / 1e3) / 1e9
    key = f"{a.workload}_s{scale}_ef{a.edgefactor}_seed{a.seed}"
    roofline = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                "frac": achieved / peak, "traffic": load_traffic(key),
                "kernel": "k_sweep (round-1 pointer sweep, TMA-staged)",
                "algorithmic_bytes_per_launch": int(sweep_bytes), "launch_ms": sweep_avg_ms,
                "share_of_step": sweep_avg_ms / ms_per_step, "peak_source": peak_src}
    if a.algorithm == "sorted":
        # round-1 pointer kernel over sorted rows: per vertex offs[u+1] 8 B + first key 8 B +
        # cur/ptr writes 16 B (a row start is the previous row's end, read once)
        r1_bytes = 32 * n
        achieved = r1_bytes / (sweep_avg_ms / 1e3) / 1e9
        roofline.update({"achieved": achieved, "frac": achieved / peak, "traffic": None,
                         "kernel": "k_sc_point (round-1 cursor pointers over sorted rows)",
                         "algorithmic_bytes_per_launch": int(r1_bytes)})

    # end-to-end through the public C ABI with host buffers (pinned): reload + run + mate D2H
    e2e = None
    if not a.no_e2e and a.e2e_steps > 0:
        cud = torch.cuda.cudart()
        regs = []
        for arr in (g.offsets, g.col, g.w):
            if arr.nbytes and not pinned_host:
                cud.cudaHostRegister(arr.ctypes.data, arr.nbytes, 0)
                regs.append(arr)
        mate_h = torch.empty(n, dtype=torch.int32, pin_memory=True)
        mate_np = mate_h.numpy()
        lm.lmatch_reload(h, g.offsets, g.col, g.w)
        lm.lmatch_run(h, mate_np)
        torch.cuda.synchronize(dev)
        if world > 1:
            dist.barrier()
        t1 = time.perf_counter()
        for _ in range(a.e2e_steps):
            lm.lmatch_reload(h, g.offsets, g.col, g.w)
            lm.lmatch_run(h, mate_np)
        el = time.perf_counter() - t1
        if world > 1:
            t = torch.tensor([el], dtype=torch.float64, device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            el = float(t.item())
        for arr in regs:
            cud.cudaHostUnregister(arr.ctypes.data)
        e2e = {"value": total_mu * a.e2e_steps / el / 1e9, "unit": UNIT,
               "h2d_bytes_per_step": int(g.offsets.nbytes + g.col.nbytes + g.w.nbytes),
               "d2h_bytes_per_step": int(4 * n), "steps": a.e2e_steps,
               "ms_per_step": el / a.e2e_steps * 1e3,
               "includes": "lmatch_reload (H2D + pack + validate + index) + lmatch_run (+ mate D2H)"}

    ooc = None
    pcie_peak = None
    if a.hbm_budget_gb > 0 or a.batches > 1:
        # the bound of the streamed round: pinned H2D copy rate of this box (1 GiB, best of 3)
        src = torch.empty(1 << 30, dtype=torch.uint8, pin_memory=True)
        dst = torch.empty(1 << 30, dtype=torch.uint8, device=dev)
        best = 0.0
        for _ in range(3):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            dst.copy_(src, non_blocking=True)
            e1.record(stream)
            e1.synchronize()
            best = max(best, (1 << 30) / (e0.elapsed_time(e1) / 1e3) / 1e9)
        del src, dst
        pcie_peak = best
    if a.hbm_budget_gb > 0 or a.batches > 1:
        ooc = {"batches": a.batches,"hbm_budget_bytes": int(a.hbm_budget_gb * 1e9),
               "resident_entries": int(last["resident_entries"]),
               "resident_frac": last["resident_entries"] / max(m, 1),
               "bytes_streamed_per_step": int(last["bytes_streamed"]),
               "stream_gbs_in_sweep": last["bytes_streamed"] / max(sweep_avg_ms, 1e-9) / 1e6,
               "pcie_h2d_peak_gbs": pcie_peak,
               "pcie_frac_in_sweep": (last["bytes_streamed"] / max(sweep_avg_ms, 1e-9) / 1e6) / pcie_peak,
               "host_cache": not a.no_host_cache,
               "cache_bytes": int(last["cache_bytes"]),
               "cache_rows_per_step": int(last["cache_rows"]),
               "host_entries_read_per_step": int(last["host_entries_read"]),
               "residual_mb": a.residual_mb, "residual_rows_per_step": int(last["residual_rows"]),
               "note": "sweep = resident HBM tiles + host chunks over PCIe (2-slot ring); later "
                       "rounds read host rows zero-copy, except rows whose pointer the top-8 "
                       "host-row key cache decides (filled in round 1; NEXT-1)"}
    mate_last = d_mate.cpu().numpy() if (g is not None and not a.no_cpu and world == 1) else None
    round_log = lm.lmatch_round_log(h)
    rounds_roofline = per_round_roofline(round_log, *lm.lmatch_round_ms(h), load_peaks()[0])
    lm.lmatch_destroy(h)
    del d_mate
    torch.cuda.empty_cache()

    cpu = None
    if rank == 0 and world == 1 and not a.no_cpu:
        cpu = cpu_baseline(a, cpu_sample_scale(a))
        if g is not None and mate_last is not None:
            # the O(m) certificate (oracle/, all host cores) on THIS line's graph and result: a
            # verifier, not a baseline -- it checks the GPU's mate[] at full size and shows what
            # the host needs for one pass over the same adjacency
            import oracle
            oracle.threads(0)
            t0 = time.perf_counter()
            code, _ = oracle.certificate(g, mate_last)
            cert_s = time.perf_counter() - t0
            cpu["certificate_on_this_graph"] = {
                "ok": code == 0, "seconds": cert_s, "cores": os.cpu_count(),
                "gteps_equivalent": m_u / cert_s / 1e9,
                "kind": "verifier (C(M) holds iff mate[] is the unique LD matching), not a matcher"}

    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": a.steps,
                "warmup": a.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
                "scaling": "strong", "vs_baseline": None, "dtype": "u64",
                "data": "synthetic",
                "config": workload_config(a, scale, n, m) | {
                    "parallelism": "1 GPU (the same graph is partitioned over the GPUs at N > 1)",
                    "l2": f"inputs larger than L2 (adjacency {8 * m / 1e9:.1f} GB >> 126 MB); no flush",
                    "gen_s": round(gen_s, 1),
                    "csr_for_create": "pinned host (device CSR + packed keys exceed HBM)" if pinned_host
                                      else "device"},
                "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e,
                **({"out_of_core": ooc} if ooc else {}),
                "gpu_launches": int(launches), "clocks": clk.summary(),
                "rounds": int(rounds[-1]), "cardinality": int(last["cardinality"]),
                "entries_swept": int(last["entries_swept"]), "frontier_total": int(last["frontier_total"]),
                "round_log": round_log.tolist(),
                "rounds_roofline": rounds_roofline,
                "matched_weight": last["weight"],
                "mmeps": int(last["cardinality"]) * a.steps / (ms / 1e3) / 1e6,
                "mmeps_note": "MMEPS-like |M|/T (P:344-356 'rate at which edges are committed'): "
                              "matched edges per second of the timed steps, in millions",
                "step_ms": {"best": float(np.min(step_ms)), "median": float(np.median(step_ms)),
                            "best_gteps": total_mu / (float(np.min(step_ms)) / 1e3) / 1e9,
                            "note": "per-step device time from the library's own events "
                                    "(paper: best of ten, P:179); value uses the whole timed region"},
                "phase_ms": {k: last[k] for k in ("ms_sweep", "ms_round1_rest", "ms_rounds",
                                                  "ms_finish", "ms_total")}}
        if sort_ms_once is not None:
            line["sort_ms_once"] = sort_ms_once
            line["sort_note"] = ("rows sorted once per loaded graph in the first warm-up step, "
                                 "outside the timed steps; e2e (reload + run) pays it every step")
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
