"""GPU versions of the graphgen generators (bit-identical to the CPU ones by construction: both
compile gg_common.h).  Used by bench.py and the GPU tests to build large inputs quickly; outputs
are torch CUDA tensors (offsets int64[n+1], col int32[m], w float32[m]).  Input preparation only.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libgraphgen_cuda.so")
_SRCS = [os.path.join(_HERE, f) for f in ("graphgen_cuda.cu", "gg_common.h")]
_lib = None

WEIGHT_MODES = {"uniform": 0, "paper": 1, "gradient": 2, "ones": 3}
INT64_MAX = (1 << 63) - 1


def build(force: bool = False) -> str:
    stale = not os.path.exists(_SO) or any(os.path.getmtime(_SO) < os.path.getmtime(s) for s in _SRCS)
    if force or stale:
        cmd = ["nvcc", "-O3", "-std=c++17", "-fmad=false", "-gencode",
               "arch=compute_100a,code=sm_100a", "-Xcompiler", "-fPIC", "-shared",
               _SRCS[0], "-o", _SO + ".tmp"]
        subprocess.check_call(cmd)
        os.replace(_SO + ".tmp", _SO)
    return _SO


def _load():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_SO)
        i64, i32, u64, f64, p = ctypes.c_int64, ctypes.c_int, ctypes.c_uint64, ctypes.c_double, ctypes.c_void_p
        L.gg_cuda_count.argtypes = [i32, i64, i32, u64, f64, f64, f64, i64, i32, i32, p, p]
        L.gg_cuda_emit.argtypes = [i32, i64, i32, u64, f64, f64, f64, i64, i64, i64, p, p, p]
        L.gg_cuda_temp_bytes.argtypes = [i64]
        L.gg_cuda_temp_bytes.restype = i64
        L.gg_cuda_sort_unique.argtypes = [p, p, i64, i32, i32, p, i64, p, ctypes.POINTER(i32), p]
        L.gg_cuda_scatter.argtypes = [p, i64, i64, u64, i32, p, p, p, p]
        L.gg_cuda_scatter_local.argtypes = [p, i64, i64, u64, i32, p, p, p, p]
        L.gg_cuda_mesh_deg.argtypes = [i64, i32, u64, p, p]
        L.gg_cuda_mesh_fill.argtypes = [i64, i32, u64, p, p, p, u64, i32, p]
        for f in ("gg_cuda_count", "gg_cuda_emit", "gg_cuda_sort_unique", "gg_cuda_scatter",
                  "gg_cuda_scatter_local",
                  "gg_cuda_mesh_deg", "gg_cuda_mesh_fill"):
            getattr(L, f).restype = i32
        _lib = L
    return _lib


@dataclass
class DeviceGraph:
    offsets: "object"  # torch int64 [n+1]
    col: "object"      # torch int32 [m]
    w: "object"        # torch float32 [m]
    n: int
    m: int
    name: str = "graph"

    @property
    def m_u(self) -> int:
        return self.m // 2

    def to_host(self, pin: bool = False):
        """graphgen.Graph with numpy arrays (optionally backed by pinned memory)."""
        import graphgen
        arrs = []
        for t in (self.offsets, self.col, self.w):
            h = t.cpu() if not pin else t.to("cpu", non_blocking=False).pin_memory()
            arrs.append(h.numpy())
        return graphgen.Graph(arrs[0], arrs[1], arrs[2], name=self.name)


def _ck(rc, what):
    if rc != 0:
        raise RuntimeError(f"{what} failed with CUDA error {rc}")


def _edge_graph(kind, n, scale, M, seed, a, b, c, weights, wseed, device, bucket_entries, name,
                host_out=False):
    """host_out: col/w (and offsets) are assembled bucket by bucket in PINNED HOST memory, so
    graphs whose CSR cannot sit on the device next to the matcher's packed keys can be built."""
    import torch
    L = _load()
    dev = torch.device(device)
    st = torch.cuda.current_stream(dev).cuda_stream
    bits = max(1, (n - 1).bit_length())
    nb = 1
    while nb < 4096 and nb * bucket_entries < 2 * M and (nb << 1) <= (1 << bits):
        nb <<= 1
    shift = bits - (nb.bit_length() - 1)
    counts = torch.zeros(nb, dtype=torch.int64, device=dev)
    _ck(L.gg_cuda_count(kind, n, scale, seed, a, b, c, M, shift, nb, counts.data_ptr(), st), "count")
    counts_h = counts.cpu().tolist()
    total, maxc = sum(counts_h), max(counts_h) if counts_h else 0
    keys = torch.empty(max(maxc, 1), dtype=torch.int64, device=dev)
    alt = torch.empty(max(maxc, 1), dtype=torch.int64, device=dev)
    temp = torch.empty(max(L.gg_cuda_temp_bytes(max(maxc, 1)), 1), dtype=torch.uint8, device=dev)
    if host_out:
        col = torch.empty(max(total, 1), dtype=torch.int32, pin_memory=True)
        w = torch.empty(max(total, 1), dtype=torch.float32, pin_memory=True)
        col_b = torch.empty(max(maxc, 1), dtype=torch.int32, device=dev)
        w_b = torch.empty(max(maxc, 1), dtype=torch.float32, device=dev)
    else:
        col = torch.empty(max(total, 1), dtype=torch.int32, device=dev)
        w = torch.empty(max(total, 1), dtype=torch.float32, device=dev)
    first = torch.full((n + 1,), INT64_MAX, dtype=torch.int64, device=dev)
    cur = torch.zeros(1, dtype=torch.int64, device=dev)
    nout = torch.zeros(1, dtype=torch.int64, device=dev)
    mode = WEIGHT_MODES[weights]
    ws = seed if wseed is None else wseed
    base = 0
    which = ctypes.c_int(0)
    for bkt in range(nb):
        if counts_h[bkt] == 0:
            continue
        lo, hi = bkt << shift, min(n, (bkt + 1) << shift)
        cur.zero_()
        _ck(L.gg_cuda_emit(kind, n, scale, seed, a, b, c, M, lo, hi, keys.data_ptr(),
                           cur.data_ptr(), st), "emit")
        _ck(L.gg_cuda_sort_unique(keys.data_ptr(), alt.data_ptr(), counts_h[bkt], 0, 32 + bits,
                                  temp.data_ptr(), temp.numel(), nout.data_ptr(),
                                  ctypes.byref(which), st), "sort_unique")
        cu = int(nout.item())
        src = keys if which.value == 0 else alt
        if host_out:
            _ck(L.gg_cuda_scatter_local(src.data_ptr(), cu, base, ws, mode, col_b.data_ptr(),
                                        w_b.data_ptr(), first.data_ptr(), st), "scatter")
            col[base:base + cu].copy_(col_b[:cu])
            w[base:base + cu].copy_(w_b[:cu])
        else:
            _ck(L.gg_cuda_scatter(src.data_ptr(), cu, base, ws, mode, col.data_ptr(),
                                  w.data_ptr(), first.data_ptr(), st), "scatter")
        base += cu
    del keys, alt, temp
    if host_out:
        del col_b, w_b
    m = base
    first[n] = m
    offsets = torch.flip(torch.cummin(torch.flip(first, [0]), 0).values, [0]).contiguous()
    if host_out:
        del first
        offsets_h = torch.empty(n + 1, dtype=torch.int64, pin_memory=True)
        offsets_h.copy_(offsets)
        offsets = offsets_h
    torch.cuda.synchronize(dev)
    return DeviceGraph(offsets, col[:m], w[:m], n, m, name)


def _edge_graph_rows(kind, n, scale, M, seed, a, b, c, weights, wseed, device, bucket_entries, name,
                     rows=None, offsets=None, host_out=False):
    """Row-range generation for one rank of a partitioned run (each rank holds only its rows):
    rows=None -> pass 1: the graph's full CSR offsets (torch int64[n+1] on `device`; col/w of each
    bucket go to scratch and are dropped); rows=(v0, v1) with the pass-1 offsets -> pass 2: the
    local CSR of rows [v0, v1) (offsets rebased to 0, GLOBAL column ids), generating only the
    buckets that hold those rows.  Same edges and weights as _edge_graph (same kernels).
    host_out (pass 2): the local CSR is assembled in pinned host memory (a rank whose rows and
    the matcher's packed keys would not fit in HBM together)."""
    import torch
    L = _load()
    dev = torch.device(device)
    st = torch.cuda.current_stream(dev).cuda_stream
    bits = max(1, (n - 1).bit_length())
    nb = 1
    while nb < 4096 and nb * bucket_entries < 2 * M and (nb << 1) <= (1 << bits):
        nb <<= 1
    shift = bits - (nb.bit_length() - 1)
    counts = torch.zeros(nb, dtype=torch.int64, device=dev)
    _ck(L.gg_cuda_count(kind, n, scale, seed, a, b, c, M, shift, nb, counts.data_ptr(), st), "count")
    counts_h = counts.cpu().tolist()
    maxc = max(counts_h) if counts_h else 0
    keys = torch.empty(max(maxc, 1), dtype=torch.int64, device=dev)
    alt = torch.empty(max(maxc, 1), dtype=torch.int64, device=dev)
    temp = torch.empty(max(L.gg_cuda_temp_bytes(max(maxc, 1)), 1), dtype=torch.uint8, device=dev)
    col_b = torch.empty(max(maxc, 1), dtype=torch.int32, device=dev)
    w_b = torch.empty(max(maxc, 1), dtype=torch.float32, device=dev)
    first = torch.full((n + 1,), INT64_MAX, dtype=torch.int64, device=dev)
    cur = torch.zeros(1, dtype=torch.int64, device=dev)
    nout = torch.zeros(1, dtype=torch.int64, device=dev)
    mode = WEIGHT_MODES[weights]
    ws = seed if wseed is None else wseed
    which = ctypes.c_int(0)
    if rows is not None:
        v0, v1 = int(rows[0]), int(rows[1])
        offs_h = offsets.cpu() if offsets.is_cuda else offsets
        S, E = int(offs_h[v0]), int(offs_h[v1])
        odev = "cpu" if host_out else dev
        col = torch.empty(max(E - S, 1), dtype=torch.int32, device=odev, pin_memory=host_out)
        w = torch.empty(max(E - S, 1), dtype=torch.float32, device=odev, pin_memory=host_out)
    base = 0
    for bkt in range(nb):
        if counts_h[bkt] == 0:
            continue
        lo, hi = bkt << shift, min(n, (bkt + 1) << shift)
        if rows is not None:
            if hi <= v0 or lo >= v1:
                continue
            base = int(offs_h[lo])
        cur.zero_()
        _ck(L.gg_cuda_emit(kind, n, scale, seed, a, b, c, M, lo, hi, keys.data_ptr(),
                           cur.data_ptr(), st), "emit")
        _ck(L.gg_cuda_sort_unique(keys.data_ptr(), alt.data_ptr(), counts_h[bkt], 0, 32 + bits,
                                  temp.data_ptr(), temp.numel(), nout.data_ptr(),
                                  ctypes.byref(which), st), "sort_unique")
        cu = int(nout.item())
        src = keys if which.value == 0 else alt
        _ck(L.gg_cuda_scatter_local(src.data_ptr(), cu, base, ws, mode, col_b.data_ptr(),
                                    w_b.data_ptr(), first.data_ptr(), st), "scatter")
        if rows is None:
            base += cu
        else:
            g0, g1 = max(base, S), min(base + cu, E)
            if g1 > g0:
                col[g0 - S:g1 - S].copy_(col_b[g0 - base:g1 - base])
                w[g0 - S:g1 - S].copy_(w_b[g0 - base:g1 - base])
    del keys, alt, temp, col_b, w_b
    if rows is None:
        first[n] = base
        offsets = torch.flip(torch.cummin(torch.flip(first, [0]), 0).values, [0]).contiguous()
        torch.cuda.synchronize(dev)
        return offsets
    del first
    loff = (offsets[v0:v1 + 1].to("cpu" if host_out else dev) - S).contiguous()
    torch.cuda.synchronize(dev)
    return DeviceGraph(loff, col[:E - S], w[:E - S], v1 - v0, E - S, name + f"_rows{v0}-{v1}")


def rmat_offsets(scale: int, edgefactor: int = 16, seed: int = 1, a: float = 0.57, b: float = 0.19,
                 c: float = 0.19, device="cuda", bucket_entries: int = 1 << 28):
    """CSR offsets (torch int64[n+1] on `device`) of rmat(scale, edgefactor, seed, ...)."""
    n = 1 << scale
    return _edge_graph_rows(1, n, scale, edgefactor * n, seed, a, b, c, "uniform", None, device,
                            bucket_entries, f"rmat_s{scale}_ef{edgefactor}")


def rmat_rows(scale: int, v0: int, v1: int, offsets, edgefactor: int = 16, seed: int = 1,
              a: float = 0.57, b: float = 0.19, c: float = 0.19, weights: str = "uniform",
              wseed: int | None = None, device="cuda", bucket_entries: int = 1 << 28,
              host_out: bool = False) -> DeviceGraph:
    """Rows [v0, v1) of rmat(scale, ...) as a local CSR (global column ids); `offsets` from
    rmat_offsets.  n / m of the result are the LOCAL row and entry counts.  host_out: pinned CPU
    tensors (built on the GPU)."""
    n = 1 << scale
    return _edge_graph_rows(1, n, scale, edgefactor * n, seed, a, b, c, weights, wseed, device,
                            bucket_entries, f"rmat_s{scale}_ef{edgefactor}", (v0, v1), offsets,
                            host_out)


def er_offsets(n: int, avg_degree: float = 16.0, seed: int = 1, device="cuda",
               bucket_entries: int = 1 << 28):
    M = int(round(n * avg_degree / 2.0))
    return _edge_graph_rows(0, n, 0, M, seed, 0.0, 0.0, 0.0, "uniform", None, device, bucket_entries,
                            f"er_n{n}_d{avg_degree:g}")


def er_rows(n: int, v0: int, v1: int, offsets, avg_degree: float = 16.0, seed: int = 1,
            weights: str = "uniform", wseed: int | None = None, device="cuda",
            bucket_entries: int = 1 << 28) -> DeviceGraph:
    M = int(round(n * avg_degree / 2.0))
    return _edge_graph_rows(0, n, 0, M, seed, 0.0, 0.0, 0.0, weights, wseed, device, bucket_entries,
                            f"er_n{n}_d{avg_degree:g}", (v0, v1), offsets)


def rmat(scale: int, edgefactor: int = 16, seed: int = 1, a: float = 0.57, b: float = 0.19,
         c: float = 0.19, weights: str = "uniform", wseed: int | None = None, device="cuda",
         bucket_entries: int = 1 << 28, host_out: bool = False) -> DeviceGraph:
    """host_out=True: offsets/col/w come back as pinned CPU tensors (built on the GPU)."""
    n = 1 << scale
    return _edge_graph(1, n, scale, edgefactor * n, seed, a, b, c, weights, wseed, device,
                       bucket_entries, f"rmat_s{scale}_ef{edgefactor}", host_out)


def er(n: int, avg_degree: float = 16.0, seed: int = 1, weights: str = "uniform",
       wseed: int | None = None, device="cuda", bucket_entries: int = 1 << 28) -> DeviceGraph:
    M = int(round(n * avg_degree / 2.0))
    return _edge_graph(0, n, 0, M, seed, 0.0, 0.0, 0.0, weights, wseed, device, bucket_entries,
                       f"er_n{n}_d{avg_degree:g}")


def mesh(side: int, keep: float = 1.0, seed: int = 1, weights: str = "uniform",
         wseed: int | None = None, device="cuda") -> DeviceGraph:
    import torch
    L = _load()
    dev = torch.device(device)
    st = torch.cuda.current_stream(dev).cuda_stream
    n = side * side
    kp = int(round(keep * 1000))
    deg = torch.empty(n, dtype=torch.int64, device=dev)
    _ck(L.gg_cuda_mesh_deg(side, kp, seed, deg.data_ptr(), st), "mesh_deg")
    offsets = torch.zeros(n + 1, dtype=torch.int64, device=dev)
    offsets[1:] = torch.cumsum(deg, 0)
    m = int(offsets[-1].item())
    col = torch.empty(max(m, 1), dtype=torch.int32, device=dev)
    w = torch.empty(max(m, 1), dtype=torch.float32, device=dev)
    _ck(L.gg_cuda_mesh_fill(side, kp, seed, offsets.data_ptr(), col.data_ptr(), w.data_ptr(),
                            seed if wseed is None else wseed, WEIGHT_MODES[weights], st), "mesh_fill")
    torch.cuda.synchronize(dev)
    return DeviceGraph(offsets, col[:m], w[:m], n, m,
                       f"mesh_{side}x{side}" + ("" if keep >= 1 else f"_keep{keep:g}"))
