"""Partitioned (multi-GPU) matching: 1-D vertex partition, pointer claims and a bitmap allgather.

SURVEY 8(e) / include/lmatch.h "Partitioned mode".  Every part owns a contiguous vertex range with
all its rows, balanced by directed entries (binary search on the CSR prefix sums).
One round (Alg. 2, with the exchange redesigned):

    pointers (owned rows)           lmatch_part_begin / lmatch_part_point    [library kernels]
    claims -> owner of the target   all-to-all      (replaces nccl_AllReduce(pointers))
    match                           lmatch_part_apply                        [library kernels]
    matched-bitmap slices           allgather       (replaces nccl_AllReduce(mate))
    compaction, frontier size       lmatch_part_compact                      [library kernels]
    termination                     allreduce of frontier sizes == 0

The round loop (`run_parts`) is written over a list of local parts and a transport:
  * `TorchTransport` -- one part per process, torch.distributed collectives (NCCL on GPUs; the
    same calls run on gloo with CPU tensors, which is how the CPU tests cover this driver);
  * `LocalTransport` -- several parts in one process (P logical partitions on one GPU), used to
    prove partition invariance of the result on a single device.
Data moves between parts only through the transport; the result is bit-identical to the
single-GPU run for every partition (Lemma III.1).
"""
from __future__ import annotations

import ctypes
from dataclasses import dataclass

import numpy as np

from . import _check, _dev_ptr, _lib, _P, _I64, make_opts, LMatchError  # noqa: F401

# ---------------------------------------------------------------------------- ctypes signatures
_sig = {
    "lmatch_create_part": ([_P, _P, _P, _I64, _I64, _I64, _I64, ctypes.c_int32, _P, _P,
                            ctypes.POINTER(_P)], ctypes.c_int),
    "lmatch_create_part_device": ([_P, _P, _P, _I64, _I64, _I64, _I64, ctypes.c_int32, _P, _P, _P,
                                   ctypes.POINTER(_P)], ctypes.c_int),
    "lmatch_part_begin": ([_P, _P, _P], ctypes.c_int),
    "lmatch_part_claims": ([_P, _P], ctypes.c_int),
    "lmatch_part_apply": ([_P, _P, _I64, _P], ctypes.c_int),
    "lmatch_part_bitmap": ([_P, _P, _P, _P, _P], ctypes.c_int),
    "lmatch_part_compact": ([_P, _P, ctypes.POINTER(_I64)], ctypes.c_int),
    "lmatch_part_point": ([_P, _P, _P], ctypes.c_int),
    "lmatch_part_finish": ([_P, _P, _P, ctypes.POINTER(ctypes.c_double), ctypes.POINTER(_I64)],
                           ctypes.c_int),
    "lmatch_part_get_claims": ([_P, ctypes.c_int32, _P, _P], ctypes.c_int),
    "lmatch_part_get_bits": ([_P, _P, _P], ctypes.c_int),
    "lmatch_part_set_bits": ([_P, _P, _I64, _I64, _P], ctypes.c_int),
    "lmatch_part_info": ([_P, ctypes.POINTER(_I64), ctypes.POINTER(ctypes.c_double)], ctypes.c_int),
    "lmatch_reload": ([_P, _P, _P, _P], ctypes.c_int),
    "lmatch_p2p_enable": ([_P, ctypes.c_int32], ctypes.c_int),
    "lmatch_p2p_attach_local": ([_P, ctypes.c_int32, _P], ctypes.c_int),
    "lmatch_p2p_export": ([_P, _P], ctypes.c_int),
    "lmatch_p2p_attach": ([_P, ctypes.c_int32, _P], ctypes.c_int),
    "lmatch_p2p_begin": ([_P, _P], ctypes.c_int),
    "lmatch_p2p_point": ([_P, _P], ctypes.c_int),
    "lmatch_p2p_match": ([_P, _P], ctypes.c_int),
    "lmatch_p2p_compact": ([_P, _P, ctypes.POINTER(_I64)], ctypes.c_int),
    "lmatch_p2p_frontier_total": ([_P, _P, ctypes.POINTER(_I64)], ctypes.c_int),
    "lmatch_p2p_sync": ([_P, _P], ctypes.c_int),
    "lmatch_kernel_launch_count": ([], _I64),
    "lmatch_partition": ([_P, _I64, ctypes.c_int32, ctypes.c_int32, _P], ctypes.c_int),
    "lmatch_dist_id_new": ([_P], ctypes.c_int),
    "lmatch_create_dist": ([_P, _P, _P, _I64, _I64, _I64, _I64, ctypes.c_int32, ctypes.c_int32, _P, _P,
                            _P, ctypes.POINTER(_P)], ctypes.c_int),
    "lmatch_create_dist_device": ([_P, _P, _P, _I64, _I64, _I64, _I64, ctypes.c_int32, ctypes.c_int32,
                                   _P, _P, _P, _P, ctypes.POINTER(_P)], ctypes.c_int),
    "lmatch_run_dist": ([_P, _P, _P], ctypes.c_int),
    "lmatch_run_dist_device": ([_P, _P, _P, _P], ctypes.c_int),
}
for _name, (_args, _res) in _sig.items():
    _f = getattr(_lib, _name)
    _f.argtypes = _args
    _f.restype = _res


# ------------------------------------------------------------------------------- partitioning
def edge_balanced_bounds(offsets: np.ndarray, nparts: int, align: int = 32) -> np.ndarray:
    """Contiguous vertex ranges with ~m/P directed entries each (binary search on the CSR prefix
    sums); every bound is a multiple of `align` (bitmap words are owned by one part).
    Computed by the library (lmatch_partition, host-only)."""
    offsets = np.ascontiguousarray(offsets, dtype=np.int64)
    n = offsets.shape[0] - 1
    b = np.zeros(nparts + 1, dtype=np.int64)
    _check(_lib.lmatch_partition(offsets.ctypes.data, n, int(nparts), int(align), b.ctypes.data),
           "lmatch_partition")
    return b


def dist_id_new() -> bytes:
    """64-byte rendezvous id for one lmatch_create_dist group (lmatch_dist_id_new)."""
    buf = ctypes.create_string_buffer(64)
    _check(_lib.lmatch_dist_id_new(buf), "lmatch_dist_id_new")
    return buf.raw


def part_words(bounds):
    """(first bitmap word, word count) owned by each part."""
    return [(int(bounds[p]) // 32, (int(bounds[p + 1]) - int(bounds[p]) + 31) // 32)
            for p in range(len(bounds) - 1)]


def local_csr(offsets, col, w, v0: int, v1: int):
    """Rows [v0, v1) with their global column ids (cut edges live in both owners' rows)."""
    offsets = np.asarray(offsets, dtype=np.int64)
    s, e = int(offsets[v0]), int(offsets[v1])
    return offsets[v0:v1 + 1] - s, np.asarray(col[s:e], dtype=np.int32), np.asarray(w[s:e], dtype=np.float32)


# --------------------------------------------------------------------------------- transports
class LocalTransport:
    """All parts live in this process (P logical partitions, e.g. on one GPU)."""

    def __init__(self, nparts: int):
        self.nparts = nparts

    def exchange(self, sends):
        import torch
        P = self.nparts
        return [torch.cat([sends[s][d] for s in range(P)]) for d in range(P)]

    def allgather(self, owns):
        return [list(owns) for _ in owns]

    def allreduce(self, xs):
        t = sum(int(x) for x in xs)
        return [t for _ in xs]


class TorchTransport:
    """One part per process; torch.distributed collectives (NCCL with CUDA tensors, gloo with
    CPU tensors).  Every rank calls every method in the same order."""

    def __init__(self, group=None):
        import torch.distributed as dist
        self.dist = dist
        self.group = group
        self.nparts = dist.get_world_size(group)
        self.rank = dist.get_rank(group)
        self._sizes = None  # owned bitmap word counts of every part (constant per run)
        # gloo moves CPU tensors only: CUDA tensors are staged through host memory
        self._host = dist.get_backend(group) == "gloo"

    def _wire(self, t):
        return t.cpu() if self._host and t.is_cuda else t

    def exchange(self, sends):
        import torch
        (send,) = sends
        dev = send[0].device
        wdev = "cpu" if self._host else dev
        cnt_out = torch.tensor([t.numel() for t in send], dtype=torch.int64, device=wdev)
        cnt_in = torch.empty_like(cnt_out)
        self.dist.all_to_all_single(cnt_in, cnt_out, group=self.group)
        in_splits = [t.numel() for t in send]
        out_splits = [int(c) for c in cnt_in.tolist()]
        recv = torch.empty(sum(out_splits), dtype=send[0].dtype, device=wdev)
        self.dist.all_to_all_single(recv, self._wire(torch.cat(list(send))), out_splits, in_splits,
                                    group=self.group)
        return [recv.to(dev)]

    def allgather(self, owns):
        import torch
        (own,) = owns
        dev = own.device
        wdev = "cpu" if self._host else dev
        if self._sizes is None:
            n = torch.tensor([own.numel()], dtype=torch.int64, device=wdev)
            sz = [torch.empty_like(n) for _ in range(self.nparts)]
            self.dist.all_gather(sz, n, group=self.group)
            self._sizes = [int(x.item()) for x in sz]
        sizes = self._sizes
        mx = max(sizes) if sizes else 0
        pad = torch.zeros(mx, dtype=own.dtype, device=wdev)
        pad[: own.numel()] = self._wire(own)
        out = torch.empty(self.nparts * mx, dtype=own.dtype, device=wdev)
        self.dist.all_gather_into_tensor(out, pad, group=self.group)
        out = out.to(dev)
        return [[out[p * mx: p * mx + sizes[p]] for p in range(self.nparts)]]

    def allreduce(self, xs):
        import torch
        (x,) = xs
        dev = "cuda" if self.dist.get_backend(self.group) == "nccl" else "cpu"
        t = torch.tensor([int(x)], dtype=torch.int64, device=dev)
        self.dist.all_reduce(t, group=self.group)
        return [int(t.item())]


# ------------------------------------------------------------------------- the GPU part backend
class LibPart:
    """One partition handle of liblmatch.so (rows [v0, v1) of a graph with n_global vertices)."""

    def __init__(self, offsets_local, col_local, w_local, v0: int, n_global: int, bounds,
                 part: int, device=None, stream=None, validate_level: int = 1, timing: bool = False,
                 **opt_kw):
        import torch
        self.torch = torch
        self.dev = torch.device("cuda") if device is None else torch.device(device)
        self.bounds = np.ascontiguousarray(bounds, dtype=np.int64)
        self.P = self.bounds.shape[0] - 1
        self.v0 = int(v0)
        self.part = int(part)
        self.n_local = int(len(offsets_local) - 1)
        self.n_global = int(n_global)
        # every call of this part (library kernels, torch copies of claims / bitmap words) is
        # ordered on ONE non-default stream (a NULL stream would make the library use its own
        # handle stream, unordered with torch's legacy default stream); tensors crossing to the
        # caller's stream are synchronised (producers) or waited for (consumers)
        if stream is None or stream.cuda_stream == 0:
            stream = torch.cuda.Stream(self.dev)
        self.stream = stream
        h = _P()
        # opt_kw: further lmatch_opts (make_opts names), e.g. hbm_budget_bytes / batches for a
        # part streamed from host memory (the paper's per-device batches N_i)
        opts = make_opts(validate_level=validate_level, timing=timing, **opt_kw)
        if hasattr(offsets_local, "is_cuda") and offsets_local.is_cuda:  # device CSR (torch)
            torch.cuda.current_stream(self.dev).synchronize()  # the arrays' producer
            self.m_local = int(col_local.numel())
            with torch.cuda.device(self.dev):
                _check(_lib.lmatch_create_part_device(
                    offsets_local.data_ptr(), col_local.data_ptr(), w_local.data_ptr(), self.n_local,
                    self.m_local, self.v0, self.n_global, self.P, self.bounds.ctypes.data,
                    ctypes.byref(opts), self._s(), ctypes.byref(h)), "lmatch_create_part_device")
        else:
            off = np.ascontiguousarray(offsets_local, dtype=np.int64)
            col = np.ascontiguousarray(col_local, dtype=np.int32)
            w = np.ascontiguousarray(w_local, dtype=np.float32)
            self.m_local = int(col.shape[0])
            with torch.cuda.device(self.dev):
                _check(_lib.lmatch_create_part(off.ctypes.data, col.ctypes.data, w.ctypes.data,
                                               self.n_local, self.m_local, self.v0, self.n_global,
                                               self.P, self.bounds.ctypes.data, ctypes.byref(opts),
                                               ctypes.byref(h)), "lmatch_create_part")
        self.h = h.value
        self.counts = np.zeros(self.P, dtype=np.int64)
        self.words = part_words(self.bounds)

    def _s(self):
        return self.stream.cuda_stream

    def _consume(self, t):
        """Order this part's stream after the caller's current stream, which produced `t`, and
        keep t's memory from being reused before this stream is done with it."""
        torch = self.torch
        self.stream.wait_stream(torch.cuda.current_stream(self.dev))
        t.record_stream(self.stream)

    def begin(self):
        _check(_lib.lmatch_part_begin(self.h, self._s(), self.counts.ctypes.data), "lmatch_part_begin")
        return self.counts.copy()

    def point(self):
        _check(_lib.lmatch_part_point(self.h, self._s(), self.counts.ctypes.data), "lmatch_part_point")
        return self.counts.copy()

    def claims(self, counts):
        torch = self.torch
        out = []
        with torch.cuda.stream(self.stream):
            for p in range(self.P):
                t = torch.empty(int(counts[p]), dtype=torch.int64, device=self.dev)
                if counts[p]:
                    _check(_lib.lmatch_part_get_claims(self.h, p, t.data_ptr(), self._s()),
                           "lmatch_part_get_claims")
                out.append(t)
        self.stream.synchronize()
        return out

    def apply(self, recv):
        if recv.numel():
            self._consume(recv)
        _check(_lib.lmatch_part_apply(self.h, recv.data_ptr() if recv.numel() else None,
                                      recv.numel(), self._s()), "lmatch_part_apply")

    def own_bits(self):
        with self.torch.cuda.stream(self.stream):
            t = self.torch.empty(self.words[self._me()][1], dtype=self.torch.int32, device=self.dev)
            if t.numel():
                _check(_lib.lmatch_part_get_bits(self.h, t.data_ptr(), self._s()),
                       "lmatch_part_get_bits")
        self.stream.synchronize()
        return t

    def set_bits(self, all_words):
        for p, t in enumerate(all_words):
            if p == self._me() or t.numel() == 0:
                continue
            src = t.to(self.dev).contiguous()
            self._consume(src)
            _check(_lib.lmatch_part_set_bits(self.h, src.data_ptr(), self.words[p][0], src.numel(),
                                             self._s()), "lmatch_part_set_bits")

    def reload(self, offsets_local, col_local, w_local):
        """Re-upload the same-shaped local CSR from host arrays (end-to-end timing)."""
        ptrs = [a.ctypes.data if isinstance(a, np.ndarray) else int(a)
                for a in (offsets_local, col_local, w_local)]
        _check(_lib.lmatch_reload(self.h, *ptrs), "lmatch_reload")

    def info(self):
        r, ms = _I64(), ctypes.c_double()
        _check(_lib.lmatch_part_info(self.h, ctypes.byref(r), ctypes.byref(ms)), "lmatch_part_info")
        return int(r.value), float(ms.value)

    def compact(self):
        nf = _I64()
        _check(_lib.lmatch_part_compact(self.h, self._s(), ctypes.byref(nf)), "lmatch_part_compact")
        return int(nf.value)

    def finish(self):
        torch = self.torch
        with torch.cuda.stream(self.stream):
            mate = torch.empty(max(self.n_local, 1), dtype=torch.int32, device=self.dev)
        w, c = ctypes.c_double(), _I64()
        _check(_lib.lmatch_part_finish(self.h, mate.data_ptr(), self._s(), ctypes.byref(w),
                                       ctypes.byref(c)), "lmatch_part_finish")
        return mate[: self.n_local], float(w.value), int(c.value)

    def _me(self):
        return self.part

    # ---- peer-memory exchange (include/lmatch.h "Peer-memory exchange")
    def p2p_enable(self):
        _check(_lib.lmatch_p2p_enable(self.h, self.part), "lmatch_p2p_enable")

    def p2p_attach_local(self, peer: int, other: "LibPart"):
        _check(_lib.lmatch_p2p_attach_local(self.h, int(peer), other.h), "lmatch_p2p_attach_local")

    def p2p_export(self) -> bytes:
        buf = ctypes.create_string_buffer(128)
        _check(_lib.lmatch_p2p_export(self.h, buf), "lmatch_p2p_export")
        return buf.raw

    def p2p_attach(self, peer: int, handles: bytes):
        buf = ctypes.create_string_buffer(bytes(handles), 128)
        _check(_lib.lmatch_p2p_attach(self.h, int(peer), buf), "lmatch_p2p_attach")

    def p2p_begin(self):
        _check(_lib.lmatch_p2p_begin(self.h, self._s()), "lmatch_p2p_begin")

    def p2p_point(self):
        _check(_lib.lmatch_p2p_point(self.h, self._s()), "lmatch_p2p_point")

    def p2p_match(self):
        _check(_lib.lmatch_p2p_match(self.h, self._s()), "lmatch_p2p_match")

    def p2p_compact(self, local_size: bool = False):
        """Compaction + frontier-size push; stream-ordered (no sync) unless local_size=True,
        which synchronises and returns this part's next frontier size."""
        if not local_size:
            _check(_lib.lmatch_p2p_compact(self.h, self._s(), None), "lmatch_p2p_compact")
            return None
        nf = _I64()
        _check(_lib.lmatch_p2p_compact(self.h, self._s(), ctypes.byref(nf)), "lmatch_p2p_compact")
        return int(nf.value)

    def p2p_frontier_total(self) -> int:
        t = _I64()
        _check(_lib.lmatch_p2p_frontier_total(self.h, self._s(), ctypes.byref(t)),
               "lmatch_p2p_frontier_total")
        return int(t.value)

    def p2p_sync(self):
        _check(_lib.lmatch_p2p_sync(self.h, self._s()), "lmatch_p2p_sync")

    def close(self):
        if self.h is not None:
            _lib.lmatch_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


# ------------------------------------------------------------- the library-owned driver (C ABI)
class DistMatcher:
    """One rank of a lmatch_create_dist group: the library partitions nothing itself here (the
    caller passes the rank's rows and the common bounds, e.g. from edge_balanced_bounds), opens
    the peers' exchange windows through the rendezvous `dist_id`, and runs the whole round loop
    with device-side barriers (include/lmatch.h "Library-owned multi-GPU driver")."""

    def __init__(self, offsets_local, col_local, w_local, v0: int, n_global: int, rank: int,
                 world: int, bounds, dist_id: bytes, device=None, stream=None, timing: bool = False,
                 max_rounds: int = 0, validate_level: int = 1, **opt_kw):
        import torch
        self.torch = torch
        self.dev = torch.device("cuda") if device is None else torch.device(device)
        self.bounds = np.ascontiguousarray(bounds, dtype=np.int64)
        self.rank, self.world = int(rank), int(world)
        self.v0, self.n_global = int(v0), int(n_global)
        self.n_local = int(len(offsets_local) - 1)
        if stream is None or stream.cuda_stream == 0:
            stream = torch.cuda.Stream(self.dev)
        self.stream = stream
        self._id = ctypes.create_string_buffer(bytes(dist_id)[:64], 64)
        opts = make_opts(validate_level=validate_level, timing=timing, max_rounds=max_rounds, **opt_kw)
        h = _P()
        with torch.cuda.device(self.dev):
            if hasattr(offsets_local, "is_cuda") and offsets_local.is_cuda:
                torch.cuda.current_stream(self.dev).synchronize()
                self.m_local = int(col_local.numel())
                _check(_lib.lmatch_create_dist_device(
                    offsets_local.data_ptr(), col_local.data_ptr(), w_local.data_ptr(), self.n_local,
                    self.m_local, self.v0, self.n_global, self.rank, self.world, self.bounds.ctypes.data,
                    self._id, ctypes.byref(opts), self.stream.cuda_stream, ctypes.byref(h)),
                    "lmatch_create_dist_device")
            else:
                off = np.ascontiguousarray(offsets_local, dtype=np.int64)
                col = np.ascontiguousarray(col_local, dtype=np.int32)
                w = np.ascontiguousarray(w_local, dtype=np.float32)
                self.m_local = int(col.shape[0])
                _check(_lib.lmatch_create_dist(
                    off.ctypes.data, col.ctypes.data, w.ctypes.data, self.n_local, self.m_local,
                    self.v0, self.n_global, self.rank, self.world, self.bounds.ctypes.data, self._id,
                    ctypes.byref(opts), ctypes.byref(h)), "lmatch_create_dist")
        self.h = h.value

    def run_device(self, d_mate=None):
        """Collective: every rank calls it.  Returns (owned mate slice as a CUDA tensor, Stats)."""
        from . import Stats
        torch = self.torch
        if d_mate is None:
            with torch.cuda.stream(self.stream):
                d_mate = torch.empty(max(self.n_local, 1), dtype=torch.int32, device=self.dev)
        st = Stats()
        _check(_lib.lmatch_run_dist_device(self.h, d_mate.data_ptr(), self.stream.cuda_stream,
                                           ctypes.byref(st)), "lmatch_run_dist_device")
        return d_mate[: self.n_local], st

    def run(self):
        """Collective; host output.  Returns (owned mate slice as numpy int32, Stats)."""
        from . import Stats
        mate = np.empty(max(self.n_local, 1), dtype=np.int32)
        st = Stats()
        _check(_lib.lmatch_run_dist(self.h, mate.ctypes.data, ctypes.byref(st)), "lmatch_run_dist")
        return mate[: self.n_local], st

    def reload(self, offsets_local, col_local, w_local):
        ptrs = [a.ctypes.data if isinstance(a, np.ndarray) else int(a)
                for a in (offsets_local, col_local, w_local)]
        _check(_lib.lmatch_reload(self.h, *ptrs), "lmatch_reload")

    def close(self):
        if self.h is not None:
            _lib.lmatch_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def match_dist_threads(offsets, col, w, nparts: int, devices=None, max_rounds: int = 0, **opt_kw):
    """P ranks of one lmatch_create_dist group as P threads of this process (one GPU each, or all
    on the current GPU): the rendezvous gives them plain device pointers.  Returns (mate, stats
    of rank 0, [stats of every rank])."""
    import threading
    offsets = np.asarray(offsets, dtype=np.int64)
    n = offsets.shape[0] - 1
    bounds = edge_balanced_bounds(offsets, nparts)
    did = dist_id_new()
    out, errs = [None] * nparts, [None] * nparts

    def rank_main(r):
        try:
            dev = None if devices is None else devices[r % len(devices)]
            v0, v1 = int(bounds[r]), int(bounds[r + 1])
            lo, lc, lw = local_csr(offsets, col, w, v0, v1)
            M = DistMatcher(lo, lc, lw, v0, n, r, nparts, bounds, did, device=dev, max_rounds=max_rounds,
                            **opt_kw)
            try:
                out[r] = M.run()
            finally:
                M.close()
        except Exception as e:  # reported by the caller
            errs[r] = e

    ts = [threading.Thread(target=rank_main, args=(r,)) for r in range(nparts)]
    for t in ts:
        t.start()
    for t in ts:
        t.join()
    # a rank that failed makes its peers time out at a barrier (ENCCL): report the cause first
    real = [e for e in errs if e is not None and getattr(e, "status", None) != -5]
    for e in real + [e for e in errs if e is not None]:
        raise e
    mate = np.concatenate([o[0] for o in out]) if n else np.zeros(0, np.int32)
    return mate, out[0][1], [o[1] for o in out]


# ----------------------------------------------------------------------------- the round loop
@dataclass
class PartResult:
    mates: list          # per local part: mate[] of its owned range (global ids)
    weight: float        # w(M) over ALL parts (fp64)
    matched: int         # matched vertices over all parts
    rounds: int          # pointing phases executed
    exchanged_claims: int  # claims sent by the local parts (all rounds)


def run_parts(parts, transport) -> PartResult:
    """Drive the rounds for the local `parts` (all parts with LocalTransport, one with
    TorchTransport).  Part objects implement begin/point/claims/apply/own_bits/set_bits/compact/
    finish (LibPart on GPUs; tests/dist_model.py on CPU)."""
    counts = [p.begin() for p in parts]
    rounds = 1
    sent = 0
    while True:
        sends = [p.claims(c) for p, c in zip(parts, counts)]
        sent += sum(int(np.sum(c)) for c in counts)
        recvs = transport.exchange(sends)
        for p, r in zip(parts, recvs):
            p.apply(r)
        alls = transport.allgather([p.own_bits() for p in parts])
        for p, a in zip(parts, alls):
            p.set_bits(a)
        nF = transport.allreduce([p.compact() for p in parts])[0]
        if nF == 0:
            break
        rounds += 1
        counts = [p.point() for p in parts]
    fin = [p.finish() for p in parts]
    w = transport_sum_float(transport, [f[1] for f in fin])
    c = transport.allreduce([f[2] for f in fin])[0]
    return PartResult([f[0] for f in fin], w, c, rounds, sent)


def kernel_launch_count() -> int:
    """Kernels liblmatch.so has launched in this process so far (lmatch_kernel_launch_count)."""
    return int(_lib.lmatch_kernel_launch_count())


def connect_p2p_local(parts):
    """Peer-memory exchange between parts living in this process (plain device pointers)."""
    for p in parts:
        p.p2p_enable()
    for p in parts:
        for q in parts:
            if q is not p:
                p.p2p_attach_local(q.part, q)


def connect_p2p_torch(part, group=None):
    """Peer-memory exchange between processes: every rank exports its window handles (CUDA IPC),
    the handles are all-gathered over torch.distributed, and every rank opens its peers'."""
    import torch.distributed as dist
    part.p2p_enable()
    mine = part.p2p_export()
    allh = [None] * dist.get_world_size(group)
    dist.all_gather_object(allh, (part.part, mine), group=group)
    for peer, h in allh:
        if peer != part.part:
            part.p2p_attach(peer, h)


def barrier_local(parts):
    """Barrier for parts in one process: drain every part's stream."""
    def b():
        for p in parts:
            p.p2p_sync()
    return b


def barrier_events(parts):
    """Barrier for parts in one process without draining any stream: every part records an
    event on its stream and every part's stream waits for all the others' events (works across
    devices too), so the phases stay ordered on the GPUs while the host runs ahead."""
    import torch

    def b():
        # gather on part 0's stream, then release everyone from it: 2(P-1) waits instead of P^2
        hub = parts[0].stream
        for p in parts[1:]:
            e = torch.cuda.Event()
            e.record(p.stream)
            hub.wait_event(e)
        if len(parts) > 1:
            e = torch.cuda.Event()
            e.record(hub)
            for p in parts[1:]:
                p.stream.wait_event(e)
    return b


def connect_events_torch(part, group=None):
    """Cross-process event barrier setup: an interprocess CUDA event per rank, its IPC handle
    all-gathered, the peers' events opened here (part.peer_events)."""
    import torch
    import torch.distributed as dist
    part.ev = torch.cuda.Event(interprocess=True)
    part.ev.record(part.stream)  # an event must be recorded once before its handle is exported
    allh = [None] * dist.get_world_size(group)
    dist.all_gather_object(allh, (part.part, part.ev.ipc_handle()), group=group)
    part.peer_events = [torch.cuda.Event.from_ipc_handle(part.dev, h) for peer, h in allh
                        if peer != part.part]


def barrier_torch_events(parts, cpu_group=None):
    """Barrier across processes that drains no stream: each rank records its interprocess event,
    a host barrier (cpu_group, e.g. gloo) guarantees every record is issued, then each rank's
    stream waits for the peers' events.  A rank may run one barrier ahead; a wait then refers to
    a later record of the peer's event, which over-orders but cannot deadlock (a record never
    waits on anything behind it)."""
    import torch.distributed as dist

    def b():
        for p in parts:
            p.ev.record(p.stream)
        dist.barrier(group=cpu_group)
        for p in parts:
            for e in p.peer_events:
                p.stream.wait_event(e)
    return b


def barrier_torch(parts, group=None):
    """Barrier across processes: drain the local streams, then a torch.distributed barrier."""
    import torch.distributed as dist

    def b():
        for p in parts:
            p.p2p_sync()
        dist.barrier(group=group)
    return b


def run_parts_p2p(parts, barrier, transport) -> PartResult:
    """The partitioned round with the exchange inside the library's kernels (peer-memory stores:
    claims into the owners' inboxes, changed bitmap words into every replica, frontier sizes into
    every part's slot).  `barrier()` separates the phases; `transport` is used only for the final
    w(M) / |M| sums.  Same result as run_parts."""
    barrier()                      # every part is done with its previous run
    for p in parts:
        p.p2p_begin()
    rounds = 1
    compacted = False
    while True:
        # claims are in the owners' inboxes, and the frontier sizes pushed by the last compaction
        # are in every slot (they were stored before each part's pointer phase)
        barrier()
        if compacted:
            totals = [p.p2p_frontier_total() for p in parts]
            if any(t != totals[0] for t in totals):
                raise LMatchError(f"frontier totals differ between parts: {totals}")
            if totals[0] == 0:
                break
            rounds += 1
        for p in parts:
            p.p2p_match()
        barrier()                  # bitmap replicas are complete
        for p in parts:
            p.p2p_compact()
        compacted = True
        # the next pointer phase runs before the termination test (two barriers per round, not
        # three): when the global frontier is empty every part's frontier is, and it does nothing
        for p in parts:
            p.p2p_point()
    fin = [p.finish() for p in parts]
    w = transport_sum_float(transport, [f[1] for f in fin])
    c = transport.allreduce([f[2] for f in fin])[0]
    return PartResult([f[0] for f in fin], w, c, rounds, 0)


def transport_sum_float(transport, xs):
    """fp64 sum over all parts (deterministic: gathered then summed in part order)."""
    if isinstance(transport, LocalTransport):
        return float(sum(xs))
    import torch
    (x,) = xs
    dev = "cuda" if transport.dist.get_backend(transport.group) == "nccl" else "cpu"
    t = torch.tensor([x], dtype=torch.float64, device=dev)
    out = [torch.empty_like(t) for _ in range(transport.nparts)]
    transport.dist.all_gather(out, t, group=transport.group)
    return float(sum(float(o.item()) for o in out))


def match_partitioned_local(offsets, col, w, nparts: int, device=None, exchange: str = "transport",
                            **opt_kw):
    """P logical partitions of one graph on one device.  exchange = "transport": LocalTransport
    moves the claims / bitmap words; "p2p": the library's kernels store them into the other parts'
    memory (peer-memory exchange), phases ordered by cross-stream events; "p2p_sync": the same with
    host-synchronising barriers.  Returns (mate, result)."""
    offsets = np.asarray(offsets, dtype=np.int64)
    n = offsets.shape[0] - 1
    bounds = edge_balanced_bounds(offsets, nparts)
    parts = []
    for p in range(nparts):
        v0, v1 = int(bounds[p]), int(bounds[p + 1])
        lo, lc, lw = local_csr(offsets, col, w, v0, v1)
        parts.append(LibPart(lo, lc, lw, v0, n, bounds, p, device=device, **opt_kw))
    if exchange in ("p2p", "p2p_sync"):
        connect_p2p_local(parts)
        barrier = barrier_events(parts) if exchange == "p2p" else barrier_local(parts)
        res = run_parts_p2p(parts, barrier, LocalTransport(nparts))
    else:
        res = run_parts(parts, LocalTransport(nparts))
    mate = np.concatenate([m.cpu().numpy() for m in res.mates]) if n else np.zeros(0, np.int32)
    for p in parts:
        p.close()
    return mate, res
