"""CPU model of one partition (test infrastructure): the same per-part interface as
paper_conf_sc_mandulakgfhs24_b200.dist.LibPart, in numpy, so the product driver `run_parts` and its
TorchTransport can be exercised on CPU with the gloo backend (world_size >= 2).

It follows the same protocol as the library: pointer = max packed key over
unmatched neighbours (R2); a claim (v | u << 32) is sent to owner(v) when owned u points to remote
v; ghost[u] = v on receipt; mutual check ptr(v) == u with ghosts for remote v; replicated matched
bitmap exchanged as owned 32-bit words; frontier = live vertices whose target got matched (R3).
"""
import numpy as np
import torch

NOPTR = 0xFFFFFFFF


class NumpyPart:
    def __init__(self, offsets_local, col_local, w_local, v0, n_global, bounds, part):
        self.off = np.asarray(offsets_local, dtype=np.int64)
        col = np.asarray(col_local, dtype=np.int64)
        w = np.asarray(w_local, dtype=np.float32)
        self.v0, self.n = int(v0), self.off.shape[0] - 1
        self.N = int(n_global)
        self.bounds = np.asarray(bounds, dtype=np.int64)
        self.P, self.part = self.bounds.shape[0] - 1, int(part)
        rows = np.repeat(np.arange(self.n, dtype=np.int64), np.diff(self.off)) + self.v0
        keys = (w.view(np.uint32).astype(np.uint64) << np.uint64(32)) | col.astype(np.uint64)
        keys[col == rows] = 0  # self-loops are ignored
        self.keys, self.col = keys, col
        self.w0 = self.bounds[self.part] // 32

    # ------------------------------------------------------------------ helpers
    def _owner(self, v):
        return int(np.searchsorted(self.bounds, v, side="right") - 1)

    def _local(self, v):
        return self.v0 <= v < self.v0 + self.n

    def _ptr_of(self, v):
        if self._local(v):
            k = int(self.best[v - self.v0])
            return (k & 0xFFFFFFFF) if k else NOPTR
        return int(self.ghost[v])

    def _point(self, i):
        s, e = self.off[i], self.off[i + 1]
        k = self.keys[s:e]
        ok = (k > 0) & ~self.bits[self.col[s:e]]
        self.best[i] = k[ok].max() if ok.any() else np.uint64(0)

    def _claims_for(self, us):
        self.out = [[] for _ in range(self.P)]
        for u in us:
            k = int(self.best[u - self.v0])
            if not k:
                continue
            v = k & 0xFFFFFFFF
            if not self._local(v):
                self.out[self._owner(v)].append(v | (u << 32))
        return np.array([len(x) for x in self.out], dtype=np.int64)

    # ------------------------------------------------------------------ interface
    def begin(self):
        self.best = np.zeros(self.n, dtype=np.uint64)
        self.ghost = np.full(self.N + 1, NOPTR, dtype=np.int64)
        self.bits = np.zeros(self.N + 1, dtype=bool)
        self.round = 1
        for i in range(self.n):
            self._point(i)
        self.F = list(range(self.v0, self.v0 + self.n))
        return self._claims_for(self.F)

    def point(self):
        for u in self.F:
            self._point(u - self.v0)
        self.round += 1
        return self._claims_for(self.F)

    def claims(self, counts):
        return [torch.tensor(np.array(x, dtype=np.uint64).view(np.int64), dtype=torch.int64)
                for x in self.out]

    def apply(self, recv):
        rc = recv.numpy().view(np.uint64)
        for c in rc:
            v, u = int(c & 0xFFFFFFFF), int(c >> np.uint64(32))
            self.ghost[u] = v
        for u in self.F:
            k = int(self.best[u - self.v0])
            if not k:
                continue
            v = k & 0xFFFFFFFF
            if self._ptr_of(v) == u:
                self.bits[u] = True
                if self._local(v):
                    self.bits[v] = True
        for c in rc:
            v, u = int(c & 0xFFFFFFFF), int(c >> np.uint64(32))
            k = int(self.best[v - self.v0])
            if k and (k & 0xFFFFFFFF) == u:
                self.bits[v] = True

    def own_bits(self):
        b = self.bits[self.bounds[self.part]:self.bounds[self.part + 1]]
        nw = (b.shape[0] + 31) // 32
        pad = np.zeros(nw * 32, dtype=np.uint64)
        pad[: b.shape[0]] = b
        words = (pad.reshape(nw, 32) << np.arange(32, dtype=np.uint64)).sum(axis=1)
        return torch.tensor(words.astype(np.uint32).view(np.int32), dtype=torch.int32)

    def set_bits(self, all_words):
        for p, t in enumerate(all_words):
            if p == self.part:
                continue
            words = t.numpy().view(np.uint32).astype(np.uint64)
            bits = ((words[:, None] >> np.arange(32, dtype=np.uint64)) & 1).astype(bool).reshape(-1)
            lo, hi = self.bounds[p], self.bounds[p + 1]
            self.bits[lo:hi] = bits[: hi - lo]

    def compact(self):
        live = []
        for u in range(self.v0, self.v0 + self.n):
            k = int(self.best[u - self.v0])
            if k and not self.bits[u]:
                live.append(u)
        self.F = [u for u in live if self.bits[int(self.best[u - self.v0]) & 0xFFFFFFFF]]
        return len(self.F)

    def finish(self):
        mate = np.full(self.n, -1, dtype=np.int32)
        w = 0.0
        c = 0
        for i in range(self.n):
            u = i + self.v0
            if self.bits[u]:
                k = int(self.best[i])
                v = k & 0xFFFFFFFF
                mate[i] = v
                c += 1
                if v > u:
                    w += float(np.uint32(k >> 32).view(np.float32))
        return torch.from_numpy(mate), w, c


class NumpyP2PPart(NumpyPart):
    """The peer-memory exchange protocol of lmatch_p2p_* (include/lmatch.h) on CPU: the exchange
    window (inbox [P][cap], counts [P], frontier-size slots [P]) and the replicated bitmap live in
    POSIX shared memory, and peers store into them directly -- the CPU stand-in for the library's
    stores over NVLink / CUDA IPC.  Same driver (dist.run_parts_p2p), same barriers."""

    def p2p_enable(self):
        from multiprocessing import shared_memory
        P = self.P
        self.cap = int(max(1, np.diff(self.bounds).max()))
        nwin = P * self.cap + 2 * P
        self._shm = [shared_memory.SharedMemory(create=True, size=8 * nwin),
                     shared_memory.SharedMemory(create=True, size=self.N + 1)]
        self.win = np.ndarray((nwin,), dtype=np.uint64, buffer=self._shm[0].buf)
        self.win[:] = 0
        self.bits = np.ndarray((self.N + 1,), dtype=bool, buffer=self._shm[1].buf)
        self.bits[:] = False
        self.peer_win = [None] * P
        self.peer_bits = [None] * P
        self._opened = []
        self.peer_win[self.part] = self.win
        self.peer_bits[self.part] = self.bits

    def p2p_export(self):
        return (self._shm[0].name, self._shm[1].name)

    def p2p_attach(self, peer, names):
        from multiprocessing import shared_memory
        a = shared_memory.SharedMemory(name=names[0])
        b = shared_memory.SharedMemory(name=names[1])
        self._opened += [a, b]
        self.peer_win[peer] = np.ndarray((self.P * self.cap + 2 * self.P,), dtype=np.uint64, buffer=a.buf)
        self.peer_bits[peer] = np.ndarray((self.N + 1,), dtype=bool, buffer=b.buf)

    def p2p_attach_local(self, peer, other):
        self.peer_win[peer] = other.win
        self.peer_bits[peer] = other.bits

    def _push_claims(self):
        P, cap = self.P, self.cap
        for d in range(P):
            out = self.out[d]
            if not out:
                continue
            w = self.peer_win[d]
            base = int(w[P * cap + self.part])
            w[self.part * cap + base: self.part * cap + base + len(out)] = np.array(out, dtype=np.uint64)
            w[P * cap + self.part] = np.uint64(base + len(out))

    def p2p_begin(self):
        self.best = np.zeros(self.n, dtype=np.uint64)
        self.ghost = np.full(self.N + 1, NOPTR, dtype=np.int64)
        self.bits[:] = False
        self.round = 1
        for i in range(self.n):
            self._point(i)
        self.F = list(range(self.v0, self.v0 + self.n))
        self._claims_for(self.F)
        self._push_claims()

    def p2p_point(self):
        self.point()
        self._push_claims()

    def p2p_match(self):
        P, cap = self.P, self.cap
        segs = [self.win[s * cap: s * cap + int(self.win[P * cap + s])] for s in range(P)]
        recv = torch.from_numpy(np.concatenate(segs).view(np.int64).copy()) if segs else \
            torch.zeros(0, dtype=torch.int64)
        self.apply(recv)
        self.win[P * cap: P * cap + P] = 0
        lo, hi = self.bounds[self.part], self.bounds[self.part + 1]
        for p in range(P):
            if p != self.part:
                self.peer_bits[p][lo:hi] = self.bits[lo:hi]

    def p2p_compact(self):
        nf = self.compact()
        P, cap = self.P, self.cap
        for p in range(P):
            self.peer_win[p][P * cap + P + self.part] = np.uint64(nf)
        return nf

    def p2p_frontier_total(self):
        P, cap = self.P, self.cap
        return int(self.win[P * cap + P: P * cap + 2 * P].sum())

    def p2p_sync(self):
        pass

    def close(self):
        for s in getattr(self, "_opened", []):
            s.close()
        for s in getattr(self, "_shm", []):
            s.close()
            s.unlink()
        self._opened, self._shm = [], []
