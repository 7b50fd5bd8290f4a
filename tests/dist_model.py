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
