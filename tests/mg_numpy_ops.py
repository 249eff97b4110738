"""Test double for the per-rank device steps of the multi-GPU protocol.

Used ONLY by the CPU (gloo, world_size >= 2) tests to exercise the host logic
and collectives of paper_conf_ipps_lopez_ortizss13_b200.dist without a GPU:
same tensor layouts as the CUDA kernels (send buffer words, split matrix),
plain numpy underneath.  The product path never imports this module.
"""
import numpy as np
import torch

_VIEW = {"u32": np.uint32, "i32": np.int32, "f32": np.float32}


def _v(t, kt):
    a = t.detach().cpu().numpy()
    return a.view(_VIEW[kt]) if a.dtype != np.float32 or kt != "f32" else a


class NumpyOps:
    def __init__(self, key_type="u32"):
        self.kt = key_type
        self._launches = 0

    def sort_(self, keys, vals, key_type):
        a = _v(keys, key_type)
        order = np.argsort(a, kind="stable")
        keys.copy_(torch.from_numpy(keys.numpy()[order].copy()))
        if vals is not None:
            vals.copy_(torch.from_numpy(vals.numpy()[order].copy()))

    def sample(self, keys, stride):
        return torch.from_numpy(keys.numpy()[::stride].copy())

    def count(self, keys, rank, cand, per_rank, stride, key_type):
        a, c = _v(keys, key_type), _v(cand, key_type)
        idx = np.arange(c.size)
        owner, j = idx // per_rank, idx % per_rank
        lt = np.searchsorted(a, c, side="left")
        le = np.searchsorted(a, c, side="right")
        out = np.where(rank < owner, le, np.where(rank == owner, j * stride, lt))
        return torch.from_numpy(out.astype(np.int64))

    def windows(self, keys, rank, world, counts, ranks, per_rank, wcap):
        C, R = counts.numpy(), ranks.numpy()
        m = keys.numel()
        words = 6 * (world - 1) + (world - 1) * wcap
        buf = np.zeros(words, dtype=np.int32)
        hdr = buf[:6 * (world - 1)].view(np.int64)
        for d in range(1, world):
            k = d * m
            below = np.nonzero(R < k)[0]
            above = np.nonzero(R >= k)[0]
            a = below[np.argmax(R[below])] if below.size else None
            b = above[np.argmin(R[above])] if above.size else None
            lo = C[a] + (1 if a // per_rank == rank else 0) if a is not None else 0
            hi = C[b] if b is not None else m
            t = k - (R[a] + 1 if a is not None else 0)
            ln = hi - lo
            assert 0 <= ln <= wcap
            hdr[3 * (d - 1):3 * d] = [lo, ln, t]
            off = 6 * (world - 1) + (d - 1) * wcap
            buf[off:off + ln] = keys.numpy().view(np.int32)[lo:hi]
        return torch.from_numpy(buf)

    def split_matrix(self, gathered, world, shard_n, wcap, key_type):
        g = gathered.numpy()
        words = 6 * (world - 1) + (world - 1) * wcap
        cm = np.zeros((world, world + 1), dtype=np.int64)
        cm[:, world] = shard_n
        for d in range(1, world):
            lo, ln, ts = [], [], None
            items = []
            for r in range(world):
                buf = g[r * words:(r + 1) * words]
                h = buf[:6 * (world - 1)].view(np.int64)
                lo.append(int(h[3 * (d - 1)]))
                ln.append(int(h[3 * (d - 1) + 1]))
                if r == 0:
                    ts = int(h[3 * (d - 1) + 2])
                off = 6 * (world - 1) + (d - 1) * wcap
                w = buf[off:off + ln[r]].view(_VIEW[key_type])
                items += [(w[p], r, p) for p in range(ln[r])]
            items.sort(key=lambda x: (x[0], x[1], x[2]))
            first = items[:ts]
            for r in range(world):
                cm[r, d] = lo[r] + sum(1 for it in first if it[1] == r)
        return torch.from_numpy(cm)

    def check(self):
        pass

    def merge_runs(self, in_k, in_v, out_k, out_v, runs, key_type):
        a = _v(in_k, key_type)
        order = np.argsort(a, kind="stable")     # runs back to back, earlier runs first
        out_k.copy_(torch.from_numpy(in_k.numpy()[order].copy()))
        if in_v is not None:
            out_v.copy_(torch.from_numpy(in_v.numpy()[order].copy()))

    # max-subarray summary (tot, pre, suf, best, pe, ss, bs, be) by plain scans
    def maxsub_tuple(self, x, offset):
        a = x.numpy().astype(np.int64)
        p = np.cumsum(a)
        pe = int(np.argmax(p))
        tot = int(p[-1])
        suffix = tot - np.concatenate([[0], p[:-1]])          # sum a[s:], s = 0..n-1
        ss = int(np.argmax(suffix))
        best, bs, be = None, 0, 0
        for s in range(a.size):
            acc = 0
            for e in range(s, a.size):
                acc += int(a[e])
                if best is None or acc > best:
                    best, bs, be = acc, s, e
        return torch.tensor([tot, int(p[pe]), int(suffix[ss]), best, pe + offset, ss + offset,
                             bs + offset, be + offset], dtype=torch.int64)

    def maxsub_combine(self, tuples):
        acc = None
        for t in tuples.tolist():
            if acc is None:
                acc = t
                continue
            L, R = acc, t
            tot = L[0] + R[0]
            pre, pe = (L[1], L[4]) if L[1] >= L[0] + R[1] else (L[0] + R[1], R[4])
            suf, ss = (R[0] + L[2], L[5]) if R[0] + L[2] >= R[2] else (R[2], R[5])
            best, bs, be = L[3], L[6], L[7]
            if L[2] + R[1] > best:
                best, bs, be = L[2] + R[1], L[5], R[4]
            if R[3] > best:
                best, bs, be = R[3], R[6], R[7]
            acc = [tot, pre, suf, best, pe, ss, bs, be]
        return torch.tensor([acc[3], acc[6], acc[7]], dtype=torch.int64)

    def launches(self):
        return self._launches
