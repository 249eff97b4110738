"""Reading R21: chunk-label index recovery for max-subarray.

The values-only NK4 (the default since r02b; -DDC_MS_VONLY=0 is the indexed
variant) folds each chunk of L elements
without indices, labels the chunk leaf by its start, combines the leaves with
the ordered tie rules of the D&C combine (R10), and then
re-scans at most four chunks for the exact (pe, ss, bs, be).  This test checks
that claim in plain Python against the oracle (lexicographically smallest
optimal (start, end), R10) and against numpy's first argmax of the prefix and
suffix sums, on tie-heavy arrays and every chunk size 1..9.  It pins the
reading only; the CUDA kernel is checked against the oracle by the maxsub tests
of tests/test_gpu_parity.py (tie-heavy, degenerate, tuple) and the indexed
variant by tests/test_gpu_variants.py.
"""
import numpy as np

import oracle

NEG = -(1 << 62)


def _combine(L, R):
    # (tot, pre, suf, best, pe, ss, bs, be); L immediately left of R
    tot = L[0] + R[0]
    lp = L[0] + R[1]
    pre, pe = (L[1], L[4]) if L[1] >= lp else (lp, R[4])
    rs = R[0] + L[2]
    suf, ss = (rs, L[5]) if rs >= R[2] else (R[2], R[5])
    best, bs, be = L[3], L[6], L[7]
    if L[2] + R[1] > best:
        best, bs, be = L[2] + R[1], L[5], R[4]
    if R[3] > best:
        best, bs, be = R[3], R[6], R[7]
    return (tot, pre, suf, best, pe, ss, bs, be)


def _chunk_recover(x, L):
    n = len(x)
    acc = None
    for c in range(0, n, L):
        tot, pre, suf, best = 0, NEG, NEG, NEG
        for v in x[c:c + L]:          # values only
            tot += v
            pre = max(pre, tot)
            suf = max(suf, 0) + v
            best = max(best, suf)
        leaf = (tot, pre, suf, best, c, c, c, c)
        acc = leaf if acc is None else _combine(acc, leaf)

    def suffix_start(c):               # first argmax of sum(x[s..chunk end])
        P, m, k = 0, 0, c
        for j in range(c, min(c + L, n) - 1):
            P += x[j]
            if P < m:
                m, k = P, j + 1
        return k

    def prefix_end(c):                 # first argmax of sum(x[c..e])
        P, m, k = 0, NEG, c
        for j in range(c, min(c + L, n)):
            P += x[j]
            if P > m:
                m, k = P, j
        return k

    B, cs, ce = acc[3], acc[6], acc[7]
    if cs == ce:                       # in-chunk Kadane, same tie rules
        best, suf, ss, s, e = NEG, NEG, cs, cs, cs
        for j in range(cs, min(cs + L, n)):
            if suf < 0:
                suf, ss = 0, j
            suf += x[j]
            if suf > best:
                best, s, e = suf, ss, j
    else:
        s, e = suffix_start(cs), prefix_end(ce)
    return B, s, e, prefix_end(acc[4]), suffix_start(acc[5])


def test_chunk_label_recovery_matches_oracle():
    rng = np.random.default_rng(21)
    for it in range(3000):
        n = int(rng.integers(1, 40))
        L = int(rng.integers(1, 10))
        if it % 4 == 0:
            x = np.full(n, int(rng.integers(-1, 2)), np.int32)
        else:
            x = rng.integers(-3 if it % 2 else -1, 2, n).astype(np.int32)
        B, s, e, pe, ss = _chunk_recover([int(v) for v in x], L)
        assert (B, s, e) == tuple(int(v) for v in oracle.maxsub(x)), (x.tolist(), L)
        a = x.astype(np.int64)
        assert pe == int(np.argmax(np.cumsum(a))), (x.tolist(), L)
        assert ss == int(np.argmax(np.cumsum(a[::-1])[::-1])), (x.tolist(), L)


def _in_chunk_prefix_rule(xs):
    """r02b's warp-parallel in-chunk recovery (maxsub_tma.cuh ms_par_kadane):
    s_e = first argmin of Q_q = P_{q-1} over q in [0, e] (P_{-1} = 0),
    e* = first argmax of P_e - Q_{s_e}; returns (value, s_{e*}, e*)."""
    best, bs, be = None, 0, 0
    P, qmin, qarg = 0, None, 0
    for e, v in enumerate(xs):
        Q = P                          # P_{e-1}
        if qmin is None or Q < qmin:   # strict: the first minimum
            qmin, qarg = Q, e
        P += v
        val = P - qmin
        if best is None or val > best:   # strict: the first maximum
            best, bs, be = val, qarg, e
    return best, bs, be


def test_in_chunk_prefix_rule_is_the_lexicographic_minimum():
    """Pins the in-chunk rule of the warp-parallel recovery against brute force
    (the lexicographically smallest optimal (start, end), reading R10) on
    tie-heavy and random chunks: every optimal (s, e) has s_e <= s with (s_e, e)
    optimal, and s_e does not decrease with e, so the first optimal e gives the
    lexicographic minimum (R21)."""
    rng = np.random.default_rng(2102)
    for it in range(4000):
        n = int(rng.integers(1, 30))
        if it % 3 == 0:
            xs = [int(v) for v in rng.integers(-1, 2, n)]
        elif it % 3 == 1:
            xs = [int(v) for v in rng.integers(-3, 3, n)]
        else:
            xs = [int(v) for v in rng.integers(-(1 << 31), 1 << 31, n, dtype=np.int64)]
        brute = max((sum(xs[s:e + 1]), -s, -e) for s in range(n) for e in range(s, n))
        assert _in_chunk_prefix_rule(xs) == (brute[0], -brute[1], -brute[2]), xs
