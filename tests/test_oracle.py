"""Pins for the CPU oracle (oracle/oracle.c) against things other than itself.

Sort (Alg 6; Alg 7):
  * brute force: every permutation of n <= 8 distinct keys; every sequence over
    {0,1,2}^n, n <= 8, with vals = index (stability is observable);
  * the library routine numpy stable argsort at random n (incl. non powers of 2),
    for u32, i32 and f32 (with +/-0.0) keys;
  * invariants: non-decreasing, same multiset, stable;
  * recurrence T(n) = aT(n/b) + f(n): per-depth combine and element
    counts a^d and n for n = 2^k, total work n(log2 n + 1)
    counting the leaves;
  * Alg 7 == Alg 6 for n = 2^k.
Max-subarray (north star instance 2; readings R9-R11 in DESIGN.md):
  * O(n^2) brute force (independent double loop / prefix-sum table);
  * exhaustive {-2..2}^n for n <= 6;
  * closed forms: all positive, all negative, all zero, single spike;
  * per-depth combine counts 2^d.
Sum (Alg 4): Python's exact integer sum.
"""
import itertools
import math

import numpy as np
import pytest

import dcgen


# ------------------------------------------------------------------ sort

def test_all_permutations_up_to_8(oracle_mod):
    for n in range(0, 9):
        expect = np.arange(n, dtype=np.uint32)
        for perm in itertools.permutations(range(n)):
            got = oracle_mod.mergesort(np.array(perm, dtype=np.uint32))
            assert np.array_equal(got, expect), perm


def test_all_ternary_sequences_stable_up_to_8(oracle_mod):
    for n in range(0, 9):
        for seq in itertools.product(range(3), repeat=n):
            keys = np.array(seq, dtype=np.uint32)
            vals = np.arange(n, dtype=np.uint32)
            k, v = oracle_mod.mergesort(keys, vals)
            # brute-force stable sort: by (key, original index)
            order = sorted(range(n), key=lambda i: (seq[i], i))
            assert k.tolist() == [seq[i] for i in order]
            assert v.tolist() == order


@pytest.mark.parametrize("n", [1, 2, 3, 5, 17, 1000, 4096, 4097, 65536 + 123, 1 << 20])
@pytest.mark.parametrize("dist", ["uniform", "few", "paper"])
def test_matches_numpy_stable_u32(oracle_mod, n, dist):
    keys = dcgen.sort_keys(n, dist, seed=11).numpy().view(np.uint32)
    vals = np.arange(n, dtype=np.uint32)
    k, v = oracle_mod.mergesort(keys, vals)
    order = np.argsort(keys, kind="stable")
    assert np.array_equal(k, keys[order])
    assert np.array_equal(v, vals[order])
    # invariants
    assert np.all(k[1:] >= k[:-1])
    eq = k[1:] == k[:-1]
    assert np.all(v[1:][eq] > v[:-1][eq])


@pytest.mark.parametrize("key_type", ["i32", "f32"])
@pytest.mark.parametrize("n", [7, 1000, 70000])
def test_matches_numpy_stable_signed_and_float(oracle_mod, key_type, n):
    t = dcgen.sort_keys(n, "uniform", seed=5, key_type=key_type)
    keys = t.numpy().view(np.int32) if key_type == "i32" else t.numpy()
    vals = np.arange(n, dtype=np.uint32)
    k, v = oracle_mod.mergesort(keys, vals, key_type=key_type)
    order = np.argsort(keys, kind="stable")
    assert np.array_equal(k.view(np.uint32), keys[order].view(np.uint32))  # bit-exact (+/-0)
    assert np.array_equal(v, vals[order])


def test_float_signed_zero_keeps_input_order(oracle_mod):
    keys = np.array([0.0, -0.0, 1.0, -0.0, 0.0, -1.0], dtype=np.float32)
    k = oracle_mod.mergesort(keys, key_type="f32")
    expect_bits = np.array([-1.0, 0.0, -0.0, -0.0, 0.0, 1.0], dtype=np.float32).view(np.uint32)
    assert np.array_equal(k.view(np.uint32), expect_bits)


@pytest.mark.parametrize("k", [1, 2, 5, 10, 16])
def test_level_counts_match_recurrence(oracle_mod, k):
    n = 1 << k
    keys = dcgen.sort_keys(n, "uniform", seed=3).numpy().view(np.uint32)
    _, lc, le = oracle_mod.mergesort(keys, counters=True)
    for d in range(k):
        assert lc[d] == 2 ** d          # a^d subproblems at level d
        assert le[d] == n               # a^d * f(n/b^d) = n merged elements
    assert np.all(lc[k:] == 0)
    # total work counting the n leaves: n (log_b n + 1)
    assert int(le.sum()) + n == n * (k + 1)


@pytest.mark.parametrize("k", [0, 1, 3, 8, 13])
def test_breadth_first_alg7_equals_alg6(oracle_mod, k):
    n = 1 << k
    keys = dcgen.sort_keys(n, "few", seed=9).numpy().view(np.uint32)
    vals = np.arange(n, dtype=np.uint32)
    a = oracle_mod.mergesort(keys, vals)
    b = oracle_mod.mergesort_bf(keys, vals)
    assert np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1])


def test_breadth_first_rejects_non_power_of_two(oracle_mod):
    with pytest.raises(ValueError):
        oracle_mod.mergesort_bf(np.arange(6, dtype=np.uint32))


# --------------------------------------------------------- max-subarray

def brute_maxsub(x):
    """Independent O(n^2) definition: max over non-empty [s, e], lexicographically
    smallest (s, e) among the maxima (ascending loops with strict '>')."""
    best = None
    for s in range(len(x)):
        acc = 0
        for e in range(s, len(x)):
            acc += int(x[e])
            if best is None or acc > best[0]:
                best = (acc, s, e)
    return best


def brute_maxsub_np(x):
    """Same definition via a prefix-sum table (for n up to a few thousand)."""
    p = np.concatenate([[0], np.cumsum(np.asarray(x, dtype=np.int64))])
    n = len(x)
    best = None
    for s in range(n):
        sums = p[s + 1:] - p[s]
        e = int(np.argmax(sums))          # first (smallest) e achieving the row max
        v = int(sums[e])
        if best is None or v > best[0]:
            best = (v, s, s + e)
    return best


def test_maxsub_exhaustive_small(oracle_mod):
    for n in range(1, 7):
        for seq in itertools.product(range(-2, 3), repeat=n):
            x = np.array(seq, dtype=np.int32)
            assert oracle_mod.maxsub(x) == brute_maxsub(seq), seq


@pytest.mark.parametrize("n", [1, 2, 31, 200, 1000, 2048])
@pytest.mark.parametrize("dist", ["small", "uniform", "negative", "positive"])
def test_maxsub_brute_force_random(oracle_mod, n, dist):
    x = dcgen.maxsub_input(n, dist, seed=13).numpy()
    assert oracle_mod.maxsub(x) == brute_maxsub_np(x)


def test_maxsub_closed_forms(oracle_mod):
    n = 5000
    pos = dcgen.maxsub_input(n, "positive", seed=4).numpy()
    assert oracle_mod.maxsub(pos) == (int(pos.astype(np.int64).sum()), 0, n - 1)
    neg = dcgen.maxsub_input(n, "negative", seed=4).numpy()
    am = int(np.argmax(neg))                       # first occurrence of the max
    assert oracle_mod.maxsub(neg) == (int(neg[am]), am, am)
    assert oracle_mod.maxsub(np.zeros(n, np.int32)) == (0, 0, 0)
    spike = np.full(n, -3, np.int32)
    spike[1234] = 99
    assert oracle_mod.maxsub(spike) == (99, 1234, 1234)
    big = np.full(4096, 2**31 - 1, np.int32)       # int64 accumulation is exact
    assert oracle_mod.maxsub(big) == ((2**31 - 1) * 4096, 0, 4095)
    small = np.full(4096, -2**31, np.int32)
    assert oracle_mod.maxsub(small) == (-2**31, 0, 0)


@pytest.mark.parametrize("k", [1, 4, 12])
def test_maxsub_level_counts(oracle_mod, k):
    n = 1 << k
    x = dcgen.maxsub_input(n, "small", seed=1).numpy()
    _, lc = oracle_mod.maxsub(x, counters=True)
    for d in range(k):
        assert lc[d] == 2 ** d
    assert np.all(lc[k:] == 0)


def test_maxsub_rejects_empty(oracle_mod):
    with pytest.raises(ValueError):
        oracle_mod.maxsub(np.zeros(0, np.int32))


# ------------------------------------------------------------------- sum

@pytest.mark.parametrize("n", [1, 2, 3, 1000, 1 << 16, 100003])
def test_dc_sum_matches_exact_sum(oracle_mod, n):
    x = dcgen.maxsub_input(n, "uniform", seed=21).numpy().astype(np.int64) * 1000
    assert oracle_mod.dc_sum(x) == sum(int(v) for v in x)


# -------------------------------------------------------------- generators

def test_splitmix64_torch_matches_python():
    z = dcgen.splitmix64(12345, 0, 64)
    for i in range(64):
        assert (int(z[i]) & ((1 << 64) - 1)) == dcgen.splitmix64_py(12345, i)
    z2 = dcgen.splitmix64(7, 1_000_000, 4)
    for j in range(4):
        assert (int(z2[j]) & ((1 << 64) - 1)) == dcgen.splitmix64_py(7, 1_000_000 + j)


def test_generators_shard_consistently():
    n = 10000
    full = dcgen.sort_keys(n, "uniform", seed=3)
    parts = [dcgen.sort_keys(n, "uniform", seed=3, start=r * 2500, count=2500) for r in range(4)]
    assert all(np.array_equal(full[r * 2500:(r + 1) * 2500].numpy(), parts[r].numpy())
               for r in range(4))


def test_generator_distributions():
    n = 1 << 14
    few = dcgen.sort_keys(n, "few").numpy().view(np.uint32)
    assert len(np.unique(few)) <= 16
    s = dcgen.sort_keys(n, "sorted").numpy().view(np.uint32)
    assert np.all(s[1:] > s[:-1])
    r = dcgen.sort_keys(n, "reverse").numpy().view(np.uint32)
    assert np.all(r[1:] < r[:-1])
    p = dcgen.sort_keys(n, "paper").numpy().view(np.uint32)
    assert p.max() <= 2 * n - 1
    f = dcgen.sort_keys(n, "uniform", key_type="f32").numpy()
    assert np.all(np.isfinite(f))
    bits = f.view(np.uint32)
    assert np.any(bits == 0x80000000) and np.any(bits == 0)
    assert math.isclose(float((dcgen.maxsub_input(n, "small").numpy() > 0).mean()), 0.5,
                        abs_tol=0.05)
