"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Tolerance 0 everywhere (north star): keys and values are compared bit for bit
(float keys included: +/-0.0 must keep their input order), max-subarray
(sum, start, end) exactly.  Sizes span one tile, several tiles and ragged
tails; BASELINE's full sizes are checked by properties that identify the
stable sort uniquely (see test_full_size_*).
"""
import numpy as np
import pytest
import torch

import dcgen

pytestmark = pytest.mark.gpu

TILE = 25088  # keys-only fused tile (512 x 49) from 2^23 keys; f32 16896, key-value 8448


@pytest.fixture(scope="module")
def dc():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_ipps_lopez_ortizss13_b200 as m
    return m


def _np_keys(t, key_type):
    a = t.cpu().numpy()
    return a.view(np.uint32) if key_type == "u32" else (a.view(np.int32) if key_type == "i32" else a)


def run_sort(dc, n, dist, key_type="u32", with_vals=False, seed=1, two=None):
    keys = dcgen.sort_keys(n, dist, seed=seed, key_type=key_type, device="cuda")
    vals = dcgen.sort_vals(n, device="cuda") if with_vals else None
    k_in = keys.clone()
    plan = dc.Plan(n)
    if two is not None:
        plan.set_two_level(two)
    plan.sort_(keys, vals, key_type=key_type)
    torch.cuda.synchronize()
    return k_in, keys, vals


SIZES = [1, 2, 3, 4, 5, 15, 16, 17, 255, 1000, TILE - 1, TILE, TILE + 1, 2 * TILE, 3 * TILE + 5,
         (1 << 16) + 3, 100_003, (1 << 20), (1 << 20) + 12345]


@pytest.mark.parametrize("n", SIZES)
@pytest.mark.parametrize("dist", ["uniform", "few"])
def test_sort_u32_sizes(dc, oracle_mod, n, dist):
    k_in, k_out, _ = run_sort(dc, n, dist)
    expect = oracle_mod.mergesort(_np_keys(k_in, "u32"))
    assert np.array_equal(_np_keys(k_out, "u32"), expect)


@pytest.mark.parametrize("dist", ["uniform", "paper", "sorted", "reverse", "few", "equal"])
@pytest.mark.parametrize("n", [(1 << 20) + 7, 1 << 22])
def test_sort_u32_distributions(dc, oracle_mod, n, dist):
    k_in, k_out, _ = run_sort(dc, n, dist, seed=3)
    assert np.array_equal(_np_keys(k_out, "u32"), oracle_mod.mergesort(_np_keys(k_in, "u32")))


@pytest.mark.parametrize("key_type", ["u32", "i32", "f32"])
@pytest.mark.parametrize("n", [5, TILE + 3, 300_001, 1 << 21])
@pytest.mark.parametrize("dist", ["uniform", "few"])
def test_sort_key_value_stable(dc, oracle_mod, key_type, n, dist):
    k_in, k_out, v_out = run_sort(dc, n, dist, key_type, with_vals=True, seed=7)
    ek, ev = oracle_mod.mergesort(_np_keys(k_in, key_type), np.arange(n, dtype=np.uint32),
                                  key_type=key_type)
    assert np.array_equal(_np_keys(k_out, key_type).view(np.uint32), ek.view(np.uint32))
    assert np.array_equal(v_out.cpu().numpy().view(np.uint32), ev)


@pytest.mark.parametrize("key_type", ["i32", "f32"])
@pytest.mark.parametrize("n", [1000, TILE * 5 + 17, 1 << 20])
def test_sort_keys_only_signed_float(dc, oracle_mod, key_type, n):
    k_in, k_out, _ = run_sort(dc, n, "uniform", key_type, seed=9)
    ek = oracle_mod.mergesort(_np_keys(k_in, key_type), key_type=key_type)
    assert np.array_equal(_np_keys(k_out, key_type).view(np.uint32), ek.view(np.uint32))


# n >= 2^23 uses the large-tile config (the one with two-level passes)
TWO_LEVEL_SIZES = [(1 << 23) + 7, 3 * (1 << 22) + 5, (1 << 24) + 3 * TILE + 11]


@pytest.mark.parametrize("n", TWO_LEVEL_SIZES)
@pytest.mark.parametrize("dist", ["uniform", "few", "reverse"])
@pytest.mark.parametrize("key_type", ["u32", "i32"])
def test_sort_two_level_vs_one_level(dc, oracle_mod, n, dist, key_type):
    """Two merge levels per HBM pass (f1) and one level per pass give the oracle's result."""
    keys = dcgen.sort_keys(n, dist, seed=13, key_type=key_type, device="cuda")
    k_in = _np_keys(keys, key_type)
    expect = oracle_mod.mergesort(k_in, key_type=key_type).view(np.uint32)
    for two in (True, False):
        k = keys.clone()
        plan = dc.Plan(n)
        plan.set_two_level(two)
        plan.sort_(k, key_type=key_type)
        assert np.array_equal(_np_keys(k, key_type).view(np.uint32), expect), two


# one group of four runs, several groups with a partial last group, ragged tails
TWO_LEVEL_EDGE = [(1 << 23) + 1, 4 * TILE * 128 + TILE * 5 + 3, 4 * 52224 * 64 + 52224 * 5 + 3, (1 << 25) - 5]


@pytest.mark.parametrize("n", TWO_LEVEL_EDGE)
@pytest.mark.parametrize("dist", ["sorted", "equal", "paper", "maxkeys", "blocks"])
def test_sort_two_level_edge_distributions(dc, oracle_mod, n, dist):
    """4-way passes: the exact 4-run selection on ties, presorted runs and pad-valued keys."""
    if dist == "maxkeys":      # real keys equal to the +inf pad of the pad-safe merges
        keys = dcgen.sort_keys(n, "few", seed=21, device="cuda")
        keys[keys.remainder(3) == 0] = -1
    elif dist == "blocks":     # runs whose key ranges are disjoint / nested
        keys = dcgen.sort_keys(n, "uniform", seed=22, device="cuda").remainder(1 << 12)
        keys += (torch.arange(n, device="cuda") // TILE % 4) * (1 << 12)
        keys = keys.to(torch.int32)
    else:
        keys = dcgen.sort_keys(n, dist, seed=23, device="cuda")
    expect = oracle_mod.mergesort(_np_keys(keys, "u32"), key_type="u32")
    plan = dc.Plan(n)
    plan.set_two_level(True)
    plan.sort_(keys, key_type="u32")
    assert np.array_equal(_np_keys(keys, "u32"), expect)


STABLE_TWO_LEVEL = [(1 << 23) + 7, 5 * 16896 * 128 + 16896 * 3 + 11, 9 * 8448 * 128 + 8448 * 5 + 13]


@pytest.mark.parametrize("n", STABLE_TWO_LEVEL)
@pytest.mark.parametrize("dist", ["uniform", "few", "equal"])
@pytest.mark.parametrize("key_type,with_vals", [("u32", True), ("i32", True), ("f32", True),
                                                ("f32", False)])
def test_sort_two_level_stable(dc, oracle_mod, n, dist, key_type, with_vals):
    """Stable 4-way passes (values, or f32 keys with +0/-0): ties keep run order."""
    k_in, k_out, v_out = run_sort(dc, n, dist, key_type, with_vals, seed=29, two=True)
    p2 = dc.Plan(n)
    p2.set_two_level(True)
    plan_sched = p2.schedule(key_type, with_vals)
    assert plan_sched["hbm_passes"] < plan_sched["global_passes"]      # 4-way passes ran
    vals_in = np.arange(n, dtype=np.uint32) if with_vals else None
    res = oracle_mod.mergesort(_np_keys(k_in, key_type), vals_in, key_type=key_type)
    ek = res[0] if with_vals else res
    assert np.array_equal(_np_keys(k_out, key_type).view(np.uint32), ek.view(np.uint32))
    if with_vals:
        assert np.array_equal(v_out.cpu().numpy().view(np.uint32), res[1])


def test_sort_max_key_values_and_pads(dc, oracle_mod):
    # real keys equal to the pad value (0xFFFFFFFF) in a ragged last tile
    n = 3 * TILE + 100
    keys = torch.full((n,), -1, dtype=torch.int32, device="cuda")
    keys[::3] = 5
    vals = dcgen.sort_vals(n, device="cuda")
    k_in = keys.clone()
    dc.Plan(n).sort_(keys, vals, key_type="u32")
    ek, ev = oracle_mod.mergesort(_np_keys(k_in, "u32"), np.arange(n, dtype=np.uint32))
    assert np.array_equal(_np_keys(keys, "u32"), ek)
    assert np.array_equal(vals.cpu().numpy().view(np.uint32), ev)


@pytest.mark.parametrize("n", [(1 << 23) + 7, 4 * TILE * 128 + TILE * 5 + 3])
@pytest.mark.parametrize("with_vals", [False, True])
def test_sort_i32_pad_valued_keys_two_level(dc, oracle_mod, n, with_vals):
    """i32 keys equal to KeyI32::kPad (INT32_MAX) -- the value the pad-safe
    4-way merges put behind every piece -- mixed with INT32_MIN and ordinary
    keys, on the two-level schedule (keys-only pad-safe path and the stable
    key-value path)."""
    keys = dcgen.sort_keys(n, "few", seed=31, key_type="i32", device="cuda")
    sel = torch.arange(n, device="cuda")
    keys[sel % 3 == 0] = 2**31 - 1
    keys[sel % 7 == 1] = -2**31
    vals = dcgen.sort_vals(n, device="cuda") if with_vals else None
    k_in = _np_keys(keys, "i32").copy()
    plan = dc.Plan(n)
    plan.set_two_level(True)
    assert plan.schedule("i32", with_vals)["hbm_passes"] < plan.schedule("i32", with_vals)["global_passes"]
    plan.sort_(keys, vals, key_type="i32")
    if with_vals:
        ek, ev = oracle_mod.mergesort(k_in, np.arange(n, dtype=np.uint32), key_type="i32")
        assert np.array_equal(vals.cpu().numpy().view(np.uint32), ev)
    else:
        ek = oracle_mod.mergesort(k_in, key_type="i32")
    assert np.array_equal(_np_keys(keys, "i32"), ek)


@pytest.mark.parametrize("n", [TILE * 3 + 11, (1 << 20) + 3, (1 << 23) + 7])
@pytest.mark.parametrize("with_vals", [False, True])
def test_sort_f32_infinities_and_signed_zeros(dc, oracle_mod, n, with_vals):
    """f32 keys include +inf (== KeyF32::kPad, the pad of ragged tiles and of
    the 4-way pieces), -inf, +0.0 and -0.0 (equal keys with distinct bits,
    which must keep their input order), on the small, one-level and two-level
    schedules, keys only and with values."""
    keys = dcgen.sort_keys(n, "uniform", seed=33, key_type="f32", device="cuda")
    sel = torch.arange(n, device="cuda")
    keys[sel % 5 == 0] = float("inf")
    keys[sel % 11 == 2] = float("-inf")
    keys[sel % 13 == 3] = 0.0
    keys[sel % 17 == 4] = -0.0
    vals = dcgen.sort_vals(n, device="cuda") if with_vals else None
    k_in = _np_keys(keys, "f32").copy()
    dc.Plan(n).sort_(keys, vals, key_type="f32")
    if with_vals:
        ek, ev = oracle_mod.mergesort(k_in, np.arange(n, dtype=np.uint32), key_type="f32")
        assert np.array_equal(vals.cpu().numpy().view(np.uint32), ev)
    else:
        ek = oracle_mod.mergesort(k_in, key_type="f32")
    assert np.array_equal(_np_keys(keys, "f32").view(np.uint32), ek.view(np.uint32))


@pytest.mark.parametrize("n", [1 << 20, (1 << 23) + 5])
def test_graph_cache_survives_scratch_reallocation(dc, oracle_mod, n):
    """a keys-only sort is captured as a CUDA graph; a key-value
    sort on other buffers then needs a larger scratch (reallocated); replaying
    keys-only on the first buffers must not touch the freed scratch."""
    plan = dc.Plan(n)
    keys = torch.empty(n, dtype=torch.int32, device="cuda")
    for seed in range(3):            # eager, capture, replay
        keys.copy_(dcgen.sort_keys(n, "uniform", seed=60 + seed, device="cuda"))
        k_in = _np_keys(keys, "u32").copy()
        plan.sort_(keys, key_type="u32")
        assert np.array_equal(_np_keys(keys, "u32"), oracle_mod.mergesort(k_in)), seed
    k2 = dcgen.sort_keys(n, "few", seed=64, device="cuda")
    v2 = dcgen.sort_vals(n, device="cuda")
    k2_in = _np_keys(k2, "u32").copy()
    plan.sort_(k2, v2, key_type="u32")                 # reallocates the scratch
    ek, ev = oracle_mod.mergesort(k2_in, np.arange(n, dtype=np.uint32))
    assert np.array_equal(_np_keys(k2, "u32"), ek)
    assert np.array_equal(v2.cpu().numpy().view(np.uint32), ev)
    del k2, v2
    torch.cuda.empty_cache()
    junk = torch.full((2 * n,), 7, dtype=torch.int32, device="cuda")   # reuse freed memory
    for seed in range(2):
        keys.copy_(dcgen.sort_keys(n, "reverse", seed=70 + seed, device="cuda"))
        k_in = _np_keys(keys, "u32").copy()
        plan.sort_(keys, key_type="u32")
        assert np.array_equal(_np_keys(keys, "u32"), oracle_mod.mergesort(k_in)), seed
    assert bool((junk == 7).all())


def test_host_submit_then_device_sort_ordering(dc, oracle_mod):
    """host-slot sorts run on their own stream with the plan
    scratch; a device sort enqueued right after them on the plan stream must
    wait for them (dc.h: later scratch users are ordered after submissions)."""
    n = (1 << 23) + 77
    plan = dc.Plan(n)
    ins = [dcgen.sort_keys(n, d, seed=80 + i).pin_memory()
           for i, d in enumerate(["uniform", "few", "reverse"])]
    outs = [torch.empty_like(t).pin_memory() for t in ins]
    dev_keys = dcgen.sort_keys(n, "uniform", seed=90, device="cuda")
    dk_in = _np_keys(dev_keys, "u32").copy()
    for t, o in zip(ins, outs):
        plan.sort_host_submit(t, o, key_type="u32")
    plan.sort_(dev_keys, key_type="u32")                # same scratch, plan stream
    plan.sort_host_wait()
    torch.cuda.synchronize()
    assert np.array_equal(_np_keys(dev_keys, "u32"), oracle_mod.mergesort(dk_in))
    for t, o in zip(ins, outs):
        assert np.array_equal(_np_keys(o, "u32"), oracle_mod.mergesort(_np_keys(t, "u32")))


@pytest.mark.parametrize("tile_class,two", [(1, True), (1, False), (2, True), (2, False)])
@pytest.mark.parametrize("key_type,with_vals", [("u32", False), ("i32", False), ("f32", False),
                                                ("u32", True)])
@pytest.mark.parametrize("n", [(1 << 20) + 3, 3 * (1 << 21) + 5])
def test_sort_every_forced_schedule(dc, oracle_mod, tile_class, two, key_type, with_vals, n):
    """Every schedule the planner can choose (quarter / full tiles x one / two
    levels per HBM pass) gives the oracle's result bit for bit."""
    keys = dcgen.sort_keys(n, "few" if n % 2 else "uniform", seed=51, key_type=key_type,
                           device="cuda")
    vals = dcgen.sort_vals(n, device="cuda") if with_vals else None
    k_np = _np_keys(keys, key_type).copy()
    plan = dc.Plan(n)
    plan.set_tile_class(tile_class)
    plan.set_two_level(two)
    sch = plan.schedule(key_type, with_vals)
    if two and sch["global_passes"] >= 2:
        assert sch["hbm_passes"] < sch["global_passes"]
    plan.sort_(keys, vals, key_type=key_type)
    if with_vals:
        ek, ev = oracle_mod.mergesort(k_np, np.arange(n, dtype=np.uint32), key_type=key_type)
        assert np.array_equal(vals.cpu().numpy().view(np.uint32), ev)
    else:
        ek = oracle_mod.mergesort(k_np, key_type=key_type)
    assert np.array_equal(_np_keys(keys, key_type).view(np.uint32), ek.view(np.uint32))


SMALL_TILE = 128 * 49        # keys-only quarter tile (the planner's choice below 2^23 keys)


@pytest.mark.parametrize("n", [SMALL_TILE - 1, SMALL_TILE, SMALL_TILE + 1, 2 * SMALL_TILE + 3,
                               7 * SMALL_TILE, (1 << 23) - 1])
@pytest.mark.parametrize("with_vals", [False, True])
def test_sort_small_config_boundaries(dc, oracle_mod, n, with_vals):
    k_in, k_out, v_out = run_sort(dc, n, "few", "u32", with_vals, seed=17)
    if with_vals:
        ek, ev = oracle_mod.mergesort(_np_keys(k_in, "u32"), np.arange(n, dtype=np.uint32))
        assert np.array_equal(v_out.cpu().numpy().view(np.uint32), ev)
    else:
        ek = oracle_mod.mergesort(_np_keys(k_in, "u32"))
    assert np.array_equal(_np_keys(k_out, "u32"), ek)


@pytest.mark.parametrize("n", [SMALL_TILE + 1, 5 * SMALL_TILE + 77, 1 << 20, (1 << 22) + 3])
@pytest.mark.parametrize("key_type,with_vals", [("u32", False), ("i32", False), ("f32", False),
                                                ("u32", True)])
def test_sort_small_partition_fused_vs_separate(dc, oracle_mod, n, key_type, with_vals):
    """L2-resident sorts: merge CTAs that find their own co-ranks (default) and
    the separate NK2 launch give the oracle's result bit for bit."""
    keys = dcgen.sort_keys(n, "few" if n % 2 else "uniform", seed=77, key_type=key_type,
                           device="cuda")
    k_np = _np_keys(keys, key_type)
    if with_vals:
        ek, ev = oracle_mod.mergesort(k_np, np.arange(n, dtype=np.uint32), key_type=key_type)
    else:
        ek = oracle_mod.mergesort(k_np, key_type=key_type)
    for fused in (True, False):
        k = keys.clone()
        v = dcgen.sort_vals(n, device="cuda") if with_vals else None
        plan = dc.Plan(n)
        plan.set_fused_partition(fused)
        plan.sort_(k, v, key_type=key_type)
        torch.cuda.synchronize()
        assert np.array_equal(_np_keys(k, key_type).view(np.uint32), ek.view(np.uint32)), fused
        if with_vals:
            assert np.array_equal(v.cpu().numpy().view(np.uint32), ev), fused


@pytest.mark.parametrize("n", [1 << 20, (1 << 23) + 5])
def test_sort_graph_replay_same_buffers(dc, oracle_mod, n):
    """First call eager, second captures a CUDA graph, later calls replay it."""
    plan = dc.Plan(n)
    keys = torch.empty(n, dtype=torch.int32, device="cuda")
    vals = torch.empty(n, dtype=torch.int32, device="cuda")
    for seed in range(4):
        keys.copy_(dcgen.sort_keys(n, "uniform", seed=40 + seed, device="cuda"))
        vals.copy_(dcgen.sort_vals(n, device="cuda"))
        k_in = _np_keys(keys, "u32")
        plan.sort_(keys, vals, key_type="u32")
        ek, ev = oracle_mod.mergesort(k_in, np.arange(n, dtype=np.uint32))
        assert np.array_equal(_np_keys(keys, "u32"), ek), seed
        assert np.array_equal(vals.cpu().numpy().view(np.uint32), ev), seed


@pytest.mark.parametrize("chunks", [0, 2, 3, 8, 16])
@pytest.mark.parametrize("n,with_vals", [((1 << 24) + 12345, False), ((1 << 23) + 77, True)])
def test_sort_chunked_pipeline(dc, oracle_mod, chunks, n, with_vals):
    """Chunk streams (each chunk's NK1 + in-chunk levels) then the top levels."""
    keys = dcgen.sort_keys(n, "few" if with_vals else "uniform", seed=19, device="cuda")
    vals = dcgen.sort_vals(n, device="cuda") if with_vals else None
    k_in = _np_keys(keys, "u32")
    plan = dc.Plan(n)
    plan.set_pipeline(chunks)
    for rep in range(3):                 # eager, graph capture, graph replay
        k = keys.clone()
        v = vals.clone() if with_vals else None
        plan.sort_(k, v, key_type="u32")
        if with_vals:
            ek, ev = oracle_mod.mergesort(k_in, np.arange(n, dtype=np.uint32))
            assert np.array_equal(v.cpu().numpy().view(np.uint32), ev), rep
        else:
            ek = oracle_mod.mergesort(k_in)
        assert np.array_equal(_np_keys(k, "u32"), ek), rep


def test_sort_repeated_runs_same_plan(dc, oracle_mod):
    n = 50_000
    plan = dc.Plan(n)
    for seed in range(3):
        keys = dcgen.sort_keys(n, "uniform", seed=seed, device="cuda")
        k_in = keys.clone()
        plan.sort_(keys, key_type="u32")
        assert np.array_equal(_np_keys(keys, "u32"), oracle_mod.mergesort(_np_keys(k_in, "u32")))


def test_sort_host_buffers(dc, oracle_mod):
    n = 123_457
    keys = dcgen.sort_keys(n, "few", seed=2).pin_memory()
    vals = dcgen.sort_vals(n).pin_memory()
    k_in = keys.clone()
    dc.Plan(n).sort_host_(keys, vals, key_type="u32")
    ek, ev = oracle_mod.mergesort(_np_keys(k_in, "u32"), np.arange(n, dtype=np.uint32))
    assert np.array_equal(_np_keys(keys, "u32"), ek)
    assert np.array_equal(vals.numpy().view(np.uint32), ev)


@pytest.mark.parametrize("with_vals", [False, True])
def test_sort_host_streaming(dc, oracle_mod, with_vals):
    """Streaming submissions (two device slots, overlapped copies) of several
    distinct inputs; the inputs stay unmodified, each output is its own sort."""
    n = 3 * 8192 + 1001 if not with_vals else (1 << 23) + 77
    plan = dc.Plan(n)
    ins = [dcgen.sort_keys(n, d, seed=s).pin_memory()
           for s, d in enumerate(["uniform", "few", "reverse", "paper", "uniform"])]
    keep = [t.clone() for t in ins]
    outs = [torch.empty_like(t).pin_memory() for t in ins]
    vin = dcgen.sort_vals(n).pin_memory() if with_vals else None
    vouts = [torch.empty_like(vin).pin_memory() if with_vals else None for _ in ins]
    for t, o, vo in zip(ins, outs, vouts):
        plan.sort_host_submit(t, o, vin, vo, key_type="u32")
    plan.sort_host_wait()
    for t, k, o, vo in zip(ins, keep, outs, vouts):
        assert torch.equal(t, k)
        ek, ev = oracle_mod.mergesort(_np_keys(k, "u32"), np.arange(n, dtype=np.uint32))
        assert np.array_equal(_np_keys(o, "u32"), ek)
        if with_vals:
            assert np.array_equal(vo.numpy().view(np.uint32), ev)


def test_sort_2pow24_against_oracle(dc, oracle_mod):
    n = 1 << 24
    k_in, k_out, v_out = run_sort(dc, n, "uniform", with_vals=True, seed=3)
    ek, ev = oracle_mod.mergesort(_np_keys(k_in, "u32"), np.arange(n, dtype=np.uint32))
    assert np.array_equal(_np_keys(k_out, "u32"), ek)
    assert np.array_equal(v_out.cpu().numpy().view(np.uint32), ev)


def _assert_is_stable_sort(k_in_u32, k_out_u32, v_out):
    """(k_out, v_out) is THE stable sort of k_in when: v_out is a permutation,
    k_out[i] == k_in[v_out[i]], keys non-decreasing, and v_out increasing inside
    every run of equal keys.  Holds at any size, no oracle needed."""
    n = k_in_u32.numel()
    v = v_out.to(torch.int64) & 0xFFFFFFFF
    assert torch.equal(torch.bincount(v, minlength=n), torch.ones(n, dtype=torch.int64,
                                                                 device=v.device))
    kin = k_in_u32.to(torch.int64) & 0xFFFFFFFF
    kout = k_out_u32.to(torch.int64) & 0xFFFFFFFF
    assert torch.equal(kin[v], kout)
    assert bool((kout[1:] >= kout[:-1]).all())
    eq = kout[1:] == kout[:-1]
    assert bool((v[1:][eq] > v[:-1][eq]).all())


@pytest.mark.parametrize("dist", ["uniform", "few"])
def test_full_size_2pow28_key_value(dc, dist):
    n = 1 << 28
    keys = dcgen.sort_keys(n, dist, seed=3, device="cuda")
    vals = dcgen.sort_vals(n, device="cuda")
    k_in = keys.clone()
    dc.Plan(n).sort_(keys, vals, key_type="u32")
    torch.cuda.synchronize()
    _assert_is_stable_sort(k_in, keys, vals)
    # sampled oracle positions: the i-th output is the i-th smallest key
    del vals
    torch.cuda.empty_cache()


def _assert_sorted_permutation_u32(k_in, k_out, samples=12, seed=0):
    """Properties that hold at any size, checked without another sort:
    the output is non-decreasing; it is a permutation of the input (histogram
    of the top 16 key bits and the exact key sum agree); and sampled outputs
    have the right rank -- out[i] = o satisfies #(in < o) <= i < #(in <= o),
    counted over the input (the definition of the i-th smallest key)."""
    n = k_in.numel()
    kin = k_in.to(torch.int64) & 0xFFFFFFFF
    kout = k_out.to(torch.int64) & 0xFFFFFFFF
    assert bool((kout[1:] >= kout[:-1]).all())
    assert int(kin.sum()) == int(kout.sum())
    assert torch.equal(torch.bincount(kin >> 16, minlength=1 << 16),
                       torch.bincount(kout >> 16, minlength=1 << 16))
    g = torch.Generator().manual_seed(seed)
    idx = [0, n - 1] + torch.randint(0, n, (samples,), generator=g).tolist()
    for i in idx:
        o = int(kout[i])
        assert int((kin < o).sum()) <= i < int((kin <= o).sum())


@pytest.mark.parametrize("dist", ["uniform", "sorted", "reverse", "few"])
def test_full_size_2pow28_keys_exact(dc, oracle_mod, dist):
    """BASELINE configs[2] at its full size, in the launch configuration bench.py
    times (the default plan, i.e. the planner's schedule for 2^28 u32 keys):
    every one of the 2^28 outputs equals the oracle's Alg 6 mergesort of the
    same input (seed 3, as bench.py), element by element."""
    n = 1 << 28
    keys = dcgen.sort_keys(n, dist, seed=3, device="cuda")
    k_in = _np_keys(keys, "u32").copy()
    plan = dc.Plan(n)
    plan.sort_(keys, key_type="u32")
    torch.cuda.synchronize()
    got = _np_keys(keys, "u32")
    del keys
    plan.close()
    torch.cuda.empty_cache()
    expect = oracle_mod.mergesort(k_in)
    assert np.array_equal(got, expect)


def test_max_size_keys(dc):
    """n = 2^31 - 1, the largest per-GPU size of the ABI (16-17 global passes
    depending on the tile, int32 co-ranks at their limit)."""
    n = (1 << 31) - 1
    keys = dcgen.sort_keys(n, "uniform", seed=7, device="cuda")
    k_in = keys.clone()
    plan = dc.Plan(n)
    sch = plan.schedule("u32")
    runs = -(-n // sch["tile"])
    assert sch["global_passes"] == (runs - 1).bit_length() >= 16
    plan.sort_(keys, key_type="u32")
    torch.cuda.synchronize()
    del plan
    _assert_sorted_permutation_u32(k_in, keys, samples=6)
    del keys, k_in
    torch.cuda.empty_cache()


# ------------------------------------------------------------ max-subarray

MS_TILE = 256 * 256      # max-subarray CTA tile (256 threads x 256-element chunks)
MS_SIZES = [1, 2, 3, 31, 32, 33, 255, 256, 257, 1000, 8191, 8192, 8193, 3 * 8192 + 77,
            MS_TILE - 1, MS_TILE, MS_TILE + 1, 5 * MS_TILE + 4097, 100_003, 1 << 20,
            (1 << 20) + 5, 1 << 24, (1 << 24) + 3]


@pytest.mark.parametrize("n", MS_SIZES)
@pytest.mark.parametrize("dist", ["uniform", "small"])
def test_maxsub_sizes(dc, oracle_mod, n, dist):
    x = dcgen.maxsub_input(n, dist, seed=2, device="cuda")
    got = dc.Plan(n).max_subarray(x)
    assert got == oracle_mod.maxsub(x.cpu().numpy())


@pytest.mark.parametrize("dist", ["negative", "positive", "zero"])
@pytest.mark.parametrize("n", [1, 777, 1 << 16, (1 << 20) + 3])
def test_maxsub_degenerate(dc, oracle_mod, n, dist):
    x = dcgen.maxsub_input(n, dist, seed=5, device="cuda")
    got = dc.Plan(n).max_subarray(x)
    assert got == oracle_mod.maxsub(x.cpu().numpy())


def test_maxsub_extremes_and_ties(dc, oracle_mod):
    n = 70_000
    x = torch.full((n,), 2**31 - 1, dtype=torch.int32, device="cuda")
    assert dc.Plan(n).max_subarray(x) == ((2**31 - 1) * n, 0, n - 1)
    x = torch.full((n,), -2**31, dtype=torch.int32, device="cuda")
    assert dc.Plan(n).max_subarray(x) == (-2**31, 0, 0)
    # many equal maxima spread over tile boundaries: lexicographically smallest wins
    x = torch.full((n,), -1, dtype=torch.int32, device="cuda")
    x[8191] = 4; x[8192] = -4; x[8193] = 4; x[20000] = 4
    got = dc.Plan(n).max_subarray(x)
    assert got == oracle_mod.maxsub(x.cpu().numpy()) == (4, 8191, 8191)
    x = torch.zeros(n, dtype=torch.int32, device="cuda")
    x[100] = -1
    assert dc.Plan(n).max_subarray(x) == oracle_mod.maxsub(x.cpu().numpy()) == (0, 0, 0)


def test_maxsub_tuple_and_combine(dc, oracle_mod):
    n = 1 << 20
    g = 4
    x = dcgen.maxsub_input(n, "small", seed=8, device="cuda")
    m = n // g
    tups = torch.empty((g, 8), dtype=torch.int64, device="cuda")
    plans = [dc.Plan(m) for _ in range(g)]
    for r in range(g):
        plans[r].max_subarray_tuple_async(x[r * m:(r + 1) * m], tups[r], index_offset=r * m)
    out = torch.empty(3, dtype=torch.int64, device="cuda")
    plans[0].maxsub_combine_async(tups, out)
    assert tuple(out.cpu().tolist()) == oracle_mod.maxsub(x.cpu().numpy())


@pytest.mark.parametrize("n", [67, 68, 69, 2176, 2177, 70_001, 1 << 20])
@pytest.mark.parametrize("lo", [-1, -2])
def test_maxsub_tie_heavy(dc, oracle_mod, n, lo):
    # values in {lo..1}: many equal maxima, equal prefix/suffix maxima across
    # lane-chunk (68) and segment (32*68) boundaries; exercises the chunk-label
    # recovery of the values-only fold (R13)
    g = torch.Generator().manual_seed(n * 7 + lo)
    x = torch.randint(lo, 2, (n,), generator=g, dtype=torch.int32)
    assert dc.Plan(n).max_subarray(x.cuda()) == oracle_mod.maxsub(x.numpy())


@pytest.mark.parametrize("n", [1, 68, 69, 4353, 1 << 20])
def test_maxsub_tuple_prefix_suffix(dc, n):
    # whole-array summary: pe = first argmax of the prefix sums, ss = first
    # argmax of the suffix sums, tot = the total (numpy brute force)
    g = torch.Generator().manual_seed(n)
    x = torch.randint(-3, 3, (n,), generator=g, dtype=torch.int32)
    tup = torch.empty(8, dtype=torch.int64, device="cuda")
    off = 1000
    dc.Plan(n).max_subarray_tuple_async(x.cuda(), tup, index_offset=off)
    t = tup.cpu().tolist()
    a = x.numpy().astype(np.int64)
    pre = np.cumsum(a)
    suf = np.cumsum(a[::-1])[::-1]
    assert t[0] == int(a.sum())
    assert (t[1], t[4]) == (int(pre.max()), int(np.argmax(pre)) + off)
    assert (t[2], t[5]) == (int(suf.max()), int(np.argmax(suf)) + off)


def test_maxsub_host_buffer(dc, oracle_mod):
    n = 300_000
    x = dcgen.maxsub_input(n, "small", seed=6).pin_memory()
    assert dc.Plan(n).max_subarray_host(x) == oracle_mod.maxsub(x.numpy())


@pytest.mark.parametrize("n,fused", [(1 << 20, True), (1 << 20, False), ((1 << 23) + 5, True)])
def test_launch_counts(dc, n, fused):
    """NK1 + per pass: NK2 + NK3 (a two-level pass: select + 4-way merge); below
    2^23 keys the fused partition makes a one-level pass a single launch."""
    p = dc.Plan(n)
    p.set_graphs(False)
    p.set_fused_partition(fused)
    keys = dcgen.sort_keys(n, "uniform", device="cuda")
    p.sort_(keys, key_type="u32")
    s = p.schedule("u32", False)
    P, H = s["global_passes"], s["hbm_passes"]
    single = P - 2 * (P - H)          # one-level passes; the rest are two-level passes
    per_single = 1 if (fused and s["tile"] == 128 * 49) else 2   # quarter tiles: fused partition
    assert p.launch_count() == 1 + per_single * single + 2 * (H - single)


# ---------------------------------------------------------------- f2 clusters
@pytest.mark.parametrize("cs", [2, 4, 8, 16])
@pytest.mark.parametrize("tile_class", [1, 2])
@pytest.mark.parametrize("key_type", ["u32", "i32"])
def test_sort_nk1_cluster_levels(dc, oracle_mod, cs, tile_class, key_type):
    """NK1 with log2(cs) cluster levels (distributed shared memory,
    nk1_blocksort_cl): bit-exact against the oracle for a partial last
    cluster, a ragged tail, a single tile, both pass kinds."""
    tile = 6272 if tile_class == 1 else 25088
    for n, dist in [(1, "uniform"), (tile - 3, "few"), (cs * tile + 1, "uniform"),
                    (3 * cs * tile + 4099, "uniform"), (5 * cs * tile // 2 + 17, "reverse"),
                    (1 << 20, "sorted")]:
        keys = dcgen.sort_keys(n, dist, seed=47, key_type=key_type, device="cuda")
        ka = keys.cpu().numpy()
        ka = ka.view(np.uint32) if key_type == "u32" else ka.view(np.int32)
        ek = oracle_mod.mergesort(ka, key_type=key_type)
        for two in (False, True):
            k = keys.clone()
            plan = dc.Plan(n)
            plan.set_tile_class(tile_class)
            plan.set_two_level(two)
            plan.set_nk1_cluster(cs)
            assert plan.schedule(key_type)["tile"] == tile * cs
            # three runs on the same buffers: eager, graph capture, graph replay
            for rep in range(3):
                k.copy_(keys)
                plan.sort_(k, None, key_type=key_type)
                torch.cuda.synchronize()
                assert np.array_equal(k.cpu().numpy().view(ek.dtype), ek), (n, dist, two, rep)


def test_sort_nk1_cluster_ignored_for_stable_sorts(dc, oracle_mod):
    """Key-value and f32 sorts run the plain NK1 whatever the cluster setting."""
    n = 3 * 25088 + 5
    plan = dc.Plan(n)
    plan.set_nk1_cluster(8)
    assert plan.schedule("u32", with_vals=True)["tile"] in (8448, 4224)
    keys = dcgen.sort_keys(n, "few", seed=5, device="cuda")
    vals = dcgen.sort_vals(n, device="cuda")
    ek, ev = oracle_mod.mergesort(keys.cpu().numpy().view(np.uint32),
                                  np.arange(n, dtype=np.uint32))
    plan.sort_(keys, vals, key_type="u32")
    torch.cuda.synchronize()
    assert np.array_equal(keys.cpu().numpy().view(np.uint32), ek)
    assert np.array_equal(vals.cpu().numpy().view(np.uint32), ev)
