"""The library-owned multi-GPU runtime (dc_plan_set_comm / dc_plan_set_loopback,
rows a7-a10 + b) on one GPU.

A loopback group runs G ranks as threads of this process, each with its own
plan and CUDA stream; the collectives are device copies between their buffers,
the protocol and kernels are the ones NCCL runs use.  The rank outputs,
concatenated in rank order, must equal the CPU oracle's stable sort /
max-subarray of the whole input, bit for bit.  NCCL itself is exercised at
world 1 (one GPU per gpurun box).
"""
import threading

import numpy as np
import pytest
import torch

import dcgen

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def dc():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_ipps_lopez_ortizss13_b200 as m
    return m


def run_ranks(dc, n, world, fn, stride=None, p2p=True):
    """fn(plan, rank, m) on `world` threads joined to one loopback group."""
    group = dc.LoopbackGroup(world)
    plans = []
    for r in range(world):
        p = dc.Plan(n)
        p.set_mg_p2p(p2p)
        if stride:
            p.set_mg_stride(stride)
        p.set_loopback(group, r)
        plans.append(p)
    results, errors = [None] * world, [None] * world

    def body(r):
        try:
            s = torch.cuda.Stream()
            with torch.cuda.stream(s):
                results[r] = fn(plans[r], r, plans[r].n)
                s.synchronize()
        except BaseException as e:   # noqa: BLE001 - surfaced by the caller
            errors[r] = e.with_traceback(None)   # no frame cycle keeping plans alive

    threads = [threading.Thread(target=body, args=(r,)) for r in range(world)]
    for t in threads:
        t.start()
    for t in threads:
        t.join(timeout=300)
    return results, errors, plans


def _view(a, key_type):
    return a.view({"u32": np.uint32, "i32": np.int32, "f32": np.float32}[key_type])


def sort_case(dc, oracle_mod, n, world, dist_name, key_type, with_vals, stride=None, seed=31,
              p2p=True, reps=1):
    def fn(plan, r, m):
        src = dcgen.sort_keys(n, dist_name, seed=seed, key_type=key_type, start=r * m, count=m,
                              device="cuda")
        keys = torch.empty_like(src)
        vals = torch.empty(m, dtype=torch.int32, device="cuda") if with_vals else None
        for _ in range(reps):              # repeated sorts reuse the shared shard buffers
            keys.copy_(src)
            if with_vals:
                vals.copy_(dcgen.sort_vals(n, start=r * m, count=m, device="cuda"))
            plan.sort_(keys, vals, key_type=key_type)
        return (keys.cpu(), (vals.cpu() if with_vals else None), plan.last_splits(),
                plan.exchange_mode())

    res, errs, plans = run_ranks(dc, n, world, fn, stride, p2p)
    for e in errs:
        if e is not None:
            raise e
    full = dcgen.sort_keys(n, dist_name, seed=seed, key_type=key_type).numpy()
    ek, ev = oracle_mod.mergesort(_view(full, key_type), np.arange(n, dtype=np.uint32),
                                  key_type=key_type)
    got = torch.cat([r[0] for r in res]).numpy()
    assert np.array_equal(got.view(np.uint32), ek.view(np.uint32))
    if with_vals:
        assert np.array_equal(torch.cat([r[1] for r in res]).numpy().view(np.uint32), ev)
    # every rank computed the same split matrix; its columns partition [0, n)
    cm = np.array(res[0][2])
    for r in res[1:]:
        assert np.array_equal(np.array(r[2]), cm)
    m = n // world
    assert np.array_equal(cm.sum(axis=0), np.arange(world + 1) * m)
    assert np.all(np.diff(cm, axis=1) >= 0)
    assert all(r[3] == ("fused" if p2p else "all_to_all") for r in res)
    return cm


@pytest.mark.parametrize("p2p", [True, False], ids=["fused", "alltoall"])
@pytest.mark.parametrize("world", [2, 3, 4, 8])
@pytest.mark.parametrize("dist_name", ["uniform", "few", "sorted", "reverse", "equal"])
def test_loopback_kv(dc, oracle_mod, world, dist_name, p2p):
    sort_case(dc, oracle_mod, world * 100_003, world, dist_name, "u32", True, p2p=p2p)


@pytest.mark.parametrize("p2p", [True, False], ids=["fused", "alltoall"])
@pytest.mark.parametrize("world", [2, 5])
def test_loopback_repeated_sorts(dc, oracle_mod, world, p2p):
    """Three sorts back to back per rank (graph replay of the local levels,
    the shard buffers rewritten while peers have just read them)."""
    sort_case(dc, oracle_mod, world * 200_001, world, "paper", "u32", True, p2p=p2p, reps=3)


@pytest.mark.parametrize("key_type", ["u32", "i32", "f32"])
@pytest.mark.parametrize("stride", [64, 1000, 4096])
def test_loopback_keys_only(dc, oracle_mod, key_type, stride):
    sort_case(dc, oracle_mod, 4 * 250_001, 4, "paper", key_type, False, stride)


@pytest.mark.parametrize("world", [2, 4, 8])
@pytest.mark.parametrize("stride", [1001, 333])
def test_loopback_odd_stride(dc, oracle_mod, world, stride):
    """odd sample strides with an even world size: every rank's
    send buffer (int64 headers) must stay aligned in the all-gathered array."""
    sort_case(dc, oracle_mod, world * 120_007, world, "uniform", "u32", True, stride)


@pytest.mark.parametrize("p2p", [True, False], ids=["fused", "alltoall"])
@pytest.mark.parametrize("world", [4, 8])
def test_loopback_many_ranks_large(dc, oracle_mod, p2p, world):
    """2^24 keys over 4 / 8 ranks: the G-way merge is one 4-way pass (G = 4)
    or a 4-way pass per group of four plus a pair pass (G = 8); in fused mode
    the 4-way pass reads four peers' shards directly."""
    sort_case(dc, oracle_mod, 1 << 24, world, "uniform", "u32", False, 4096, p2p=p2p)


@pytest.mark.parametrize("p2p", [True, False], ids=["fused", "alltoall"])
def test_loopback_large_shards(dc, oracle_mod, p2p):
    """2^25 keys over 2 ranks: 16M-key shards use the full-size tile config."""
    sort_case(dc, oracle_mod, 1 << 25, 2, "uniform", "u32", False, p2p=p2p)


def test_loopback_equal_keys_split_exactly(dc, oracle_mod):
    """All keys equal: the stable order is (rank, position), so rank r keeps its
    own shard and nothing moves."""
    world = 4
    cm = sort_case(dc, oracle_mod, world * 70_001, world, "equal", "u32", True)
    m = 70_001
    for r in range(world):
        assert cm[r][r + 1] - cm[r][r] == m


@pytest.mark.parametrize("world", [1, 2, 3, 8])
@pytest.mark.parametrize("kind", ["uniform", "negative", "small"])
def test_loopback_maxsub(dc, oracle_mod, world, kind):
    n = world * 300_007

    def fn(plan, r, m):
        x = dcgen.maxsub_input(n, kind, seed=5, start=r * m, count=m, device="cuda")
        return plan.max_subarray(x)

    res, errs, _ = run_ranks(dc, n, world, fn)
    for e in errs:
        if e is not None:
            raise e
    full = dcgen.maxsub_input(n, kind, seed=5).numpy()
    expect = tuple(int(v) for v in oracle_mod.maxsub(full))
    for r in res:
        assert tuple(r) == expect


def test_loopback_failing_member_releases_others(dc):
    """A rank whose call fails validation aborts the group: the other rank gets
    DC_ERR_NCCL promptly instead of waiting in a barrier."""
    n = 2 * 50_000
    lib = dc.lib()

    def fn(plan, r, m):
        keys = dcgen.sort_keys(n, "uniform", seed=1, start=r * m, count=m, device="cuda")
        if r == 1:
            st = lib.dc_run_mergesort(plan._h, 7, keys.data_ptr(), None)   # bad key type
            assert st == 1
            return "failed"
        plan.sort_(keys)
        return "sorted"

    import time
    t0 = time.time()
    res, errs, _ = run_ranks(dc, n, 2, fn)
    assert time.time() - t0 < 60
    assert res[1] == "failed"
    assert isinstance(errs[0], dc.DcError) and errs[0].status == 5


def test_comm_validation(dc):
    g = dc.LoopbackGroup(2)
    p = dc.Plan(1001)
    with pytest.raises(dc.DcError):              # n % world != 0
        p.set_loopback(g, 0)
    p = dc.Plan(1000)
    with pytest.raises(dc.DcError):
        p.set_loopback(g, 2)                     # rank out of range
    p.set_loopback(g, 0)
    assert (p.rank, p.world, p.n, p.n_global) == (0, 2, 500, 1000)
    q = dc.Plan(1000)
    with pytest.raises(dc.DcError):              # rank already joined
        q.set_loopback(g, 0)
    with pytest.raises(dc.DcError):              # second communicator
        p.set_loopback(g, 1)
    r = dc.Plan(1024)
    r.sort_(dcgen.sort_keys(1024, "uniform", seed=1, device="cuda"))
    with pytest.raises(dc.DcError):              # after the first run
        r.set_loopback(g, 1)
    with pytest.raises(dc.DcError):              # host-buffer paths are single-GPU
        p.sort_host_(torch.zeros(500, dtype=torch.int32).pin_memory())


def test_nccl_world1_sort_and_maxsub(dc, oracle_mod):
    """NCCL communicator of one rank: dlopen, unique id, init, collectives."""
    n = 3 * 8192 + 101
    p = dc.Plan(n)
    p.set_comm(dc.get_unique_id(), 0, 1)
    assert (p.rank, p.world, p.n) == (0, 1, n)
    keys = dcgen.sort_keys(n, "few", seed=4, device="cuda")
    vals = dcgen.sort_vals(n, device="cuda")
    k_in = keys.cpu().numpy().view(np.uint32)
    p.sort_(keys, vals)
    ek, ev = oracle_mod.mergesort(k_in, np.arange(n, dtype=np.uint32))
    assert np.array_equal(keys.cpu().numpy().view(np.uint32), ek)
    assert np.array_equal(vals.cpu().numpy().view(np.uint32), ev)
    x = dcgen.maxsub_input(n, "uniform", seed=8, device="cuda")
    assert p.max_subarray(x) == tuple(int(v) for v in oracle_mod.maxsub(x.cpu().numpy()))


@pytest.mark.parametrize("key_type", ["u32", "i32", "f32"])
@pytest.mark.parametrize("runs", [1, 2, 3, 4, 5, 7, 8, 16, 17])
@pytest.mark.parametrize("with_vals", [True, False])
def test_merge_peers_separate_buffers(dc, oracle_mod, key_type, runs, with_vals):
    """dc_mg_merge_peers on runs that each live in their own buffer at an
    arbitrary offset (unaligned starts, ragged lengths, empty runs): groups of
    four runs in one 4-way pass read straight from their buffers (outputs at
    unaligned offsets when G > 4), pairs in one pair-mode pass, lone runs
    copied; keys only (pad-safe 4-way merges for u32/i32) and with values."""
    rng = np.random.default_rng(runs)
    lens = [int(rng.integers(0, 40_000 if runs < 8 else 90_000)) for _ in range(runs)]
    if runs > 2:
        lens[1] = 0
    total = sum(lens)
    plan = dc.Plan(max(total, 1))
    bufs, vbufs, offs, allk, allv, pos = [], [], [], [], [], 0
    view = {"u32": np.uint32, "i32": np.int32, "f32": np.float32}[key_type]
    for r, ln in enumerate(lens):
        off = int(rng.integers(0, 37))
        k = dcgen.sort_keys(off + ln + 11, "few", seed=r, key_type=key_type)
        seg = k[off:off + ln].numpy().view(view)
        srt = np.sort(seg, kind="stable")
        k[off:off + ln] = torch.from_numpy(srt.copy().view(np.int32)
                                           if key_type != "f32" else srt.copy())
        v = torch.arange(pos - off, pos - off + k.numel(), dtype=torch.int32)
        bufs.append(k.cuda())
        vbufs.append(v.cuda())
        offs.append(off)
        allk.append(k[off:off + ln].numpy().view(view))
        allv.append(v[off:off + ln].numpy().view(np.uint32))
        pos += ln
    out_k = torch.empty(max(total, 1), dtype=bufs[0].dtype, device="cuda")
    out_v = torch.empty(max(total, 1), dtype=torch.int32, device="cuda")
    tk = torch.empty_like(out_k)
    tv = torch.empty_like(out_v)
    if not with_vals:
        out_v = tv = None
    plan.mg_merge_peers([(bufs[r], vbufs[r] if with_vals else None, offs[r], lens[r])
                         for r in range(runs)], out_k, out_v, tk, tv, key_type=key_type)
    cat_k = np.concatenate(allk)
    cat_v = np.concatenate(allv)
    ek, ev = oracle_mod.mergesort(cat_k, cat_v, key_type=key_type)   # stable: earlier run wins
    got = out_k[:total].cpu().numpy().view(view)
    assert np.array_equal(got.view(np.uint32), ek.view(np.uint32))
    if with_vals:
        assert np.array_equal(out_v[:total].cpu().numpy().view(np.uint32), ev)


@pytest.mark.parametrize("p2p", [True, False], ids=["fused", "alltoall"])
def test_loopback_phase_times(dc, p2p):
    """Phase accounting with timing on: one entry per sort, keys received from
    peers = shard size minus the rank's own part of its output slice."""
    world, n = 3, 3 * 150_001

    def fn(plan, r, m):
        plan.enable_timing(True)
        keys = dcgen.sort_keys(n, "uniform", seed=3, start=r * m, count=m, device="cuda")
        plan.sort_(keys, key_type="u32")
        ph = plan.mg_phase_times()
        cm = plan.last_splits()
        plan.enable_timing(False)
        return ph, cm

    res, errs, _ = run_ranks(dc, n, world, fn, p2p=p2p)
    for e in errs:
        if e is not None:
            raise e
    m = n // world
    for r, (ph, cm) in enumerate(res):
        assert ph["sorts"] == 1
        assert ph["keys_received"] == m - (cm[r][r + 1] - cm[r][r])
        assert ph["local_sort"] > 0 and ph["splitters"] > 0 and ph["exchange_merge"] > 0


@pytest.mark.parametrize("runs", [[5], [3, 0, 7], [1000, 1, 2, 50_000, 7, 0, 13], [40_000] * 4,
                                  [40_000] * 8, [60_001, 3, 77_777, 50_000, 0, 9, 25_344, 1],
                                  [20_000] * 16, [9_999] * 17])
@pytest.mark.parametrize("key_type,with_vals", [("u32", True), ("u32", False), ("i32", False),
                                                ("f32", True)])
def test_merge_runs_kernel(dc, oracle_mod, runs, key_type, with_vals):
    """dc_mg_merge_runs (a9): back-to-back sorted runs -> their stable merge
    (earlier runs win ties) in ceil(log4 G) passes, bit for bit against the
    oracle's stable sort of the concatenation."""
    total = sum(runs)
    view = {"u32": np.uint32, "i32": np.int32, "f32": np.float32}[key_type]
    parts, off = [], 0
    for r in runs:
        k = dcgen.sort_keys(total, "few", seed=31, key_type=key_type, start=off,
                            count=r).numpy().view(view)
        parts.append(np.sort(k, kind="stable"))
        off += r
    keys_in = np.concatenate(parts)
    vals_in = np.arange(total, dtype=np.uint32)
    ik = torch.from_numpy(keys_in.view(np.int32).copy()).cuda()
    iv = torch.from_numpy(vals_in.view(np.int32).copy()).cuda() if with_vals else None
    ok = torch.empty_like(ik)
    ov = torch.empty_like(iv) if with_vals else None
    dc.Plan(total).mg_merge_runs(ik, iv, ok, ov, runs, key_type=key_type)
    ek, ev = oracle_mod.mergesort(keys_in, vals_in, key_type=key_type)
    assert np.array_equal(ok.cpu().numpy().view(np.uint32), ek.view(np.uint32))
    if with_vals:
        assert np.array_equal(ov.cpu().numpy().view(np.uint32), ev)
