"""Host-side tests of the C ABI (no GPU needed): the library loads, exports
every function include/dc.h declares, validates arguments, and its plan
(level table, schedule, scratch accounting) matches the closed forms of the
recurrence T(n) = aT(n/b) + f(n) and the paper's 2n
working space."""
import ctypes
import json
import math
import os
import re
import subprocess

import pytest

import paper_conf_ipps_lopez_ortizss13_b200 as dc

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_functions():
    names = []
    for fn in os.listdir(os.path.join(ROOT, "include")):
        if fn.endswith(".h"):
            text = open(os.path.join(ROOT, "include", fn)).read()
            text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
            names += re.findall(r"\b(dc_\w+)\s*\(", text)
    return sorted(set(names))


def test_library_exports_every_declared_symbol():
    lib = dc.lib()
    names = declared_functions()
    assert "dc_plan" in names and "dc_run_mergesort" in names and "dc_free" in names
    for name in names:
        assert hasattr(lib, name), name
    out = subprocess.run(["nm", "-D", "--defined-only", dc._build.LIB], capture_output=True,
                         text=True, check=True).stdout
    exported = set(re.findall(r" T (dc_\w+)", out))
    assert set(names) <= exported


def test_library_is_sm100a():
    out = subprocess.run(["cuobjdump", "--list-elf", dc._build.LIB], capture_output=True,
                         text=True, check=True).stdout
    assert "sm_100a" in out


def plan_raw(n, a=2, b=2, base=1):
    h = ctypes.c_void_p()
    st = dc.lib().dc_plan(n, a, b, base, ctypes.byref(h))
    return st, h


@pytest.mark.parametrize("args", [(0, 2, 2, 1), (-5, 2, 2, 1), (2**31, 2, 2, 1), (16, 1, 2, 1),
                                  (16, 2, 1, 1), (16, 2, 2, 0), (16, 2, 2, 17), (16, 2000, 2, 1)])
def test_plan_validation(args):
    st, h = plan_raw(*args)
    assert st == 1 and not h.value
    assert dc.lib().dc_last_error()


def test_free_accepts_null():
    assert dc.lib().dc_free(None) == 0


@pytest.mark.parametrize("k", [0, 1, 5, 20, 28, 30])
def test_level_table_closed_form_binary(k):
    n = 1 << k
    p = dc.Plan(n)
    lv = p.levels()
    assert len(lv) == k + 1                      # levels 0..log2 n
    for i, (nodes, size) in enumerate(lv):
        assert nodes == 2 ** i and size == n // 2 ** i
    # leaves: n^{log_b a} = n at level log_b n
    assert lv[-1] == (n, 1)


@pytest.mark.parametrize("n,a,b,base", [(1000, 2, 2, 1), (3**7, 3, 3, 1), (12345, 4, 4, 16),
                                        (10**6, 8, 2, 100), (7, 2, 2, 7)])
def test_level_table_general(n, a, b, base):
    lv = dc.Plan(n, a, b, base).levels()
    for i, (nodes, size) in enumerate(lv):
        assert nodes == a ** i
        assert size == -(-n // b ** i)
    assert lv[-1][1] <= base
    if len(lv) > 1:
        assert lv[-2][1] > base


def test_runs_need_binary_split():
    p = dc.Plan(1024, 4, 4, 1)
    h = p._h
    st = dc.lib().dc_run_mergesort(h, 0, ctypes.c_void_p(1 << 20), None)
    assert st == 2                               # UNSUPPORTED, before any device work


def test_run_validation_before_device_work():
    p = dc.Plan(1024)
    assert dc.lib().dc_run_mergesort(p._h, 0, None, None) == 1
    assert dc.lib().dc_run_mergesort(p._h, 0, ctypes.c_void_p(0x1004), None) == 1   # misaligned
    assert dc.lib().dc_run_mergesort(p._h, 7, ctypes.c_void_p(0x1000), None) == 1   # key type


@pytest.mark.parametrize("n", [1, 100, 8192, 8193, 1 << 20, 1 << 23, 1 << 28, (1 << 31) - 1])
@pytest.mark.parametrize("kt,vals", [("u32", False), ("i32", False), ("f32", False), ("u32", True)])
def test_schedule(n, kt, vals):
    """dc_plan_schedule reports the planner's choice (dc_model_sort_schedule),
    with the level counts of the recurrence: fused = ceil(log2 tile) levels on
    chip, P = ceil(log2 ceil(n / tile)) levels above, in P passes (one level
    each) or P mod 2 + P div 2 passes (two levels per pass)."""
    s = dc.Plan(n).schedule(kt, vals)
    m = dc.model_sort_schedule(n, kt, vals)
    t = s["tile"]
    assert t == m["tile"] and s["hbm_passes"] == m["hbm_passes"]
    assert s["fused_levels"] == math.ceil(math.log2(t)) == m["fused_levels"]
    assert s["global_passes"] == max(0, math.ceil(math.log2(math.ceil(n / t)))) == m["global_levels"]
    P = s["global_passes"]
    assert s["hbm_passes"] == (P % 2 + P // 2 if (m["two_level"] and P >= 2) else P)
    # least predicted time, or a full-tile schedule within 3 % of it (near-tie rule)
    assert m["predicted_ms"] <= 1.03 * min(v for v in m["candidates_ms"].values())
    # forced choices are honoured and reported
    for tc in (1, 2):
        for two in (False, True):
            p2 = dc.Plan(n)
            p2.set_tile_class(tc)
            p2.set_two_level(two)
            s2 = p2.schedule(kt, vals)
            m2 = dc.model_sort_schedule(n, kt, vals, tile_class=tc, two_level=int(two))
            assert (m2["tile_class"], m2["two_level"]) == (tc, two)
            assert s2["tile"] == m2["tile"] and s2["hbm_passes"] == m2["hbm_passes"]
            assert s2["hbm_passes"] == (s2["global_passes"] % 2 + s2["global_passes"] // 2
                                        if two and s2["global_passes"] >= 2
                                        else s2["global_passes"])
    # fused + global levels cover the whole tree: ceil(log2 n) combine levels
    if n > 1:
        assert s["fused_levels"] + s["global_passes"] >= math.ceil(math.log2(n))


@pytest.mark.parametrize("cs", [2, 4, 8, 16])
@pytest.mark.parametrize("n", [100, 25088 * 3 + 1, 1 << 20, 1 << 28])
def test_nk1_cluster_schedule(cs, n):
    """f2 cluster levels (dc_plan_set_nk1_cluster): keys-only u32/i32 sorts fuse
    cs tiles per run (log2 cs more levels on chip, as many fewer above); key-value
    and f32 sorts ignore the setting; the planner's rule leaves it off (cs = 1);
    any size other than 0/1/2/4/8/16 is rejected."""
    for kt in ("u32", "i32"):
        p0 = dc.Plan(n)
        base = p0.schedule(kt)
        assert p0.schedule(kt) == base
        p = dc.Plan(n)
        p.set_nk1_cluster(cs)
        s = p.schedule(kt)
        assert s["tile"] == base["tile"] * cs
        assert s["fused_levels"] == math.ceil(math.log2(s["tile"]))
        assert s["global_passes"] == max(0, math.ceil(math.log2(math.ceil(n / s["tile"]))))
        p.set_nk1_cluster(1)
        assert p.schedule(kt) == base
        p.set_nk1_cluster(0)
        assert p.schedule(kt) == base                 # the planner's rule: no cluster levels
    for kt, vals in (("u32", True), ("f32", False)):
        p = dc.Plan(n)
        ref = p.schedule(kt, vals)
        p.set_nk1_cluster(cs)
        assert p.schedule(kt, vals) == ref


@pytest.mark.parametrize("cs", [-1, 3, 5, 32])
def test_nk1_cluster_rejects_other_sizes(cs):
    p = dc.Plan(1 << 20)
    with pytest.raises(Exception):
        p.set_nk1_cluster(cs)
    assert dc.lib().dc_plan_set_nk1_cluster(p._h, cs) == 1   # DC_ERR_INVALID_ARG


def test_scratch_is_the_papers_2n_working_space():
    # "working space of 2n*sizeof(int)" -> input + one n-int temp
    golden = json.load(open(os.path.join(ROOT, "tests", "golden", "paper_numbers.json")))
    ws = golden["working_space"]
    n = ws["n"]
    p = dc.Plan(n)
    extra = p.scratch_bytes(False)
    assert n * 4 + n * 4 <= n * 4 + extra             # input + scratch >= 2n ints
    assert (n * 4 + extra) - ws["bytes"] < 0.01 * ws["bytes"]   # ... and not much more
    assert p.scratch_bytes(True) >= 2 * n * 4


# ------------------------------------------------ library communicator (host side)

def test_unique_id_is_128_bytes():
    a, b = dc.get_unique_id(), dc.get_unique_id()
    assert len(a) == 128 and len(b) == 128 and a != b


def test_comm_info_without_communicator():
    p = dc.Plan(12345)
    r, w, m = ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int64()
    assert dc.lib().dc_plan_comm_info(p._h, ctypes.byref(r), ctypes.byref(w), ctypes.byref(m)) == 0
    assert (r.value, w.value, m.value) == (0, 1, 12345)
    buf = (ctypes.c_int64 * 4)()
    assert dc.lib().dc_plan_last_splits(p._h, buf) == 1          # no multi-GPU sort yet


@pytest.mark.parametrize("rank,world,n", [(0, 0, 1000), (-1, 2, 1000), (2, 2, 1000),
                                          (0, 3, 1000)])
def test_set_comm_validates_before_joining(rank, world, n):
    """Invalid rank / world / divisibility is rejected before NCCL is touched
    (a valid call would block in ncclCommInitRank waiting for the peers)."""
    p = dc.Plan(n)
    uid = ctypes.create_string_buffer(dc.get_unique_id(), 128)
    assert dc.lib().dc_plan_set_comm(p._h, uid, rank, world) == 1
    assert dc.lib().dc_plan_set_comm(p._h, None, 0, 1) == 1


def test_set_comm_rejects_non_binary_plans():
    p = dc.Plan(1024, 4, 4, 1)
    uid = ctypes.create_string_buffer(dc.get_unique_id(), 128)
    assert dc.lib().dc_plan_set_comm(p._h, uid, 0, 2) == 2


def test_mg_stride_range():
    p = dc.Plan(1000)
    assert dc.lib().dc_plan_set_mg_stride(p._h, 0) == 1
    assert dc.lib().dc_plan_set_mg_stride(p._h, 1 << 21) == 1
    assert dc.lib().dc_plan_set_mg_stride(p._h, 1024) == 0
    assert dc.lib().dc_loopback_free(None) == 0


# ------------------------------------------------ binding argument checks

def test_sendbuf_words_keep_every_rank_aligned():
    """Back-to-back send buffers of all ranks stay 16-byte aligned for any
    stride (the int64 headers of rank r sit at r * words * 4 bytes)."""
    for world in (2, 3, 4, 8):
        for wcap in (1, 63, 333, 1000, 1001, 4096):
            w = dc.lib().dc_mg_sendbuf_words(world, wcap)
            assert w % 4 == 0
            assert w >= 6 * (world - 1) + (world - 1) * wcap
            assert w < 6 * (world - 1) + (world - 1) * wcap + 4
    assert dc.lib().dc_mg_sendbuf_words(1, 100) == 0


def _host(n, dtype=None):
    import torch
    return torch.zeros(n, dtype=dtype or torch.int32)


@pytest.mark.parametrize("call", [
    lambda p: p.sort_host_(_host(99)),
    lambda p: p.sort_host_(_host(100), _host(99)),
    lambda p: p.sort_host_(_host(100, __import__("torch").int64)),
    lambda p: p.sort_host_submit(_host(100), _host(99)),
    lambda p: p.sort_host_submit(_host(100), _host(100), _host(100), None),
    lambda p: p.max_subarray_host(_host(99)),
    lambda p: p.max_subarray_host(_host(200)[::2]),
])
def test_host_entry_points_check_sizes_before_the_c_call(call):
    """Host buffers the C side copies n*4 bytes into or out of are checked for
    length, element size and contiguity first (a short tensor used to
    overflow the host heap)."""
    p = dc.Plan(100)
    with pytest.raises(ValueError):
        call(p)


@pytest.mark.parametrize("call", [
    lambda p: p.max_subarray(_host(100)),
    lambda p: p.max_subarray_async(_host(100), _host(3, __import__("torch").int64)),
    lambda p: p.max_subarray_tuple_async(_host(100), _host(8, __import__("torch").int64)),
    lambda p: p.sum(_host(100)),
    lambda p: p.sum_async(_host(100), _host(1, __import__("torch").int64)),
    lambda p: p.sum_alg5(_host(100, __import__("torch").int64)),
    lambda p: p.sort_(_host(100)),
])
def test_device_entry_points_reject_host_tensors(call):
    p = dc.Plan(100)
    with pytest.raises(ValueError):
        call(p)
