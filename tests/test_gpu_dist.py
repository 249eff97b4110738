"""The multi-GPU protocol (rows a7-a10) on one GPU: G virtual ranks as threads
(LoopbackComm), every device step in the library's kernels.  The concatenated
rank outputs must equal the CPU oracle's stable sort / max-subarray of the
whole input, bit for bit.  (Real NCCL runs need gpurun --gpus N; see bench.py.)
"""
import numpy as np
import pytest
import torch

import dcgen

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def dist():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ipps_lopez_ortizss13_b200 import dist as d
    return d


def _run_sort(dist, n, world, dist_name, key_type, with_vals, stride):
    m = n // world

    def rank_fn(comm):
        r = comm.rank
        keys = dcgen.sort_keys(n, dist_name, seed=29, key_type=key_type, start=r * m, count=m,
                               device="cuda")
        vals = dcgen.sort_vals(n, start=r * m, count=m, device="cuda") if with_vals else None
        info = dist.sort_(keys, vals, comm, key_type=key_type, stride=stride)
        return keys.cpu(), (vals.cpu() if with_vals else None), info

    return dist.run_loopback(world, rank_fn)


@pytest.mark.parametrize("world", [2, 3, 4, 8])
@pytest.mark.parametrize("dist_name", ["uniform", "few", "sorted", "reverse", "equal"])
def test_loopback_sort_u32_kv(dist, oracle_mod, world, dist_name):
    n = world * 100_003
    res = _run_sort(dist, n, world, dist_name, "u32", True, 4096)
    keys = torch.cat([r[0] for r in res]).numpy().view(np.uint32)
    vals = torch.cat([r[1] for r in res]).numpy().view(np.uint32)
    full = dcgen.sort_keys(n, dist_name, seed=29).numpy().view(np.uint32)
    ek, ev = oracle_mod.mergesort(full, np.arange(n, dtype=np.uint32))
    assert np.array_equal(keys, ek)
    assert np.array_equal(vals, ev)


@pytest.mark.parametrize("key_type", ["u32", "i32", "f32"])
@pytest.mark.parametrize("stride", [64, 1000, 4096])
def test_loopback_sort_keys_only(dist, oracle_mod, key_type, stride):
    world, n = 4, 4 * 250_001
    res = _run_sort(dist, n, world, "uniform", key_type, False, stride)
    got = torch.cat([r[0] for r in res]).numpy().view(np.uint32)
    full = dcgen.sort_keys(n, "uniform", seed=29, key_type=key_type).numpy()
    view = {"u32": np.uint32, "i32": np.int32, "f32": np.float32}[key_type]
    ek = oracle_mod.mergesort(full.view(view), key_type=key_type)
    assert np.array_equal(got, ek.view(np.uint32))


def test_loopback_sort_large(dist, oracle_mod):
    world, n = 8, 1 << 24
    res = _run_sort(dist, n, world, "uniform", "u32", False, 4096)
    got = torch.cat([r[0] for r in res]).numpy().view(np.uint32)
    full = dcgen.sort_keys(n, "uniform", seed=29).numpy().view(np.uint32)
    assert np.array_equal(got, oracle_mod.mergesort(full))
    cm = np.array(res[0][2].cmat)
    m = n // world
    assert all(cm[:, d].sum() == d * m for d in range(world + 1))


@pytest.mark.parametrize("runs", [[5], [3, 0, 7], [1000, 1, 2, 50_000, 7, 0, 13],
                                  [40_000] * 8])
def test_merge_runs_kernel(dist, oracle_mod, runs):
    from paper_conf_ipps_lopez_ortizss13_b200 import Plan

    total = sum(runs)
    parts, off = [], 0
    for r in runs:
        k = dcgen.sort_keys(total, "few", seed=31, start=off, count=r).numpy().view(np.uint32)
        parts.append(np.sort(k, kind="stable"))
        off += r
    keys_in = np.concatenate(parts)
    vals_in = np.arange(total, dtype=np.uint32)
    ik = torch.from_numpy(keys_in.view(np.int32).copy()).cuda()
    iv = torch.from_numpy(vals_in.view(np.int32).copy()).cuda()
    ok, ov = torch.empty_like(ik), torch.empty_like(iv)
    Plan(total).mg_merge_runs(ik, iv, ok, ov, runs, key_type="u32")
    ek, ev = oracle_mod.mergesort(keys_in, vals_in)     # stable: earlier runs win ties
    assert np.array_equal(ok.cpu().numpy().view(np.uint32), ek)
    assert np.array_equal(ov.cpu().numpy().view(np.uint32), ev)


@pytest.mark.parametrize("sizes", [[1 << 20, 1 << 20], [100_000, 3, 777_777, 50_000]])
@pytest.mark.parametrize("dist_name", ["uniform", "small", "negative"])
def test_loopback_maxsub(dist, oracle_mod, sizes, dist_name):
    n = sum(sizes)

    def rank_fn(comm):
        start = sum(sizes[:comm.rank])
        x = dcgen.maxsub_input(n, dist_name, seed=37, start=start, count=sizes[comm.rank],
                               device="cuda")
        return dist.max_subarray(x, comm)

    res = dist.run_loopback(len(sizes), rank_fn)
    expect = oracle_mod.maxsub(dcgen.maxsub_input(n, dist_name, seed=37).numpy())
    assert all(r == expect for r in res)
