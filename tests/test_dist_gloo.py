"""Multi-process (gloo, CPU) tests of the multi-GPU path's host side.

The distributed sort runs inside the library (csrc/mg_runtime.cu); its device
steps need a GPU (tests/test_gpu_native_mg.py runs them in a loopback group).
Here, with world sizes 2 and 3 and real torch.distributed collectives, every
rank drives the runtime's own host step -- dc_mg_exchange_sizes, the exchange
plan the runtime derives from the split matrix -- through the C ABI, performs
the exchange with a real gloo all-to-all, and the result is checked
(a) bit for bit on rank 0 against the CPU oracle's stable sort of the whole
input, and (b) collectively by dist.verify_global_sort, the check bench.py
runs after every multi-GPU timed loop (fingerprints all-reduced, slices
sorted, boundaries ordered), including that it FAILS on corrupted output.

The stand-ins for the GPU steps are plain definitions, not a second copy of
the protocol: the local levels are the oracle's stable sort of the shard, the
split matrix is read off the oracle's global stable order (c[r][d] = number
of rank-r elements among the first d*m outputs), and the local G-way merge is
the oracle's stable sort of the received runs in rank order.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _split_matrix_by_definition(shards_sorted, oracle):
    """c[r][d] = #rank-r elements among the first d*m of the global stable
    order of the concatenated (locally sorted) shards -- the definition the
    runtime's mg_split_matrix kernel computes exactly."""
    G = len(shards_sorted)
    m = shards_sorted[0].size
    cat = np.concatenate(shards_sorted)
    _, order = oracle.mergesort(cat, np.arange(cat.size, dtype=np.uint32))
    src = order.astype(np.int64) // m
    cm = np.zeros((G, G + 1), dtype=np.int64)
    for d in range(1, G + 1):
        cm[:, d] = np.bincount(src[:d * m], minlength=G)
    return cm


def _worker(rank, world, port, n, dist_name, corrupt, result_q):
    import sys

    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import dcgen
        import oracle
        import paper_conf_ipps_lopez_ortizss13_b200 as dc
        from paper_conf_ipps_lopez_ortizss13_b200 import dist as dcdist

        oracle.build()
        # the NCCL id travels as init_dist sends it (rank 0 creates, broadcast)
        uid = dc.broadcast_unique_id()
        ids = [None] * world
        dist.all_gather_object(ids, uid)
        assert len(uid) == 128 and all(i == uid for i in ids)

        m = n // world
        keys = dcgen.sort_keys(n, dist_name, seed=17, start=rank * m, count=m)
        vals = torch.arange(rank * m, (rank + 1) * m, dtype=torch.int32)
        in_fp = dcdist.fingerprint(keys)
        # levels >= log2 G: the shard's own stable sort
        sk, sv = oracle.mergesort(keys.numpy().view(np.uint32), vals.numpy().view(np.uint32))
        allsk = [torch.empty(m, dtype=torch.int32) for _ in range(world)]
        dist.all_gather(allsk, torch.from_numpy(sk.view(np.int32).copy()))
        cm = _split_matrix_by_definition([t.numpy().view(np.uint32) for t in allsk], oracle)
        # the runtime's host step, through the C ABI
        xs = dc.mg_exchange_sizes(cm.tolist(), rank, m)
        assert sum(xs["recv_cnt"]) == m and sum(xs["send_cnt"]) == m
        assert xs["send_off"] == cm[rank, :world].tolist()
        # a8: the exchange with a real all-to-all
        rk = torch.empty(m, dtype=torch.int32)
        rv = torch.empty(m, dtype=torch.int32)
        dist.all_to_all_single(rk, torch.from_numpy(sk.view(np.int32).copy()),
                               xs["recv_cnt"], xs["send_cnt"])
        dist.all_to_all_single(rv, torch.from_numpy(sv.view(np.int32).copy()),
                               xs["recv_cnt"], xs["send_cnt"])
        # runs land back to back in rank order at recv_off
        offs = np.cumsum([0] + xs["recv_cnt"][:-1]).tolist()
        assert offs == xs["recv_off"]
        # a9: stable merge of the runs (earlier rank wins ties)
        ok_, ov_ = oracle.mergesort(rk.numpy().view(np.uint32), rv.numpy().view(np.uint32))
        out_k = torch.from_numpy(ok_.view(np.int32).copy())
        out_v = torch.from_numpy(ov_.view(np.int32).copy())
        if corrupt == "value" and rank == world - 1:
            out_k[m // 2] = out_k[m // 2] ^ 1
        if corrupt == "swap" and rank == 0:
            out_k[-1] = -1                              # 0xFFFFFFFF at the end of rank 0
        check = dcdist.verify_global_sort(in_fp, out_k)
        gk = [torch.empty_like(out_k) for _ in range(world)]
        gv = [torch.empty_like(out_v) for _ in range(world)]
        dist.all_gather(gk, out_k)
        dist.all_gather(gv, out_v)
        if rank == 0:
            result_q.put((torch.cat(gk).numpy().copy(), torch.cat(gv).numpy().copy(), check,
                          cm.tolist()))
    finally:
        dist.destroy_process_group()


def _run(world, n, dist_name, corrupt=None):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    mp.start_processes(_worker, args=(world, _free_port(), n, dist_name, corrupt, q),
                       nprocs=world, join=True, start_method="spawn")
    return q.get(timeout=60)


@pytest.mark.parametrize("world", [2, 3])
@pytest.mark.parametrize("dist_name", ["uniform", "few", "equal", "reverse"])
def test_gloo_exchange_then_merge_is_the_global_stable_sort(oracle_mod, world, dist_name):
    import dcgen

    n = 3 * 4 * 601
    keys_out, vals_out, check, cm = _run(world, n, dist_name)
    full = dcgen.sort_keys(n, dist_name, seed=17).numpy().view(np.uint32)
    ek, ev = oracle_mod.mergesort(full, np.arange(n, dtype=np.uint32))
    assert np.array_equal(keys_out.view(np.uint32), ek)
    assert np.array_equal(vals_out.view(np.uint32), ev)          # stability across ranks
    assert check["ok"] and check["multiset_fingerprint_equal"]
    assert check["descents"] == 0 and check["rank_boundaries_ordered"]
    m = n // world
    assert all(sum(r[d] for r in cm) == d * m for d in range(world + 1))


@pytest.mark.parametrize("corrupt", ["value", "swap"])
def test_gloo_global_check_detects_corruption(oracle_mod, corrupt):
    _, _, check, _ = _run(2, 2 * 3001, "uniform", corrupt)
    assert not check["ok"]
    if corrupt == "value":
        assert not check["multiset_fingerprint_equal"]
    else:
        assert not check["rank_boundaries_ordered"] or check["descents"] > 0
        assert not check["multiset_fingerprint_equal"]


def test_exchange_sizes_reject_inconsistent_matrices():
    import paper_conf_ipps_lopez_ortizss13_b200 as dc

    good = [[0, 3, 5], [0, 2, 5]]
    xs = dc.mg_exchange_sizes(good, 1, 5)
    # rank 1 keeps [2, 5) of its shard, sends [0, 2) to rank 0, and receives
    # rank 0's [3, 5) then its own [2, 5): runs of 2 and 3 back to back
    assert xs == {"send_cnt": [2, 3], "send_off": [0, 2], "recv_cnt": [2, 3],
                  "recv_off": [0, 2]}
    for bad in ([[0, 6, 5], [0, 2, 5]],        # row not monotone
                [[1, 3, 5], [0, 2, 5]],        # row does not start at 0
                [[0, 3, 4], [0, 2, 5]],        # row does not end at shard_n
                [[0, 1, 5], [0, 1, 5]]):       # rank 1 would receive 8 != 5
        with pytest.raises(dc.DcError):
            dc.mg_exchange_sizes(bad, 1, 5)


def test_fingerprint_is_a_multiset_invariant():
    from paper_conf_ipps_lopez_ortizss13_b200 import dist as dcdist

    g = torch.Generator().manual_seed(3)
    k = torch.randint(-2**31, 2**31 - 1, (50_000,), generator=g, dtype=torch.int32)
    perm = k[torch.randperm(k.numel(), generator=g)]
    assert torch.equal(dcdist.fingerprint(k), dcdist.fingerprint(perm))
    k2 = k.clone()
    k2[7] ^= 1 << 20
    assert not torch.equal(dcdist.fingerprint(k), dcdist.fingerprint(k2))
    k3 = k.clone()
    k3[1], k3[2] = k[2] + 1, k[1] - 1                # same key sum, different multiset
    assert not torch.equal(dcdist.fingerprint(k), dcdist.fingerprint(k3))
    assert dcdist.locally_sorted(torch.sort(k.to(torch.int64) & 0xFFFFFFFF).values
                                 .to(torch.int32)) == 0
