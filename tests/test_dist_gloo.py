"""Multi-process (gloo, CPU) tests of the multi-GPU protocol's host logic.

World sizes 2 and 3, real torch.distributed collectives (all-gather,
all-reduce, all-to-all), the per-rank device steps replaced by the numpy test
double in tests/mg_numpy_ops.py.  Rank 0 gathers every rank's output slice and
compares the concatenation with the CPU oracle (Alg 6 stable mergesort /
recursive max-subarray) on the whole input, bit for bit.
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


def _sort_worker(rank, world, port, n, dist_name, key_type, with_vals, stride, result_q):
    import sys

    sys.path.insert(0, ROOT)
    sys.path.insert(0, os.path.join(ROOT, "tests"))
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import dcgen
        from mg_numpy_ops import NumpyOps
        from paper_conf_ipps_lopez_ortizss13_b200 import dist as dcdist

        m = n // world
        keys = dcgen.sort_keys(n, dist_name, seed=17, key_type=key_type, start=rank * m, count=m)
        vals = dcgen.sort_vals(n, start=rank * m, count=m) if with_vals else None
        info = dcdist.sort_(keys, vals, dcdist.TorchComm(), key_type=key_type, stride=stride,
                            ops=NumpyOps(key_type))
        assert sum(info.recv_splits) == m
        gk = [torch.empty_like(keys) for _ in range(world)]
        dist.all_gather(gk, keys)
        gv = None
        if with_vals:
            gv = [torch.empty_like(vals) for _ in range(world)]
            dist.all_gather(gv, vals)
        if rank == 0:
            result_q.put((torch.cat(gk).numpy().copy(),
                          None if gv is None else torch.cat(gv).numpy().copy(), info.cmat))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
@pytest.mark.parametrize("dist_name,key_type,with_vals", [
    ("uniform", "u32", True), ("few", "u32", True), ("equal", "u32", True),
    ("reverse", "i32", False), ("uniform", "f32", True)])
def test_gloo_distributed_sort(oracle_mod, world, dist_name, key_type, with_vals):
    import dcgen

    n = 3 * 4 * 601                       # divisible by 2 and 3; m not a multiple of stride
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    mp.start_processes(_sort_worker, args=(world, _free_port(), n, dist_name, key_type,
                                           with_vals, 64, q), nprocs=world, join=True,
                       start_method="spawn")
    keys_out, vals_out, cmat = q.get(timeout=60)
    full = dcgen.sort_keys(n, dist_name, seed=17, key_type=key_type).numpy()
    view = {"u32": np.uint32, "i32": np.int32, "f32": np.float32}[key_type]
    ek, ev = oracle_mod.mergesort(full.view(view), np.arange(n, dtype=np.uint32),
                                  key_type=key_type)
    assert np.array_equal(keys_out.view(np.uint32), ek.view(np.uint32))
    if with_vals:
        assert np.array_equal(vals_out.view(np.uint32), ev)
    # split matrix: every column of boundaries sums to d*m, rows are monotone
    m = n // world
    cm = np.array(cmat)
    assert all(cm[:, d].sum() == d * m for d in range(world + 1))
    assert np.all(np.diff(cm, axis=1) >= 0)


def _maxsub_worker(rank, world, port, sizes, result_q):
    import sys

    sys.path.insert(0, ROOT)
    sys.path.insert(0, os.path.join(ROOT, "tests"))
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import dcgen
        from mg_numpy_ops import NumpyOps
        from paper_conf_ipps_lopez_ortizss13_b200 import dist as dcdist

        n = sum(sizes)
        start = sum(sizes[:rank])
        x = dcgen.maxsub_input(n, "small", seed=23, start=start, count=sizes[rank])
        res = dcdist.max_subarray(x, dcdist.TorchComm(), ops=NumpyOps())
        allres = [None] * world
        dist.all_gather_object(allres, res)
        if rank == 0:
            result_q.put(allres)
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("sizes", [[150, 150], [100, 37, 211]])
def test_gloo_distributed_maxsub(oracle_mod, sizes):
    import dcgen

    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    mp.start_processes(_maxsub_worker, args=(len(sizes), _free_port(), sizes, q),
                       nprocs=len(sizes), join=True, start_method="spawn")
    allres = q.get(timeout=60)
    n = sum(sizes)
    expect = oracle_mod.maxsub(dcgen.maxsub_input(n, "small", seed=23).numpy())
    assert all(tuple(r) == expect for r in allres)


def test_split_sizes_host_logic():
    from paper_conf_ipps_lopez_ortizss13_b200.dist import split_sizes

    cm = [[0, 2, 5, 6], [0, 1, 2, 6], [0, 3, 5, 6]]   # 3 ranks x (3+1), m = 6
    assert split_sizes(cm, 0) == ([2, 3, 1], [2, 1, 3])
    assert split_sizes(cm, 2) == ([3, 2, 1], [1, 4, 1])
    for r in range(3):
        s, rcv = split_sizes(cm, r)
        assert sum(s) == 6 and sum(rcv) == 6
