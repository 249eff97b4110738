"""Multi-GPU path: the top log2(G) levels of the breadth-first sort (rows a7-a10).

One process per GPU (torchrun); rank r holds the shard of global positions
[r*m, (r+1)*m).  Levels below log2(G) are independent subproblems: each rank
sorts its shard with the single-GPU path (NK1 + NK2/NK3 levels).  The top
log2(G) levels become one exchange step:

  a7  exact splitters: samples -> all-gather -> composite counts (kernel) ->
      all-reduce -> brackets + windows (kernels) -> all-gather -> split matrix
      (kernel); composite order (key, rank, position) = the global stable order;
  a8  all-to-all of the key (and value) ranges over NVLink (NCCL);
  a9  local stable G-way merge of the received runs (kernels);
  a10 max-subarray: per-rank summary tuple -> all-gather -> ordered combine.

The product path for N GPUs is the library-owned runtime (``init_dist`` /
dc_plan_set_comm: the same steps in C++ over NCCL); this module composes the
per-rank steps over any torch.distributed group, which is how the protocol's
host logic is tested on CPU with gloo.  Collectives go through a tiny
interface (:class:`Comm`): :class:`TorchComm`
wraps a torch.distributed process group (NCCL on GPUs; gloo in the CPU tests)
and :class:`LoopbackComm` runs G virtual ranks as threads in one process on
one GPU (the 1-GPU test of the whole protocol).  Every step on the data runs
in the library's kernels; this module only moves tensors between them.
"""
from __future__ import annotations

import threading
from dataclasses import dataclass

import torch

from . import Plan, _KEY_NAMES

DEFAULT_STRIDE = 4096     # sample stride S: candidates = G*ceil(m/S); windows < S keys


# ------------------------------------------------------------------- comms

class Comm:
    """Collectives used by the protocol (all ranks call them in the same order)."""

    rank: int
    world: int

    def all_gather(self, t: torch.Tensor) -> torch.Tensor:  # [world * t.numel()], rank order
        raise NotImplementedError

    def all_reduce_sum_(self, t: torch.Tensor) -> None:
        raise NotImplementedError

    def all_to_all(self, send: torch.Tensor, send_splits: list[int],
                   recv_splits: list[int]) -> torch.Tensor:
        raise NotImplementedError

    def barrier(self) -> None:
        raise NotImplementedError


class TorchComm(Comm):
    """torch.distributed process group (NCCL over NVLink on B200 boxes)."""

    def __init__(self, group=None):
        import torch.distributed as dist

        self.dist = dist
        self.group = group
        self.rank = dist.get_rank(group)
        self.world = dist.get_world_size(group)

    def all_gather(self, t):
        t = t.contiguous()
        out = torch.empty(self.world * t.numel(), dtype=t.dtype, device=t.device)
        self.dist.all_gather_into_tensor(out, t.view(-1), group=self.group)
        return out

    def all_reduce_sum_(self, t):
        self.dist.all_reduce(t, op=self.dist.ReduceOp.SUM, group=self.group)

    def all_to_all(self, send, send_splits, recv_splits):
        out = torch.empty(sum(recv_splits), dtype=send.dtype, device=send.device)
        self.dist.all_to_all_single(out, send, recv_splits, send_splits, group=self.group)
        return out

    def barrier(self):
        self.dist.barrier(group=self.group)


class _LoopbackState:
    def __init__(self, world):
        self.world = world
        self.barrier = threading.Barrier(world)
        self.slots = [None] * world


class LoopbackComm(Comm):
    """G virtual ranks as threads of one process sharing one GPU (testing)."""

    def __init__(self, state: _LoopbackState, rank: int):
        self.s = state
        self.rank = rank
        self.world = state.world

    def _exchange(self, obj, consume):
        """Publish obj, then consume(everyone's objs) while all ranks still hold
        their inputs unchanged (between the two barriers)."""
        cuda = torch.cuda.is_available()
        if cuda:
            torch.cuda.synchronize()
        self.s.slots[self.rank] = obj
        self.s.barrier.wait()
        out = consume(list(self.s.slots))
        if cuda:
            torch.cuda.synchronize()
        self.s.barrier.wait()
        return out

    def all_gather(self, t):
        return self._exchange(t.contiguous(),
                              lambda xs: torch.cat([x.reshape(-1) for x in xs]))

    def all_reduce_sum_(self, t):
        def add(xs):
            acc = xs[0].clone()
            for x in xs[1:]:
                acc += x
            return acc

        t.copy_(self._exchange(t, add))

    def all_to_all(self, send, send_splits, recv_splits):
        pieces = list(torch.split(send, send_splits))
        out = self._exchange(pieces, lambda ps: torch.cat([ps[r][self.rank]
                                                           for r in range(self.world)]))
        assert out.numel() == sum(recv_splits)
        return out

    def barrier(self):
        self._exchange(None, lambda xs: None)


def run_loopback(world: int, fn):
    """Run fn(comm) for `world` virtual ranks (threads); returns the results."""
    state = _LoopbackState(world)
    results, errors = [None] * world, []

    def body(r):
        try:
            results[r] = fn(LoopbackComm(state, r))
        except BaseException as e:   # noqa: BLE001 - surfaced below
            errors.append(e)
            state.barrier.abort()

    threads = [threading.Thread(target=body, args=(r,)) for r in range(world)]
    for t in threads:
        t.start()
    for t in threads:
        t.join()
    if errors:
        raise errors[0]
    return results


# -------------------------------------------------------------- local ops

class DcOps:
    """Per-rank device steps of the protocol, all in libdcb200 kernels."""

    def __init__(self, n: int):
        self.plan = Plan(n)

    def sort_(self, keys, vals, key_type):
        self.plan.sort_(keys, vals, key_type=key_type)

    def sample(self, keys, stride):
        return self.plan.mg_sample(keys, stride)

    def count(self, keys, rank, cand, per_rank, stride, key_type):
        return self.plan.mg_count(keys, rank, cand, per_rank, stride, key_type=key_type)

    def windows(self, keys, rank, world, counts, ranks, per_rank, wcap):
        return self.plan.mg_windows(keys, rank, world, counts, ranks, per_rank, wcap)

    def split_matrix(self, gathered, world, shard_n, wcap, key_type):
        return self.plan.mg_split_matrix(gathered, world, shard_n, wcap, key_type)

    def check(self):
        if self.plan.mg_error():
            raise RuntimeError("splitter window overflow (unsorted shard?)")

    def merge_runs(self, in_k, in_v, out_k, out_v, runs, key_type):
        self.plan.mg_merge_runs(in_k, in_v, out_k, out_v, runs, key_type=key_type)

    def maxsub_tuple(self, x, offset):
        out = torch.empty(8, dtype=torch.int64, device=x.device)
        return self.plan.max_subarray_tuple_async(x, out, index_offset=offset)

    def maxsub_combine(self, tuples):
        out = torch.empty(3, dtype=torch.int64, device=tuples.device)
        return self.plan.maxsub_combine_async(tuples, out)

    def launches(self) -> int:
        return self.plan.launch_count()


# ---------------------------------------------------------------- protocol

@dataclass
class ExchangeInfo:
    cmat: list            # world x (world+1): c[r][d]
    send_splits: list
    recv_splits: list


def split_sizes(cmat, rank: int):
    """Send / receive counts of `rank` from the split matrix c[r][d] (host logic):
    rank r sends [c[r][d], c[r][d+1]) to rank d and receives [c[s][r], c[s][r+1])
    from every rank s."""
    world = len(cmat)
    send = [int(cmat[rank][d + 1] - cmat[rank][d]) for d in range(world)]
    recv = [int(cmat[s][rank + 1] - cmat[s][rank]) for s in range(world)]
    return send, recv


def sort_(keys: torch.Tensor, vals: torch.Tensor | None = None, comm: Comm | None = None,
          key_type: str = "u32", stride: int = DEFAULT_STRIDE, ops=None) -> ExchangeInfo | None:
    """Distributed stable sort, in place.

    On entry rank r's ``keys`` (and ``vals``) hold global positions
    [r*m, (r+1)*m) of the input (every rank the same m); on exit they hold
    global positions [r*m, (r+1)*m) of the stable sorted order.
    """
    if key_type not in _KEY_NAMES:
        raise ValueError(f"unknown key type {key_type!r}")
    m = keys.numel()
    ops = ops or DcOps(m)
    ops.sort_(keys, vals, key_type)                                  # levels >= log2 G
    if comm is None or comm.world == 1:
        return None
    G, me = comm.world, comm.rank
    wcap = stride
    q = -(-m // stride)
    samples = ops.sample(keys, stride)                               # a7
    cand = comm.all_gather(samples)                                  # C1: all-gather
    counts = ops.count(keys, me, cand, q, stride, key_type)
    granks = counts.clone()
    comm.all_reduce_sum_(granks)                                     # C2: all-reduce
    sendbuf = ops.windows(keys, me, G, counts, granks, q, wcap)
    gathered = comm.all_gather(sendbuf)                              # C3: all-gather
    cmat_t = ops.split_matrix(gathered, G, m, wcap, key_type)
    ops.check()
    cmat = cmat_t.cpu().tolist()                                     # the one host sync
    send, recv = split_sizes(cmat, me)
    rk = comm.all_to_all(keys, send, recv)                           # a8: all-to-all
    rv = comm.all_to_all(vals, send, recv) if vals is not None else None
    ops.merge_runs(rk, rv, keys, vals, recv, key_type)               # a9: local G-way merge
    return ExchangeInfo(cmat, send, recv)


def max_subarray(x: torch.Tensor, comm: Comm | None = None, ops=None):
    """(sum, start, end) of the whole distributed array; rank r holds the r-th
    consecutive piece (pieces may differ in length).  Same answer on every rank."""
    ops = ops or DcOps(x.numel())
    if comm is None or comm.world == 1:
        t = ops.maxsub_tuple(x, 0)
        return tuple(int(v) for v in ops.maxsub_combine(t.view(1, 8)).cpu().tolist())
    sizes = comm.all_gather(torch.tensor([x.numel()], dtype=torch.int64, device=x.device))
    offset = int(sizes[:comm.rank].sum().item())
    t = ops.maxsub_tuple(x, offset)                                  # a10: local summary
    allt = comm.all_gather(t)                                        # all-gather G tuples
    res = ops.maxsub_combine(allt.view(comm.world, 8))               # ordered combine
    return tuple(int(v) for v in res.cpu().tolist())


# ------------------------------------------------------------ N>1 bench

def bench_main(args, wl, workloads, metric):
    """bench.py under torchrun: 2^30 keys sharded over WORLD_SIZE GPUs (configs[4]).

    The product path: a plan of the global size bound to a library-owned NCCL
    communicator (``init_dist``); every step is one ``dc_run_mergesort`` per
    rank -- local levels, splitters, all-to-all and G-way merge in the library."""
    import json
    import os
    import statistics

    import torch.distributed as tdist

    import dcgen

    from . import init_dist

    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    tdist.init_process_group("nccl", device_id=dev)
    G, me = tdist.get_world_size(), tdist.get_rank()
    desc, n_total, kind = workloads[wl]
    if n_total % G:
        raise SystemExit("n must be divisible by the number of GPUs")
    plan = init_dist(n_total)
    m = plan.n
    pristine = dcgen.sort_keys(n_total, args.dist, seed=5, start=me * m, count=m, device=dev)
    keys = torch.empty_like(pristine)
    flush = torch.ones(64 << 20, dtype=torch.int64, device=dev)   # 512 MiB, read per flush
    fsum = torch.empty((), dtype=torch.int64, device=dev)
    stream = torch.cuda.current_stream(dev)

    def max_over_ranks(ms):
        t = torch.tensor([ms], dtype=torch.float64, device=dev)
        tdist.all_reduce(t, op=tdist.ReduceOp.MAX)
        return float(t.item())

    times = []
    l0 = None
    for i in range(args.warmup + args.steps):
        keys.copy_(pristine)
        torch.sum(flush, dtype=torch.int64, out=fsum)   # read-based L2 flush
        if i == args.warmup:
            l0 = plan.launch_count()
        tdist.barrier()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        plan.sort_(keys, key_type="u32")
        e1.record(stream)
        torch.cuda.synchronize()
        if i >= args.warmup:
            times.append(max_over_ranks(e0.elapsed_time(e1)))
    launches = plan.launch_count() - l0
    u = keys.to(torch.int64) & 0xFFFFFFFF
    desc_at = torch.nonzero(u[1:] < u[:-1]).flatten()
    unsorted = int(desc_at.numel())
    first_desc = desc_at[:4].tolist()
    ends = torch.stack([u[0], u[-1]])                  # rank boundaries: last(r) <= first(r+1)
    allends = torch.empty(2 * G, dtype=ends.dtype, device=dev)
    tdist.all_gather_into_tensor(allends, ends)
    e = allends.view(G, 2).cpu()
    boundaries_ok = bool(all(e[r, 1] <= e[r + 1, 0] for r in range(G - 1)))
    del u, desc_at
    ms = statistics.mean(times)
    splits = plan.last_splits() if G > 1 else [[0, m]]

    # kernel + phase breakdown (rank 0): second loop with per-launch events
    plan.enable_timing(True)
    if G > 1:
        plan.mg_reset_phases()
    for i in range(args.steps):
        keys.copy_(pristine)
        torch.sum(flush, dtype=torch.int64, out=fsum)   # read-based L2 flush
        tdist.barrier()
        plan.sort_(keys, key_type="u32")
    torch.cuda.synchronize()
    kt = plan.kernel_times()
    phases = plan.mg_phase_times() if G > 1 else None
    plan.enable_timing(False)
    exchange = None
    if phases and phases["sorts"]:
        ns = phases["sorts"]
        xms = phases["exchange_merge"] / ns
        recv_b = 4 * phases["keys_received"] / ns          # bytes in over NVLink per step
        exchange = {"mode": plan.exchange_mode(),
                    "local_sort_ms": phases["local_sort"] / ns,
                    "splitters_ms": phases["splitters"] / ns,
                    "exchange_merge_ms": xms,
                    "nvlink_bytes_in_per_rank": recv_b,
                    "nvlink_gbs_in": recv_b / (xms / 1e3) / 1e9 if xms else None,
                    "nvlink_frac_of_900": recv_b / (xms / 1e3) / 900e9 if xms else None,
                    "note": "exchange_merge overlaps the NVLink reads with the first merge "
                            "round when fused, so its GB/s is a lower bound on link use"}
    nk3_ms, nk3_n = kt["nk3_merge"]
    nk3_avg = nk3_ms / max(nk3_n, 1)

    # end to end through the public API: pinned host shard -> device -> sort -> host
    host = pristine.cpu().pin_memory()
    back = torch.empty_like(host).pin_memory()
    e2e = []
    for i in range(args.warmup + args.steps):
        tdist.barrier()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        keys.copy_(host, non_blocking=True)
        plan.sort_(keys, key_type="u32")
        back.copy_(keys, non_blocking=True)
        e1.record(stream)
        torch.cuda.synchronize()
        if i >= args.warmup:
            e2e.append(max_over_ranks(e0.elapsed_time(e1)))
    e2e_ms = statistics.mean(e2e)
    peak = 6650.0
    try:
        peak = float(json.load(open(os.path.join(os.path.dirname(os.path.dirname(
            os.path.abspath(__file__))), "MEASURED_PEAKS.json")))["hbm_gbs"])
    except Exception:
        pass
    moved = sum(splits[me][d + 1] - splits[me][d] for d in range(G) if d != me)
    if me == 0:
        ach = 8 * m / (nk3_avg / 1e3) / 1e9 if nk3_n else None
        print(json.dumps({
            "metric": metric, "value": n_total / (ms / 1e3), "unit": "keys/s", "n_gpus": G,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u32",
            "data": "synthetic (counter-based splitmix64)",
            "config": {"workload": wl, "description": desc, "n": n_total, "per_gpu": m,
                       "dist": args.dist, "parallelism": f"key-range sharding x{G}",
                       "runtime": "library-owned NCCL communicator (dc_plan_set_comm)",
                       "l2": "flushed before every step (512 MiB read)",
                       "local_descents": unsorted, "first_descents": first_desc,
                       "rank_boundaries_ordered": boundaries_ok, "rank0_keys_sent": moved,
                       "timing": "per-step CUDA events on every rank, max over ranks"},
            "roofline": {"kernel": "nk3_merge (rank 0, local merge levels + G-way merge)",
                         "bound": "hbm", "achieved": ach, "peak": peak, "unit": "GB/s",
                         "frac": ach / peak if ach else None, "traffic": None,
                         "avg_launch_ms": nk3_avg,
                         "kernels_ms_per_step": {k: v[0] / args.steps for k, v in kt.items()}},
            "gpu_launches": launches,
            "multi_gpu_phases": exchange,
            "e2e": {"value": n_total / (e2e_ms / 1e3), "unit": "keys/s", "ms_per_step": e2e_ms,
                    "h2d_bytes_per_step": 4 * n_total, "d2h_bytes_per_step": 4 * n_total},
            "cpu_baseline": None,
        }), flush=True)
    plan.close()
    tdist.destroy_process_group()
