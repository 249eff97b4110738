"""Multi-GPU bench driver and its global verification (rows a7-a10, e).

The distributed method itself lives in the library (``csrc/mg_runtime.cu``):
a plan of global size n bound to a library-owned NCCL communicator
(:func:`paper_conf_ipps_lopez_ortizss13_b200.init_dist`) sorts rank r's shard
of global positions [r*m, (r+1)*m) with one ``dc_run_mergesort`` call --
local levels (independent subproblems), exact composite-order splitters
(sample all-gather, counts all-reduce, window all-gather, split matrix), the
exchange (NCCL all-to-all, or fused into the 4-way merge reading the peers'
shards over NVLink) and the local G-way merge (Alg 7's top log2 G levels).
This module only drives it under torchrun for ``bench.py`` and checks the
result globally; it holds no copy of the protocol.

Verification (pure torch, any process group -- NCCL here, gloo in the CPU
tests): every rank's output slice is non-decreasing, the slices are ordered
across rank boundaries, and the output is a permutation of the input, proven
by an all-reduced multiset fingerprint (sum of the keys and sum of a 64-bit
mix of every key, both mod 2^64) that must equal the input's.
"""
from __future__ import annotations

import torch

_M1 = 0xBF58476D1CE4E5B9 - (1 << 64)     # splitmix64 finaliser constants as int64
_M2 = 0x94D049BB133111EB - (1 << 64)
_GOLD = 0x9E3779B97F4A7C15 - (1 << 64)
_CHUNK = 1 << 24


def _mix64(x: torch.Tensor) -> torch.Tensor:
    """splitmix64 finaliser on int64 (wrapping multiplies; logical shifts
    emulated by masking the sign-extended bits)."""
    def srl(v, s):
        return (v >> s) & ((1 << (64 - s)) - 1)

    z = x * _GOLD
    z = (z ^ srl(z, 30)) * _M1
    z = (z ^ srl(z, 27)) * _M2
    return z ^ srl(z, 31)


def fingerprint(keys: torch.Tensor) -> torch.Tensor:
    """int64[3] of a 32-bit key tensor: (count, sum of keys, sum of mix64(key)),
    sums wrapping mod 2^64.  Equal multisets give equal fingerprints; a
    changed, lost or duplicated key changes the mix sum except with
    probability ~2^-64."""
    out = torch.zeros(3, dtype=torch.int64, device=keys.device)
    flat = keys.reshape(-1)
    out[0] = flat.numel()
    for i in range(0, flat.numel(), _CHUNK):
        u = flat[i:i + _CHUNK].to(torch.int64) & 0xFFFFFFFF
        out[1] += u.sum()
        out[2] += _mix64(u).sum()
    return out


def locally_sorted(keys: torch.Tensor) -> int:
    """Number of descents (positions i with key[i+1] < key[i], unsigned)."""
    flat = keys.reshape(-1)
    bad = 0
    for i in range(0, max(flat.numel() - 1, 0), _CHUNK):
        u = flat[i:i + _CHUNK + 1].to(torch.int64) & 0xFFFFFFFF
        bad += int((u[1:] < u[:-1]).sum())
    return bad


def verify_global_sort(in_fp: torch.Tensor, out_keys: torch.Tensor, group=None) -> dict:
    """Collective check that the rank slices form the global sorted order of
    the input whose per-rank fingerprints are in_fp: all-reduced fingerprints
    equal, every slice non-decreasing, last(r) <= first(r+1) for every r."""
    import torch.distributed as tdist

    G = tdist.get_world_size(group)
    fin = in_fp.clone()
    fout = fingerprint(out_keys)
    tdist.all_reduce(fin, group=group)
    tdist.all_reduce(fout, group=group)
    desc = torch.tensor([locally_sorted(out_keys)], dtype=torch.int64, device=out_keys.device)
    tdist.all_reduce(desc, group=group)
    u = out_keys.reshape(-1)
    ends = (torch.stack([u[0], u[-1]]).to(torch.int64) & 0xFFFFFFFF) if u.numel() else \
        torch.tensor([1 << 32, -1], dtype=torch.int64, device=out_keys.device)
    allends = [torch.empty_like(ends) for _ in range(G)]
    tdist.all_gather(allends, ends, group=group)
    e = torch.stack(allends).cpu()
    boundaries = all(int(e[r, 1]) <= int(e[r + 1, 0]) for r in range(G - 1))
    same = bool(torch.equal(fin.cpu(), fout.cpu()))
    return {"multiset_fingerprint_equal": same, "descents": int(desc.item()),
            "rank_boundaries_ordered": boundaries,
            "ok": same and int(desc.item()) == 0 and boundaries}


# ------------------------------------------------------------ N>1 bench

def _nvlink_peak() -> float:
    return 900.0


def bench_main(args, wl, workloads, metric):
    """bench.py under torchrun: 2^30 keys sharded over WORLD_SIZE GPUs (configs[4]).

    Both exchange modes of the library runtime are timed on the same input:
    the default NCCL all-to-all (value, headline) and the fused exchange (the
    4-way merge reading the peers' shards over NVLink); each is verified
    globally (verify_global_sort) after its timed loop.  Step time = CUDA
    events on every rank, max over ranks."""
    import json
    import os
    import statistics

    import torch.distributed as tdist

    import dcgen

    from . import init_dist

    if "RANK" not in os.environ:          # DC_BENCH_DIST=1 without torchrun: a world of one
        import socket

        sk = socket.socket()
        sk.bind(("127.0.0.1", 0))
        os.environ.update(RANK="0", WORLD_SIZE="1", LOCAL_RANK="0", MASTER_ADDR="127.0.0.1",
                          MASTER_PORT=str(sk.getsockname()[1]))
        sk.close()
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    tdist.init_process_group("nccl", device_id=dev)
    G, me = tdist.get_world_size(), tdist.get_rank()
    desc, n_total, kind = workloads[wl]
    if n_total % G:
        raise SystemExit("n must be divisible by the number of GPUs")
    m = n_total // G
    pristine = dcgen.sort_keys(n_total, args.dist, seed=5, start=me * m, count=m, device=dev)
    in_fp = fingerprint(pristine)
    keys = torch.empty_like(pristine)
    flush = torch.ones(64 << 20, dtype=torch.int64, device=dev)   # 512 MiB, read per flush
    fsum = torch.empty((), dtype=torch.int64, device=dev)
    stream = torch.cuda.current_stream(dev)

    def max_over_ranks(ms):
        t = torch.tensor([ms], dtype=torch.float64, device=dev)
        tdist.all_reduce(t, op=tdist.ReduceOp.MAX)
        return float(t.item())

    def prep():
        keys.copy_(pristine)
        torch.sum(flush, dim=0, out=fsum)   # read-based L2 flush

    def run_mode(p2p: bool) -> dict:
        plan = init_dist(n_total)
        plan.set_mg_p2p(p2p)
        times, l0 = [], None
        for i in range(args.warmup + args.steps):
            prep()
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
        check = verify_global_sort(in_fp, keys, None)
        mode = plan.exchange_mode()
        splits = plan.last_splits() if G > 1 else [[0, m]]
        # phase + kernel breakdown: a second loop with per-launch events
        plan.enable_timing(True)
        if G > 1:
            plan.mg_reset_phases()
        for _ in range(args.steps):
            prep()
            tdist.barrier()
            plan.sort_(keys, key_type="u32")
        torch.cuda.synchronize()
        kt = plan.kernel_times()
        phases = plan.mg_phase_times() if G > 1 else None
        plan.enable_timing(False)
        ms = statistics.mean(times)
        out = {"mode": mode, "ms_per_step": ms, "keys_per_s": n_total / (ms / 1e3),
               "step_ms_min": min(times), "step_ms_max": max(times), "verify": check,
               "gpu_launches": launches,
               "kernels_ms_per_step": {k: v[0] / args.steps for k, v in kt.items()},
               "rank0_keys_sent": sum(splits[me][d + 1] - splits[me][d] for d in range(G)
                                      if d != me)}
        if phases and phases["sorts"]:
            ns = phases["sorts"]
            xms = phases["exchange_merge"] / ns
            recv_b = 4 * phases["keys_received"] / ns     # bytes in over NVLink per step
            out.update({
                "local_sort_ms": phases["local_sort"] / ns,
                "splitters_ms": phases["splitters"] / ns,
                "exchange_merge_ms": xms,
                "nvlink_bytes_in_per_rank": recv_b,
                "nvlink_gbs_in": recv_b / (xms / 1e3) / 1e9 if xms else None,
                "nvlink_frac_of_900": (recv_b / (xms / 1e3) / 1e9 / _nvlink_peak()
                                       if xms else None),
                "note": "exchange_merge = exchange + G-way merge on the plan stream (rank 0); "
                        "its GB/s is a lower bound on link use (the merge shares the time)"})
        nk3_ms, nk3_n = kt["nk3_merge"]
        out["nk3_avg_ms"] = nk3_ms / max(nk3_n, 1)
        return out, plan

    primary, plan = run_mode(False)       # default: NCCL all-to-all
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
    plan.close()
    torch.cuda.empty_cache()
    fused = None
    if G > 1 or os.environ.get("DC_BENCH_FUSED", "1") == "1":
        try:
            fused, fplan = run_mode(True)
            fplan.close()
        except Exception as e:  # noqa: BLE001 - reported in the JSON line
            fused = {"error": repr(e)[:300]}
    peak = 6650.0
    try:
        peak = float(json.load(open(os.path.join(os.path.dirname(os.path.dirname(
            os.path.abspath(__file__))), "MEASURED_PEAKS.json")))["hbm_gbs"])
    except Exception:
        pass
    if me == 0:
        ms = primary["ms_per_step"]
        ach = 8 * m / (primary["nk3_avg_ms"] / 1e3) / 1e9 if primary["nk3_avg_ms"] else None
        print(json.dumps({
            "metric": metric, "value": n_total / (ms / 1e3), "unit": "keys/s", "n_gpus": G,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u32",
            "data": "synthetic (counter-based splitmix64)",
            "config": {"workload": wl, "description": desc, "n": n_total, "per_gpu": m,
                       "dist": args.dist, "parallelism": f"key-range sharding x{G}",
                       "runtime": "library-owned NCCL communicator (dc_plan_set_comm)",
                       "exchange": primary["mode"],
                       "l2": "flushed before every step (512 MiB read)",
                       "timing": "per-step CUDA events on every rank, max over ranks"},
            "verify": primary["verify"],
            "roofline": {"kernel": "nk3_merge4 / nk3_merge (rank 0: local passes + G-way merge)",
                         "bound": "hbm", "achieved": ach, "peak": peak, "unit": "GB/s",
                         "frac": ach / peak if ach else None, "traffic": None,
                         "avg_launch_ms": primary["nk3_avg_ms"],
                         "kernels_ms_per_step": primary["kernels_ms_per_step"]},
            "gpu_launches": primary["gpu_launches"],
            "modes": {"all_to_all": primary, "fused": fused},
            "e2e": {"value": n_total / (e2e_ms / 1e3), "unit": "keys/s", "ms_per_step": e2e_ms,
                    "h2d_bytes_per_step": 4 * n_total, "d2h_bytes_per_step": 4 * n_total},
            "cpu_baseline": None,
        }), flush=True)
    tdist.destroy_process_group()
