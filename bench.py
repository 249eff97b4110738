#!/usr/bin/env python
"""Benchmark of the breadth-first D&C hot path on B200 (one JSON line on rank 0).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl dc|reference]
                    [--workload sort_u32|sort_kv|sort_u32_small|maxsub] [--dist uniform]

A step is one pass of the whole hot path over one batch of synthetic input:
for the sort workloads, NK1 (fused bottom levels) + every global merge level
(NK2 + NK3) of a stable mergesort of n keys; for max-subarray, NK4 + NK5.

Default workload (N=1): BASELINE configs[2], mergesort of 2^28 uniform uint32
keys on one B200 -- the configuration the metric "sorted keys/sec (32-bit,
2^28-2^30)" is quoted on.  N>1: configs[4], 2^30 keys sharded over N GPUs with
the cross-GPU top-level merge (see paper_conf_ipps_lopez_ortizss13_b200/dist.py).

Timing: inputs resident in HBM; before every step (untimed) the keys are
restored from a pristine device copy and L2 is flushed by READING a 512 MiB
buffer (a read leaves L2 full of clean lines, so the timed kernels do not pay
for write-backs of a dirty flush buffer); each step is bracketed by CUDA events on the launching stream; W
warm-up steps, then exactly K timed steps between barrier + synchronize.
Per-kernel device times come from the library's own event instrumentation
(dc_plan_kernel_time) over the same timed steps.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

WORKLOADS = {
    # name: (description, n, kind)
    "sort_u32": ("mergesort of 2^28 uint32 keys on 1 B200 (BASELINE configs[2])", 1 << 28, "sort"),
    "sort_kv": ("stable mergesort of 2^28 uint32 key + uint32 value pairs (configs[3])", 1 << 28,
                "sort_kv"),
    "sort_u32_small": ("mergesort of 2^20 uniform uint32 keys (configs[0])", 1 << 20, "sort"),
    "maxsub": ("max-subarray-sum D&C on 2^24 int32 values (configs[1])", 1 << 24, "maxsub"),
    "sum": ("D&C sum (Alg 4, SURVEY f4) of 2^24 int32 values, exact int64", 1 << 24, "sum"),
    "sort_u32_2p30": ("mergesort of 2^30 uint32 keys sharded over N B200 (configs[4])", 1 << 30,
                      "sort"),
}
METRIC = "sorted keys/sec (32-bit, 2^28-2^30) at 1/2/4/8 B200; per-pass HBM GB/s vs peak"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["dc", "reference"], default="dc")
    ap.add_argument("--workload", choices=sorted(WORKLOADS), default=None)
    ap.add_argument("--dist", default="uniform")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    return ap.parse_args()


# ----------------------------------------------------------------- helpers

def peaks():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        d = json.load(open(path))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md: 6.65 TB/s)"


class L2Flush:
    """Evicts L2 (126 MB) by reading a 512 MiB buffer (sum into a scalar).
    The buffer is written once at setup; every flush is a pure read, so L2
    is left holding clean lines and the next kernel's misses cost no
    write-backs (a write-based flush dirtied L2 and taxed every small-n line)."""

    def __init__(self, dev, mib: int = 512):
        import torch

        self.buf = torch.ones((mib << 20) // 8, dtype=torch.int64, device=dev)
        self.out = torch.empty((), dtype=torch.int64, device=dev)

    def __call__(self):
        import torch

        torch.sum(self.buf, dim=0, out=self.out)


def ncu_entry(kernel: str, workload: str, key: str):
    """One field of the committed ncu --set full summary (profiles/ncu_summary.json)."""
    path = os.path.join(ROOT, "profiles", "ncu_summary.json")
    try:
        return json.load(open(path))[workload][kernel][key]
    except Exception:
        return None


def ncu_traffic(kernel: str, workload: str):
    """dram bytes per launch of `kernel` from the committed ncu --set full summary."""
    path = os.path.join(ROOT, "profiles", "ncu_summary.json")
    try:
        d = json.load(open(path))
        return d[workload][kernel]["dram_bytes_per_launch"]
    except Exception:
        return None


class ClockSampler:
    """SM clocks + throttle reasons sampled through NVML every 10 ms during the
    timed region (the recipe's nvidia-smi clocks line, at a finer interval so a
    ~100 ms region still gets many samples)."""

    REASONS = {"hw_slowdown": "nvmlClocksEventReasonHwSlowdown",
               "hw_thermal_slowdown": "nvmlClocksEventReasonHwThermalSlowdown",
               "sw_thermal_slowdown": "nvmlClocksEventReasonSwThermalSlowdown",
               "sw_power_cap": "nvmlClocksEventReasonSwPowerCap"}

    def __init__(self, index: int):
        self.index = index
        self.samples = []
        self.stop = None
        self.err = None

    def _run(self):
        import pynvml as nv

        try:
            nv.nvmlInit()
            h = nv.nvmlDeviceGetHandleByIndex(self.index)
            mx = nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_SM)
            while True:
                sm = nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM)
                rs = nv.nvmlDeviceGetCurrentClocksEventReasons(h)
                self.samples.append((sm, mx, rs))
                self.ready.set()
                if self.stop.wait(0.01):
                    break
        except Exception as e:  # noqa: BLE001 - reported in the JSON line
            self.err = repr(e)
        finally:
            self.ready.set()

    def __enter__(self):
        import threading

        self.stop = threading.Event()
        self.ready = threading.Event()   # set after NVML init + the first sample
        self.t = threading.Thread(target=self._run, daemon=True)
        self.t.start()
        self.ready.wait(timeout=30)
        return self

    def __exit__(self, *a):
        self.stop.set()
        self.t.join(timeout=5)

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None,
                    "reasons": ["nvml unavailable: %s" % self.err]}
        import pynvml as nv

        reasons = sorted({name for _, _, rs in self.samples for name, attr in
                          self.REASONS.items() if rs & getattr(nv, attr)})
        return {"sm_mhz": statistics.median(s[0] for s in self.samples),
                "sm_max_mhz": max(s[1] for s in self.samples), "reasons": reasons,
                "samples": len(self.samples), "source": "NVML, 10 ms interval"}


def cpu_info():
    model = "unknown"
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                model = line.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    return model, os.cpu_count()


# --------------------------------------------------------- oracle timings

def oracle_sort_sample(n_total: int, dist: str, kv: bool, budget_s: float = 12.0,
                       sample_n: int | None = None):
    """The oracle (Alg 6, 1 thread) on the workload, as it stands.  By default
    on the FULL input (sample_n = n_total: one run, ~30 s at 2^28 on the box's
    host) so the CPU rate is the rate at the config size (mergesort's per-key
    rate falls with log n); a smaller sample_n times prefixes, repeated for
    budget_s."""
    import numpy as np

    import dcgen
    import oracle

    sample_n = n_total if sample_n is None else min(sample_n, n_total)
    keys = dcgen.sort_keys(n_total, dist, seed=3, start=0, count=sample_n).numpy().view(np.uint32)
    vals = np.arange(sample_n, dtype=np.uint32) if kv else None
    reps, t0 = 0, time.perf_counter()
    while True:
        oracle.mergesort(keys, vals)
        reps += 1
        el = time.perf_counter() - t0
        if el > budget_s or reps >= 20:
            break
    return reps * sample_n / el, reps, sample_n, el


def oracle_maxsub_sample(n_total: int, dist: str, budget_s: float = 12.0):
    import dcgen
    import oracle

    x = dcgen.maxsub_input(n_total, dist, seed=2).numpy()
    reps, t0 = 0, time.perf_counter()
    while True:
        oracle.maxsub(x)
        reps += 1
        el = time.perf_counter() - t0
        if el > budget_s or reps >= 50:
            break
    return reps * x.size / el, reps, x.size, el


# ------------------------------------------------------------ reference arm

def run_reference(args, wl):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    desc, n, kind = WORKLOADS[wl]
    model, cores = cpu_info()
    step_times = []
    if kind == "maxsub":
        import dcgen
        import oracle

        x = dcgen.maxsub_input(n, args.dist, seed=2).numpy()
        sample_n = n
        for i in range(args.warmup + args.steps):
            t0 = time.perf_counter()
            oracle.maxsub(x)
            if i >= args.warmup:
                step_times.append(time.perf_counter() - t0)
        unit = "elements/s"
        sample = f"oracle recursive D&C max-subarray of the full 2^24 input, 1 thread, per step"
    else:
        import numpy as np

        import dcgen
        import oracle

        # Largest power-of-two prefix whose (W + K) one-thread sorts fit in
        # about three minutes, from a 2^20 calibration run (the full 2^28 takes
        # ~30 s per step on the box's host, too long for K = 10).
        cal = dcgen.sort_keys(n, args.dist, seed=3, count=1 << 20).numpy().view(np.uint32)
        t0 = time.perf_counter()
        oracle.mergesort(cal)
        per_key = (time.perf_counter() - t0) / (1 << 20) * 1.15   # log n growth to 2^26
        sample_n = 1 << 20
        while sample_n * 2 <= n and (args.warmup + args.steps) * per_key * sample_n * 2 <= 180.0:
            sample_n *= 2
        keys = dcgen.sort_keys(n, args.dist, seed=3, count=sample_n).numpy().view(np.uint32)
        vals = np.arange(sample_n, dtype=np.uint32) if kind == "sort_kv" else None
        for i in range(args.warmup + args.steps):
            t0 = time.perf_counter()
            oracle.mergesort(keys, vals)
            if i >= args.warmup:
                step_times.append(time.perf_counter() - t0)
        unit = "keys/s"
        sample = (f"oracle Alg 6 recursive mergesort (1 thread) of the first 2^"
                  f"{sample_n.bit_length() - 1} keys of the {desc} workload, per step (the "
                  f"largest power-of-two prefix whose {args.warmup + args.steps} steps fit ~3 min)")
    t = statistics.mean(step_times)
    v = sample_n / t
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": v, "unit": unit, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": t * 1e3,
        "higher_is_better": True, "scaling": "strong" if args.gpus > 1 else "weak",
        "vs_baseline": None, "dtype": "u32" if kind != "maxsub" else "i32",
        "data": "synthetic (counter-based splitmix64)",
        "config": {"workload": wl, "description": desc, "n": n, "dist": args.dist,
                   "sample_n": sample_n},
        "cpu_baseline": {"value": v, "unit": unit, "cores": 1, "kind": "oracle",
                         "sample": sample, "cpu": model, "host_cores": cores},
        "e2e": {"value": v, "unit": unit, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)


# ------------------------------------------------------------------ our arm

def run_dc(args, wl):
    import torch

    import dcgen
    import paper_conf_ipps_lopez_ortizss13_b200 as dc

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1 or os.environ.get("DC_BENCH_DIST"):   # DC_BENCH_DIST=1: that path at N=1
        from paper_conf_ipps_lopez_ortizss13_b200 import dist as dcdist

        return dcdist.bench_main(args, wl, WORKLOADS, METRIC)
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    desc, n, kind = WORKLOADS[wl]
    if kind == "maxsub":
        return run_dc_maxsub(args, wl, desc, n)
    if kind == "sum":
        return run_dc_sum(args, wl, desc, n)

    kv = kind == "sort_kv"
    pristine_k = dcgen.sort_keys(n, args.dist, seed=3, device=dev)
    keys = torch.empty_like(pristine_k)
    vals = torch.empty_like(pristine_k) if kv else None
    pristine_v = dcgen.sort_vals(n, device=dev) if kv else None
    flush = L2Flush(dev)
    plan = dc.Plan(n)
    stream = torch.cuda.current_stream(dev)
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
          for _ in range(args.warmup + args.steps)]

    def prep():
        keys.copy_(pristine_k)
        if kv:
            vals.copy_(pristine_v)
        flush()

    for i in range(args.warmup):
        prep()
        ev[i][0].record(stream)
        plan.sort_(keys, vals, key_type="u32")
        ev[i][1].record(stream)
    torch.cuda.synchronize()
    # Timed region: K steps exactly as a user runs them (CUDA-graph replay of
    # the level sequence, no instrumentation).
    launches0 = plan.launch_count()
    with ClockSampler(local) as clk:
        torch.cuda.synchronize()
        for i in range(args.warmup, args.warmup + args.steps):
            prep()
            ev[i][0].record(stream)
            plan.sort_(keys, vals, key_type="u32")
            ev[i][1].record(stream)
        torch.cuda.synchronize()
    launches = plan.launch_count() - launches0
    step_ms = [ev[i][0].elapsed_time(ev[i][1]) for i in range(args.warmup, args.warmup + args.steps)]
    ms = statistics.mean(step_ms)
    value = n / (ms / 1e3)
    # Kernel breakdown: the same K steps again with per-launch CUDA events on the
    # plan stream (dc_plan_kernel_time; graphs are off while timing is on).
    plan.enable_timing(True)
    bk = []
    for i in range(args.steps):
        prep()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        plan.sort_(keys, vals, key_type="u32")
        e1.record(stream)
        bk.append((e0, e1))
    torch.cuda.synchronize()
    kt = plan.kernel_times()
    plan.enable_timing(False)
    ms_instr = statistics.mean(a.elapsed_time(b) for a, b in bk)

    # correctness spot-check of the last timed output (cheap invariant, untimed)
    k64 = keys.to(torch.int64) & 0xFFFFFFFF
    sorted_ok = bool((k64[1:] >= k64[:-1]).all())
    del k64

    sched = plan.schedule("u32", kv)
    peak, peak_src = peaks()
    bytes_per_key = 16 if kv else 8
    nk3_ms, nk3_n = kt["nk3_merge"]
    nk1_ms, nk1_n = kt["nk1_blocksort"]
    nk2_ms, nk2_n = kt["nk2_partition"]
    nk3_avg = nk3_ms / max(nk3_n, 1)
    achieved = bytes_per_key * n / (nk3_avg / 1e3) / 1e9 if nk3_n else None
    nk1_avg = nk1_ms / max(nk1_n, 1)
    two = sched["hbm_passes"] < sched["global_passes"]
    roofline = {
        "kernel": ("nk3_merge4 (one HBM pass = two merge levels: 4-way tile merge; the pass's "
                   "exact 4-run selection is nk2_partition)") if two
                  else "nk3_merge (one global merge level)",
        "levels_per_launch": 2 if two else 1,
        "bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
        "frac": achieved / peak if achieved else None,
        "traffic": ncu_traffic("nk3_merge4" if two else "nk3_merge", wl),
        "algorithmic_bytes_per_launch": bytes_per_key * n,
        "avg_launch_ms": nk3_avg, "peak_source": peak_src,
        "share_of_step": nk3_ms / args.steps / ms_instr if ms_instr else None,
        "measured": "per-launch CUDA events on the plan stream over a second loop of the same K "
                    "steps (the timed loop runs uninstrumented, graph replay)",
    }
    kernels = {
        "nk1_blocksort": {"avg_ms": nk1_avg, "launches_per_step": nk1_n / args.steps,
                          "hbm_gbs": bytes_per_key * n / (nk1_avg / 1e3) / 1e9 if nk1_n else None,
                          "share_of_step": nk1_ms / args.steps / ms_instr},
        "nk2_partition": {"kernel": "nk2_select4" if two else "nk2_partition",
                          "avg_ms": nk2_ms / max(nk2_n, 1), "launches_per_step": nk2_n / args.steps,
                          "share_of_step": nk2_ms / args.steps / ms_instr},
        "nk3_merge": {"kernel": "nk3_merge4" if two else "nk3_merge",
                      "avg_ms": nk3_avg, "launches_per_step": nk3_n / args.steps,
                      "hbm_gbs": achieved, "share_of_step": nk3_ms / args.steps / ms_instr},
    }

    # Shared-memory roofline of the two merge kernels (both bound by shared-memory
    # wavefronts): LSU wavefronts per launch from the committed
    # ncu capture of the same workload / live launch time, against one wavefront
    # per clock per SM at the clock NVML saw during the timed loop.
    csum = clk.summary()
    mhz = csum.get("sm_mhz") or csum.get("sm_max_mhz")
    if mhz and args.dist == "uniform":   # (the ncu capture is of the uniform workload)
        speak = torch.cuda.get_device_properties(local).multi_processor_count * float(mhz) * 1e6
        smem = {"unit": "wavefronts/s", "peak": speak,
                "peak_source": "1 wavefront / clock / SM x SMs x NVML SM clock; TMA traffic excluded",
                "wavefronts_source": "profiles/ncu_summary.json (ncu l1tex shared ld + st wavefronts)"}
        for name, kern, avg in (("nk1_blocksort", "nk1_blocksort", nk1_avg),
                                ("nk3_merge", "nk3_merge4" if two else "nk3_merge", nk3_avg)):
            w = ncu_entry(kern, wl, "smem_wavefronts_per_launch")
            if w and avg:
                kernels[name]["smem_roofline"] = dict(smem, wavefronts_per_launch=w,
                                                      achieved=w / (avg / 1e3),
                                                      frac=w / (avg / 1e3) / speak)

    e2e = None
    if not args.no_e2e:
        e2e = e2e_sort(args, plan, n, kv, pristine_k, pristine_v)

    cpu = None
    if not args.no_cpu_baseline:
        v, reps, sn, el = oracle_sort_sample(n, args.dist, kv)
        model, cores = cpu_info()
        cpu = {"value": v, "unit": "keys/s", "cores": 1, "kind": "oracle",
               "sample": (f"oracle Alg 6 recursive mergesort, 1 thread, the full {sn}-key input "
                          f"of this workload ({el:.1f} s)" if sn == n else
                          f"oracle Alg 6 recursive mergesort, 1 thread, {reps} x the first {sn} "
                          f"keys of this workload ({el:.1f} s)"),
               "cpu": model, "host_cores": cores}

    print(json.dumps({
        "metric": METRIC, "value": value, "unit": "keys/s", "n_gpus": 1, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "u32", "data": "synthetic (counter-based splitmix64)",
        "config": {"workload": wl, "description": desc, "n": n, "dist": args.dist,
                   "key_type": "u32", "values": kv, "tile": sched["tile"],
                   "fused_levels": sched["fused_levels"], "global_passes": sched["global_passes"],
                   "hbm_passes": sched["hbm_passes"],
                   "l2": "flushed before every step (512 MiB read); input "
                         + (f"{n * (8 if kv else 4) / 2**30:.0f} GiB > L2" if n * 4 > (126 << 20)
                            else f"{n * (8 if kv else 4) / 2**20:.0f} MiB, L2-resident after the first level"),
                   "step_ms_min": min(step_ms), "step_ms_max": max(step_ms),
                   "instrumented_step_ms": ms_instr,
                   "sorted_check": sorted_ok},
        "roofline": roofline, "kernels": kernels, "gpu_launches": launches,
        "clocks": csum, "e2e": e2e, "cpu_baseline": cpu,
    }), flush=True)


def e2e_sort(args, plan, n, kv, pristine_k, pristine_v):
    """Same metric through the C ABI with pinned HOST buffers: every step
    uploads its input, sorts and downloads its result (dc_sort_host_submit);
    consecutive steps overlap upload / sort / download on separate streams.
    Timed with CUDA events on the plan stream, which the submissions follow
    and dc_sort_host_wait joins."""
    import torch

    hk = pristine_k.cpu().pin_memory()          # never modified by the call
    hv = pristine_v.cpu().pin_memory() if kv else None
    ok = torch.empty_like(hk).pin_memory()
    ov = torch.empty_like(hv).pin_memory() if kv else None
    stream = torch.cuda.current_stream()
    for _ in range(args.warmup):
        plan.sort_host_submit(hk, ok, hv, ov, key_type="u32")
    plan.sort_host_wait()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(args.steps):
        plan.sort_host_submit(hk, ok, hv, ov, key_type="u32")
    plan.sort_host_wait()
    e1.record(stream)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / args.steps
    return {"value": n / (ms / 1e3), "unit": "keys/s", "ms_per_step": ms,
            "h2d_bytes_per_step": n * 4 * (2 if kv else 1),
            "d2h_bytes_per_step": n * 4 * (2 if kv else 1),
            "mode": "streamed host sorts, 3 device slots, copies overlapped across steps",
            "copy_bound": "tools/pcie_probe.py (profiles/r01/pcie_probe.json): pinned 1 GiB H2D ~55 GB/s, D2H ~57 GB/s alone, 45-50 GB/s each way concurrent (varies by box) = 21.5-23.5 ms per GiB in + GiB out"}


def run_dc_maxsub(args, wl, desc, n):
    import torch

    import dcgen
    import paper_conf_ipps_lopez_ortizss13_b200 as dc

    dev = torch.device("cuda", torch.cuda.current_device())
    x = dcgen.maxsub_input(n, args.dist if args.dist != "uniform" else "uniform", seed=2,
                           device=dev)
    out = torch.empty(3, dtype=torch.int64, device=dev)
    flush = L2Flush(dev)
    plan = dc.Plan(n)
    stream = torch.cuda.current_stream(dev)
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
          for _ in range(args.warmup + args.steps)]
    for i in range(args.warmup):
        flush()
        ev[i][0].record(stream)
        plan.max_subarray_async(x, out)
        ev[i][1].record(stream)
    torch.cuda.synchronize()
    # Timed region: K steps as a user runs them (no per-kernel instrumentation;
    # r02 timed this loop with the plan's per-launch events on, which added
    # their records to every step).
    l0 = plan.launch_count()
    with ClockSampler(dev.index) as clk:
        for i in range(args.warmup, args.warmup + args.steps):
            flush()
            ev[i][0].record(stream)
            plan.max_subarray_async(x, out)
            ev[i][1].record(stream)
        torch.cuda.synchronize()
    launches = plan.launch_count() - l0
    step_ms = [ev[i][0].elapsed_time(ev[i][1]) for i in range(args.warmup, args.warmup + args.steps)]
    ms = statistics.mean(step_ms)
    # Kernel time: the same K steps again with per-launch CUDA events on the
    # plan stream (dc_plan_kernel_time).
    plan.enable_timing(True)
    for i in range(args.steps):
        flush()
        plan.max_subarray_async(x, out)
    torch.cuda.synchronize()
    kt = plan.kernel_times()
    plan.enable_timing(False)
    k_ms, k_n = kt["nk4_maxsub"]
    avg = k_ms / max(k_n, 1)
    peak, src = peaks()
    ach = 4 * n / (avg / 1e3) / 1e9
    # e2e through the C ABI with a pinned host buffer
    hx = x.cpu().pin_memory()
    times = []
    for i in range(args.warmup + args.steps):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        plan.max_subarray_host(hx)
        if i >= args.warmup:
            times.append(time.perf_counter() - t0)
    e2e_ms = statistics.mean(times) * 1e3
    cpu = None
    if not args.no_cpu_baseline:
        v, reps, sn, el = oracle_maxsub_sample(n, "uniform")
        model, cores = cpu_info()
        cpu = {"value": v, "unit": "elements/s", "cores": 1, "kind": "oracle",
               "sample": f"oracle recursive D&C max-subarray, 1 thread, {reps} x the full input "
                         f"({el:.1f} s)", "cpu": model, "host_cores": cores}
    print(json.dumps({
        "metric": "max-subarray elements/sec (2^24 int32)", "value": n / (ms / 1e3),
        "unit": "elements/s", "n_gpus": 1, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": ms, "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
        "dtype": "i32->i64", "data": "synthetic (counter-based splitmix64)",
        "config": {"workload": wl, "description": desc, "n": n, "dist": args.dist,
                   "l2": "flushed before every step (512 MiB read)"},
        "roofline": {"kernel": "nk4_maxsub (tiles + last-CTA top combine)", "bound": "hbm",
                     "achieved": ach, "peak": peak, "unit": "GB/s", "frac": ach / peak,
                     "traffic": ncu_traffic("nk4_maxsub", wl), "avg_launch_ms": avg,
                     "algorithmic_bytes_per_launch": 4 * n, "peak_source": src},
        "gpu_launches": launches, "clocks": clk.summary(),
        "e2e": {"value": n / (e2e_ms / 1e3), "unit": "elements/s", "ms_per_step": e2e_ms,
                "h2d_bytes_per_step": 4 * n, "d2h_bytes_per_step": 24},
        "cpu_baseline": cpu,
    }), flush=True)


def run_dc_sum(args, wl, desc, n):
    """f4 instance: the D&C sum through the generic O(1)-combine template."""
    import torch

    import dcgen
    import paper_conf_ipps_lopez_ortizss13_b200 as dc

    dev = torch.device("cuda", torch.cuda.current_device())
    x = dcgen.maxsub_input(n, "uniform", seed=2, device=dev)
    out = torch.empty(1, dtype=torch.int64, device=dev)
    flush = L2Flush(dev)
    plan = dc.Plan(n)
    stream = torch.cuda.current_stream(dev)
    times = []
    l0 = None
    with ClockSampler(dev.index) as clk:
        for i in range(args.warmup + args.steps):
            flush()
            if i == args.warmup:
                l0 = plan.launch_count()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            plan.sum_async(x, out)
            e1.record(stream)
            if i >= args.warmup:
                times.append((e0, e1))
        torch.cuda.synchronize()
    launches = plan.launch_count() - l0
    ms = statistics.mean(a.elapsed_time(b) for a, b in times)
    peak, src = peaks()
    ach = 4 * n / (ms / 1e3) / 1e9
    print(json.dumps({
        "metric": "D&C sum elements/sec (2^24 int32, SURVEY f4)", "value": n / (ms / 1e3),
        "unit": "elements/s", "n_gpus": 1, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": ms, "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
        "dtype": "i32->i64", "data": "synthetic (counter-based splitmix64)",
        "config": {"workload": wl, "description": desc, "n": n,
                   "l2": "flushed before every step (512 MiB read)"},
        "roofline": {"kernel": "breadth_first_reduce<SumI64> (one launch = the step)",
                     "bound": "hbm", "achieved": ach, "peak": peak, "unit": "GB/s",
                     "frac": ach / peak, "traffic": ncu_traffic("breadth_first_reduce", wl),
                     "avg_launch_ms": ms,
                     "algorithmic_bytes_per_launch": 4 * n, "peak_source": src},
        "gpu_launches": launches, "clocks": clk.summary(), "e2e": None, "cpu_baseline": None,
    }), flush=True)


def main():
    args = parse()
    wl = args.workload or ("sort_u32" if args.gpus == 1 else "sort_u32_2p30")
    if args.impl == "reference":
        return run_reference(args, wl)
    return run_dc(args, wl)


if __name__ == "__main__":
    main()
