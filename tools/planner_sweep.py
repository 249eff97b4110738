"""Measured sweep for the schedule planner (model.cu).

For every key class (u32 keys, f32 keys, u32 key-value), size n and forced
schedule (tile class 1/2 x one/two levels per pass) it times whole sorts the
way bench.py does (graph replay, inputs restored and L2 flushed by a 512 MiB
read before every sort, CUDA events on the plan stream; median of K) and,
in a second loop with per-launch events, the per-kernel-class times.
Writes JSON lines to stdout; tools/planner_fit.py fits the planner's
coefficients to them.
"""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import dcgen  # noqa: E402
import paper_conf_ipps_lopez_ortizss13_b200 as dc  # noqa: E402

K, W = 7, 3
SIZES = [1 << k for k in range(14, 29)] + [3 << 21, 3 << 23, 3 << 25]
if os.environ.get("DC_SWEEP_SIZES"):      # e.g. "24,26,28": powers of two only
    SIZES = [1 << int(k) for k in os.environ["DC_SWEEP_SIZES"].split(",")]
CLASSES = [("u32", False), ("f32", False), ("u32", True)]
if len(sys.argv) > 1:
    CLASSES = [c for c in CLASSES if f"{c[0]}{'_kv' if c[1] else ''}" in sys.argv[1].split(",")]

dev = torch.device("cuda", 0)
flush = torch.ones(64 << 20, dtype=torch.int64, device=dev)
fsum = torch.empty((), dtype=torch.int64, device=dev)
stream = torch.cuda.current_stream(dev)
for kt, kv in CLASSES:
    for n in sorted(SIZES):
        pk = dcgen.sort_keys(n, "uniform", seed=3, key_type=kt, device=dev)
        pv = dcgen.sort_vals(n, device=dev) if kv else None
        keys = torch.empty_like(pk)
        vals = torch.empty_like(pv) if kv else None
        for tc in (1, 2):
            for two in (False, True):
                plan = dc.Plan(n)
                plan.set_tile_class(tc)
                plan.set_two_level(two)
                sch = plan.schedule(kt, kv)

                def one():
                    keys.copy_(pk)
                    if kv:
                        vals.copy_(pv)
                    torch.sum(flush, dim=0, out=fsum)
                    e0 = torch.cuda.Event(enable_timing=True)
                    e1 = torch.cuda.Event(enable_timing=True)
                    e0.record(stream)
                    plan.sort_(keys, vals, key_type=kt)
                    e1.record(stream)
                    return e0, e1

                for _ in range(W):
                    one()
                evs = [one() for _ in range(K)]
                torch.cuda.synchronize()
                ms = statistics.median(a.elapsed_time(b) for a, b in evs)
                # diagnostic: the output equals torch.sort of the input (keys)
                if kt == "u32":
                    ref = torch.sort(pk.to(torch.int64) & 0xFFFFFFFF).values
                    ok = bool(torch.equal(keys.to(torch.int64) & 0xFFFFFFFF, ref))
                else:
                    ok = bool(torch.equal(keys, torch.sort(pk).values))

                plan.enable_timing(True)
                for _ in range(3):
                    one()
                torch.cuda.synchronize()
                kt_ms = {k: (v[0] / 3, v[1] / 3) for k, v in plan.kernel_times().items()}
                plan.enable_timing(False)
                print(json.dumps({"class": kt + ("_kv" if kv else ""), "n": n, "tile_class": tc,
                                  "two_level": two, "ms": ms, "schedule": sch, "sorted_ok": ok,
                                  "kernels": kt_ms}), flush=True)
                plan.close()
        del pk, pv, keys, vals
        torch.cuda.empty_cache()
