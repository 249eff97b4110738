"""Measured sweep for the NK1 cluster rule (dc_api.cu cluster_rule).

u32 keys-only sorts at every size n, NK1 cluster size cs in {1, 2, 4, 8, 16},
tile class 1/2 and one/two levels per pass, timed like bench.py (graph
replay, input restored and L2 flushed by a 512 MiB read before every sort,
CUDA events; median of K).  One JSON line per point on stdout.
"""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import dcgen  # noqa: E402
import paper_conf_ipps_lopez_ortizss13_b200 as dc  # noqa: E402

K, W = 9, 3
SIZES = [1 << k for k in (16, 18, 20, 22, 24, 26)]
if os.environ.get("DC_SWEEP_SIZES"):
    SIZES = [1 << int(k) for k in os.environ["DC_SWEEP_SIZES"].split(",")]
dev = torch.device("cuda", 0)
flush = torch.ones(64 << 20, dtype=torch.int64, device=dev)
fsum = torch.empty((), dtype=torch.int64, device=dev)
stream = torch.cuda.current_stream(dev)
for n in SIZES:
    pk = dcgen.sort_keys(n, "uniform", seed=3, device=dev)
    keys = torch.empty_like(pk)
    ref = torch.sort(pk.to(torch.int64) & 0xFFFFFFFF).values
    for tc in (1, 2):
        for two in (False, True):
            for cs in (1, 2, 4, 8, 16):
                plan = dc.Plan(n)
                plan.set_tile_class(tc)
                plan.set_two_level(two)
                plan.set_nk1_cluster(cs)
                sch = plan.schedule("u32")

                def one():
                    keys.copy_(pk)
                    torch.sum(flush, dim=0, out=fsum)
                    e0 = torch.cuda.Event(enable_timing=True)
                    e1 = torch.cuda.Event(enable_timing=True)
                    e0.record(stream)
                    plan.sort_(keys, None, key_type="u32")
                    e1.record(stream)
                    return e0, e1

                try:
                    for _ in range(W):
                        one()
                    evs = [one() for _ in range(K)]
                    torch.cuda.synchronize()
                    ms = statistics.median(a.elapsed_time(b) for a, b in evs)
                    ok = bool(torch.equal(keys.to(torch.int64) & 0xFFFFFFFF, ref))
                    err = None
                except RuntimeError as e:
                    ms, ok, err = None, False, str(e)[:200]
                print(json.dumps({"n": n, "tile_class": tc, "two_level": two, "cs": cs,
                                  "ms": ms, "schedule": sch, "sorted_ok": ok, "error": err}),
                      flush=True)
