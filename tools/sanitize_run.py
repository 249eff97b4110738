#!/usr/bin/env python
"""Small invocations of every kernel path, for compute-sanitizer.

  compute-sanitizer --tool {memcheck,racecheck,synccheck,initcheck} python tools/sanitize_run.py [--large]
Checks results against the CPU oracle as it goes; exits non-zero on mismatch.
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import dcgen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_ipps_lopez_ortizss13_b200 as dc  # noqa: E402
import threading  # noqa: E402


def check_sort(n, key_type="u32", vals=False, graphs=False, dist_name="few"):
    keys = dcgen.sort_keys(n, dist_name, seed=5, key_type=key_type, device="cuda")
    v = dcgen.sort_vals(n, device="cuda") if vals else None
    view = {"u32": np.uint32, "i32": np.int32, "f32": np.float32}[key_type]
    k_in = keys.cpu().numpy().view(view)
    p = dc.Plan(n)
    p.set_graphs(graphs)
    p.sort_(keys, v, key_type=key_type)
    torch.cuda.synchronize()
    ek = oracle.mergesort(k_in, np.arange(n, dtype=np.uint32) if vals else None, key_type=key_type)
    ek = ek[0] if vals else ek
    assert np.array_equal(keys.cpu().numpy().view(np.uint32), ek.view(np.uint32)), (n, key_type)


def main():
    large = "--large" in sys.argv
    for n in (1, 17, 6528 * 3 + 5, 100_003):
        check_sort(n)
        check_sort(n, "i32")
        check_sort(n, "f32", vals=True)
        check_sort(n, vals=True)
    if large:   # the large-tile config (>= 2^23 keys) incl. two-level passes
        n = (1 << 23) + 25088 + 3
        check_sort(n)
        check_sort(n, vals=True)
        keys = dcgen.sort_keys(n, "uniform", seed=6, device="cuda")
        k_in = keys.cpu().numpy().view(np.uint32)
        p = dc.Plan(n)
        p.set_two_level(True)
        p.set_graphs(False)
        p.sort_(keys, key_type="u32")
        assert np.array_equal(keys.cpu().numpy().view(np.uint32), oracle.mergesort(k_in))
    for n in (1, 1000, 70_001):
        x = dcgen.maxsub_input(n, "small", seed=2, device="cuda")
        assert dc.Plan(n).max_subarray(x) == oracle.maxsub(x.cpu().numpy())
        assert dc.Plan(n).sum(x) == oracle.dc_sum(x.cpu().numpy())
    # multi-GPU runtime (library), loopback ranks sharing this GPU, both exchanges
    n, G = 4 * 20_011, 4
    full = dcgen.sort_keys(n, "few", seed=7).numpy().view(np.uint32)
    for p2p in (False, True):
        group = dc.LoopbackGroup(G)
        plans = []
        for r in range(G):
            p = dc.Plan(n)
            p.set_mg_p2p(p2p)
            p.set_mg_stride(256)
            p.set_loopback(group, r)
            plans.append(p)
        out = [None] * G

        def body(r):
            m = n // G
            s = torch.cuda.Stream()
            with torch.cuda.stream(s):
                k = dcgen.sort_keys(n, "few", seed=7, start=r * m, count=m, device="cuda")
                plans[r].sort_(k, key_type="u32")
                s.synchronize()
                out[r] = k.cpu()

        ts = [threading.Thread(target=body, args=(r,)) for r in range(G)]
        for t in ts:
            t.start()
        for t in ts:
            t.join()
        assert np.array_equal(torch.cat(out).numpy().view(np.uint32), oracle.mergesort(full)), p2p
        for p in plans:
            p.close()
        group.close()
    print("sanitize_run ok")


if __name__ == "__main__":
    main()
