"""Loopback run of the library's multi-GPU sort (G ranks as threads on one
GPU) for profiling its kernels (mg_sample / mg_count / mg_brackets /
mg_windows / mg_split_matrix, the G-way merge's nk2_select4 + nk3_merge4 in
custom mode and the pair-mode nk2_partition_ab + nk3_merge_ab):
    ncu ... python tools/mg_profile.py <world> <log2 total n> <p2p 0|1>
Checks the result against torch.sort (diagnostic)."""
import os
import sys
import threading

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import dcgen  # noqa: E402
import paper_conf_ipps_lopez_ortizss13_b200 as dc  # noqa: E402

G = int(sys.argv[1]) if len(sys.argv) > 1 else 4
n = 1 << (int(sys.argv[2]) if len(sys.argv) > 2 else 26)
p2p = (sys.argv[3] == "1") if len(sys.argv) > 3 else False
m = n // G
group = dc.LoopbackGroup(G)
plans = []
for r in range(G):
    p = dc.Plan(n)
    p.set_mg_p2p(p2p)
    p.set_loopback(group, r)
    plans.append(p)
out = [None] * G


def body(r):
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        k = dcgen.sort_keys(n, "uniform", seed=5, start=r * m, count=m, device="cuda")
        plans[r].sort_(k, key_type="u32")
        s.synchronize()
        out[r] = k


ts = [threading.Thread(target=body, args=(r,)) for r in range(G)]
for t in ts:
    t.start()
for t in ts:
    t.join()
got = torch.cat(out).to(torch.int64) & 0xFFFFFFFF
ref = torch.sort(dcgen.sort_keys(n, "uniform", seed=5, device="cuda").to(torch.int64)
                 & 0xFFFFFFFF).values
print(f"mg_profile G={G} n=2^{n.bit_length() - 1} mode={plans[0].exchange_mode()} "
      f"sorted_ok={bool(torch.equal(got, ref))}")
