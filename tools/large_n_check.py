"""Sortedness + multiset checks of the single-GPU sort at large n (diagnostic)."""
import sys

import torch

import dcgen
import paper_conf_ipps_lopez_ortizss13_b200 as dc


def check(n, dist="uniform", vals=False, graphs=True, reps=1, comm=False, flush=False):
    pristine = dcgen.sort_keys(n, dist, seed=5, device="cuda")
    u = pristine.to(torch.int64) & 0xFFFFFFFF
    s0, x0 = int(u.sum()), int((u * u % 1000003).sum())
    del u
    k = torch.empty_like(pristine)
    v = dcgen.sort_vals(n, device="cuda") if vals else None
    p = dc.Plan(n)
    p.set_graphs(graphs)
    if comm:
        p.set_comm(dc.get_unique_id(), 0, 1)
    fl = torch.empty(512 << 20, dtype=torch.uint8, device="cuda") if flush else None
    for _ in range(reps):
        k.copy_(pristine)
        if fl is not None:
            fl.zero_()
        p.sort_(k, v, key_type="u32")
    torch.cuda.synchronize()
    u = k.to(torch.int64) & 0xFFFFFFFF
    bad = torch.nonzero(u[1:] < u[:-1])
    s1, x1 = int(u.sum()), int((u * u % 1000003).sum())
    first = bad[:5].flatten().tolist()
    print(f"n={n} reps={reps} graphs={graphs} comm={comm} flush={flush} dist={dist} vals={vals} unsorted_at={bad.numel()} first={first} "
          f"multiset_ok={s0 == s1 and x0 == x1} sched={p.schedule('u32', vals)}", flush=True)
    del k, v, u, p, pristine
    torch.cuda.empty_cache()


if __name__ == "__main__":
    reps = int(sys.argv[1])
    mode = sys.argv[2]
    for arg in sys.argv[3:]:
        check(int(eval(arg)), reps=reps, comm="comm" in mode, flush="flush" in mode)
