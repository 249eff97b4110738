"""Host<->device copy bandwidth on the GPU box (the bound of the e2e legs):
pinned 1 GiB H2D alone, D2H alone, and both at once on two streams."""
import json
import torch

N = 1 << 28                      # 1 GiB of u32
h_in = torch.empty(N, dtype=torch.int32).pin_memory()
h_out = torch.empty(N, dtype=torch.int32).pin_memory()
d_a = torch.empty(N, dtype=torch.int32, device="cuda")
d_b = torch.empty(N, dtype=torch.int32, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()


def timed(fn, reps=5):
    best = None
    for _ in range(reps):
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        for s in (s1, s2):
            torch.cuda.current_stream().wait_stream(s)
        e1.record()
        torch.cuda.synchronize()
        t = e0.elapsed_time(e1) / 1e3
        best = t if best is None else min(best, t)
    return best


def h2d():
    with torch.cuda.stream(s1):
        d_a.copy_(h_in, non_blocking=True)


def d2h():
    with torch.cuda.stream(s2):
        h_out.copy_(d_b, non_blocking=True)


def both():
    h2d()
    d2h()


for s in (s1, s2):
    s.wait_stream(torch.cuda.current_stream())
gb = 4 * N / 1e9
r = {"h2d_gbs": gb / timed(h2d), "d2h_gbs": gb / timed(d2h)}
t = timed(both)
r["concurrent_each_gbs"] = gb / t
r["concurrent_ms_per_GiB_pair"] = t * 1e3
print(json.dumps(r))
