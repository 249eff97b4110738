import torch, statistics
x = torch.randint(-1000, 1000, (1 << 24,), dtype=torch.int32, device="cuda")
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
def t(fn, flush_mode):
    ts = []
    for i in range(13):
        if flush_mode == "dirty": flush.zero_()
        elif flush_mode == "clean": flush.zero_(); torch.cuda.synchronize(); _ = flush.sum()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
        e0.record(); fn(); e1.record(); torch.cuda.synchronize()
        if i >= 3: ts.append(e0.elapsed_time(e1) * 1000)
    return statistics.median(ts)
for mode in ["dirty", "clean", "none"]:
    print(mode, "sum_i64 %.1f us" % t(lambda: x.sum(dtype=torch.int64), mode),
          "max %.1f us" % t(lambda: x.max(), mode), "clone %.1f us" % t(lambda: x.clone(), mode))
