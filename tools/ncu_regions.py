#!/usr/bin/env python
"""Stall samples of an ncu source page (csv[.gz], --print-source sass) grouped
into contiguous regions: prints every run of instructions with its sample
share and the top stall reasons, so the hot loops of a kernel are visible."""
import csv
import gzip
import io
import sys

path = sys.argv[1]
minshare = float(sys.argv[2]) if len(sys.argv) > 2 else 0.5
op = gzip.open if path.endswith(".gz") else open
rows = list(csv.reader(io.StringIO(op(path, "rt").read())))
hi = [i for i, r in enumerate(rows) if "Source" in r and "Address" in r][0]
h = rows[hi]
col = {n: i for i, n in enumerate(h)}
reasons = [n for n in h if n.startswith("stall_") and "Not Issued" not in n]
data = []
for r in rows[hi + 1:]:
    try:
        s = int(r[col["Warp Stall Sampling (All Samples)"]])
        ex = int(r[col["Instructions Executed"]] or 0)
    except (ValueError, IndexError):
        continue
    rs = {n: int(r[col[n]] or 0) for n in reasons}
    data.append((r[col["Address"]], r[col["Source"]].strip(), s, ex, rs))
tot = sum(d[2] for d in data) or 1
texe = sum(d[3] for d in data) or 1
print(f"samples {tot}, instructions executed {texe}")
# regions: split where a branch target / label gap occurs -> use fixed windows of 16
W = 16
for i in range(0, len(data), W):
    blk = data[i:i + W]
    s = sum(d[2] for d in blk)
    if 100.0 * s / tot < minshare:
        continue
    ex = sum(d[3] for d in blk)
    agg = {n: sum(d[4][n] for d in blk) for n in reasons}
    top = sorted(agg.items(), key=lambda kv: -kv[1])[:4]
    ops = " ".join(d[1].split()[0] if not d[1].startswith("@") else d[1].split()[1] for d in blk)
    print(f"{blk[0][0][-5:]} {100.0 * s / tot:5.1f}% smp {100.0 * ex / texe:5.1f}% exe  "
          + " ".join(f"{n[6:]}={100.0 * v / max(s, 1):.0f}%" for n, v in top) + f"  | {ops[:110]}")
