#!/usr/bin/env python
"""Top SASS lines by warp-stall samples from an ncu report's source page."""
import csv
import io
import subprocess
import sys

path = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
out = subprocess.run(["ncu", "-i", path, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hi = [i for i, r in enumerate(rows) if "Source" in r and "Address" in r][0]
h = rows[hi]
si, ai = h.index("Source"), h.index("Warp Stall Sampling (All Samples)")
ei = h.index("Instructions Executed") if "Instructions Executed" in h else None
data = []
for r in rows[hi + 1:]:
    try:
        data.append((int(r[ai]), r[si].strip(), r[ei] if ei is not None else ""))
    except (ValueError, IndexError):
        pass
tot = sum(d[0] for d in data) or 1
print(f"total samples {tot}, instructions {len(data)}")
for s, src, ex in sorted(data, key=lambda d: -d[0])[:top]:
    print(f"{100.0 * s / tot:5.1f}%  {ex:>10}  {src}")
