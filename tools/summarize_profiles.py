#!/usr/bin/env python
"""Turn gpurun_out/ ncu artefacts into the committed profiles/<round>/ summaries.

  python tools/summarize_profiles.py r01
writes profiles/<round>/launches_<workload>.csv (dc:: launches of one step),
profiles/<round>/ncu_<kernel>.json (headline metrics + stalls of one launch) and
profiles/ncu_summary.json (DRAM bytes per launch, read by bench.py as
roofline.traffic).
"""
import collections
import csv
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from ncu_summary import summarise  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
rnd = sys.argv[1] if len(sys.argv) > 1 else "r01"
out = os.path.join(ROOT, "profiles", rnd)
os.makedirs(out, exist_ok=True)
G = os.path.join(ROOT, "gpurun_out")


def to_us(v, u):
    v = float(v.replace(",", ""))
    return v * 1e3 if u == "ms" else (v / 1e3 if u == "ns" else v)


# ---- launch list: keep the dc:: kernels, report one step (the last one)
lpath = os.path.join(G, "launches.csv")
if os.path.exists(lpath):
    rows = list(csv.reader(open(lpath)))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    h = rows[hi]
    ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
    seq = [(r[ki].split("(")[0].replace("void ", ""), to_us(r[vi], r[ui]))
           for r in rows[hi + 1:] if "dc::" in r[ki]]
    starts = [i for i, (n, _) in enumerate(seq) if "nk1_blocksort" in n]
    step = seq[starts[-1]:] if starts else seq
    tot = sum(t for _, t in step)
    with open(os.path.join(out, "launches_sort_u32.csv"), "w") as f:
        f.write("# ncu --metrics gpu__time_duration.sum --clock-control none, bench.py default "
                "(2^28 u32), last step; cold-cache serialised launches: compare SHARES\n")
        f.write("kernel,us,share\n")
        for n, t in step:
            f.write(f"{n},{t:.3f},{t / tot:.4f}\n")
    agg = collections.OrderedDict()
    for n, t in step:
        k = n.split("<")[0].replace("dc::", "")
        a = agg.setdefault(k, [0, 0.0])
        a[0] += 1
        a[1] += t
    print("launch list (one step):", {k: (c, round(t, 1), round(t / tot, 3)) for k, (c, t) in agg.items()})

# ---- full captures
summary = {}
caps = {"prof_nk1": ("sort_u32", "nk1_blocksort"), "prof_nk2": ("sort_u32", "nk2_select4"),
        "prof_nk3": ("sort_u32", "nk3_merge4"), "prof_nk3_kv": ("sort_kv", "nk3_merge4"),
        "prof_nk4": ("maxsub", "nk4_maxsub"), "prof_nk1_kv": ("sort_kv", "nk1_blocksort"),
        "prof_sum": ("sum", "breadth_first_reduce")}
def load_summary(cap):
    """Summary of one capture: the .ncu-rep if it came back, else the JSON the
    box wrote with tools/ncu_summary.py (reports are summarised and deleted
    there to keep gpurun_out/ under the 64 MiB copy-back limit)."""
    p = os.path.join(G, cap + ".ncu-rep")
    if os.path.exists(p):
        return summarise(p)
    j = os.path.join(G, cap + ".summary.json")
    if os.path.exists(j):
        text = open(j).read()
        return json.loads(text[text.index("["):])
    return None


for cap, (wl, kern) in caps.items():
    ss = load_summary(cap)
    if not ss:
        continue
    s = ss[0]
    json.dump(s, open(os.path.join(out, f"ncu_{wl}_{kern}.json"), "w"), indent=1)
    rd = float(s["dram__bytes_read.sum"].split()[0]) * (1e9 if "Gbyte" in s["dram__bytes_read.sum"] else 1e6 if "Mbyte" in s["dram__bytes_read.sum"] else 1e3)
    wr = float(s["dram__bytes_write.sum"].split()[0]) * (1e9 if "Gbyte" in s["dram__bytes_write.sum"] else 1e6 if "Mbyte" in s["dram__bytes_write.sum"] else 1e3)
    ent = {"dram_bytes_per_launch": rd + wr, "duration": s["gpu__time_duration.sum"],
           "source": f"profiles/{rnd}/ncu_{wl}_{kern}.json"}
    try:   # shared-memory wavefronts of LSU loads + stores (TMA traffic not included)
        ent["smem_wavefronts_per_launch"] = (
            float(s["l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum"])
            + float(s["l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum"]))
    except (KeyError, ValueError):
        pass
    summary.setdefault(wl, {})[kern] = ent
    print(wl, kern, s["gpu__time_duration.sum"], f"dram {(rd + wr) / 1e9:.4f} GB")
json.dump(summary, open(os.path.join(ROOT, "profiles", "ncu_summary.json"), "w"), indent=1)

# ---- multi-GPU kernels in loopback (tools/mg_profile.py under ncu): one JSON per mode
for mode in ("a2a", "fused"):
    ss = load_summary(f"prof_mg_{mode}")
    if ss:
        json.dump(ss, open(os.path.join(out, f"ncu_mg_{mode}.json"), "w"), indent=1)
        print("mg", mode, [(x["kernel"][:40], x.get("gpu__time_duration.sum")) for x in ss][:8])

# ---- bench lines of the same build (last JSON line of each gpurun_out/bench_*.json)
import glob  # noqa: E402

for bp in sorted(glob.glob(os.path.join(G, "bench_*.json"))) + [os.path.join(G, "pcie_probe.json")]:
    if not os.path.exists(bp):
        continue
    lines = [ln for ln in open(bp).read().splitlines() if ln.startswith("{")]
    if not lines:
        continue
    with open(os.path.join(out, os.path.basename(bp)), "w") as f:
        f.write(lines[-1] + "\n")
    d = json.loads(lines[-1])
    if "ms_per_step" in d:
        print(os.path.basename(bp), round(d["ms_per_step"], 4), "ms", d.get("value"), d.get("unit"))
