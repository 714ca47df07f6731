"""Summarise an ncu launch list (CSV) and a --set full report into markdown for profiles/."""
import csv
import json
import os
import subprocess
import sys

launches_csv, rep, out_md, tag = sys.argv[1], sys.argv[2], sys.argv[3], sys.argv[4]
rows = list(csv.reader(open(launches_csv)))
hdr = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
h = rows[hdr]
ki, vi = h.index("Kernel Name"), h.index("Metric Value")
lst = [(r[ki], float(r[vi])) for r in rows[hdr + 1:] if len(r) > vi]
# second reduce step only (the first launches are the generator + warm-up step)
names = [n for n, _ in lst]
start = max(i for i, n in enumerate(names) if "k_prep" in n and i > 0 and "k_prep" not in names[i - 1]) if names else 0
step = lst[start:]
tot = sum(v for _, v in step)
lines = [f"# {tag}: ncu summaries (C2, 1 x B200)", "",
         "## Launch list of one reduce step (`ncu --metrics gpu__time_duration.sum --clock-control none`)",
         "Cold-cache, serialised launches: compare shares, not absolutes.", "",
         "| kernel | ns | share |", "|---|---:|---:|"]
for n, v in step:
    short = n.split("(")[0].split("::")[-1]
    lines.append(f"| {short} | {v:.0f} | {v / tot:.3f} |")
lines.append(f"| **total** | {tot:.0f} | 1.000 |")
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
r = list(csv.reader(raw.splitlines()))
H = r[0]
want = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum", "launch__registers_per_thread",
        "launch__occupancy_limit_shared_mem", "lts__t_bytes.sum"]
lines += ["", "## `ncu --set full` (one launch each)", "",
          "| kernel | " + " | ".join(w.split("__")[1] if "__" in w else w for w in want) + " |",
          "|---|" + "---:|" * len(want)]
traffic = {}
for row in r[2:]:
    name = row[H.index("Kernel Name")].split("(")[0].split("::")[-1]
    vals = []
    for w in want:
        vals.append(row[H.index(w)] if w in H else "")
    lines.append(f"| {name} | " + " | ".join(vals) + " |")
    try:
        rd = float(row[H.index("dram__bytes_read.sum")]); wr = float(row[H.index("dram__bytes_write.sum")])
        ur = r[1][H.index("dram__bytes_read.sum")]; uw = r[1][H.index("dram__bytes_write.sum")]
        mul = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
        traffic[name] = rd * mul.get(ur, 1) + wr * mul.get(uw, 1)
    except Exception:
        pass
lines.append("")
lines.append("Units row: " + ", ".join(f"{w}={r[1][H.index(w)]}" for w in want if w in H))
open(out_md, "w").write("\n".join(lines) + "\n")
# merge into the existing table: a capture that skipped a kernel keeps that kernel's earlier entry
tpath = os.path.join(os.path.dirname(out_md), "traffic.json")
old = json.load(open(tpath)) if os.path.exists(tpath) else {}
merged = dict(old.get("all", {}))
merged.update(traffic)
srcs = dict(old.get("sources", {}))
srcs.update({k: rep for k in traffic})
json.dump({"what": "dram__bytes_read.sum + dram__bytes_write.sum per launch (ncu --set full, C2)", "all": merged,
           "sources": srcs, "tag": tag}, open(tpath, "w"), indent=1)
print("\n".join(lines))
