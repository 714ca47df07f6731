"""Summarise one kernel of gpurun_out/prof_full.ncu-rep: headline metrics, stall reasons, top source lines.
usage: python tools/ncu_k.py [report] [n_lines]"""
import csv, collections, subprocess, sys

rep = sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/prof_full.ncu-rep"
nl = int(sys.argv[2]) if len(sys.argv) > 2 else 30
ncu = "/usr/local/cuda/bin/ncu"
det = subprocess.run([ncu, "-i", rep, "--page", "details", "--csv"], capture_output=True, text=True).stdout
keys = ["Duration", "DRAM Throughput", "L1/TEX Cache Throughput", "L2 Cache Throughput", "Issue Slots Busy",
        "Eligible Warps Per Scheduler", "Achieved Active Warps Per SM", "L1/TEX Hit Rate", "L2 Hit Rate"]
for r in csv.reader(det.splitlines()):
    if len(r) > 14 and r[12] in keys:
        print(f"{r[12]:32s} {r[14]} {r[13]}")
raw = list(csv.reader(subprocess.run([ncu, "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                                     text=True).stdout.splitlines()))
h, v = raw[0], raw[2]
st = {}
for i, k in enumerate(h):
    if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued"):
        try:
            st[k[len("smsp__pcsamp_warps_issue_stalled_"):]] = float(v[i])
        except ValueError:
            pass
tot = sum(st.values()) or 1
print("stalls:", ", ".join(f"{k} {x / tot * 100:.0f}%" for k, x in sorted(st.items(), key=lambda x: -x[1]) if x / tot > 0.02))
for i, k in enumerate(h):
    if k in ("smsp__inst_executed.sum", "inst_executed"):
        print(k, v[i])
src = list(csv.reader(subprocess.run([ncu, "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                                     capture_output=True, text=True).stdout.splitlines()))
hh = src[2]
ei = hh.index("Instructions Executed")
agg = collections.defaultdict(lambda: [0, 0])
text = {}
line = None
fn = ""
for r in src[3:]:
    if not r:
        continue
    if r[0] in ("File Path", "Function Name", "Line No"):
        if r[0] == "File Path":
            fn = r[1].split("/")[-1]
        continue
    if r[0] != "":
        line = (fn, int(r[0]))
        text[line] = r[1][:90]
    elif len(r) > ei:
        try:
            agg[line][0] += int(r[ei] or 0)
            agg[line][1] += int(r[4] or 0)
        except ValueError:
            pass
ti = sum(x[0] for x in agg.values()) or 1
ts = sum(x[1] for x in agg.values()) or 1
print(f"instructions {ti}")
for l, (n, s) in sorted(agg.items(), key=lambda x: -x[1][1])[:nl]:
    print(f"{l[0][:14]:14s}:{l[1]:5d} inst {n / ti * 100:5.1f}%  stall {s / ts * 100:5.1f}%  {text.get(l, '')}")
