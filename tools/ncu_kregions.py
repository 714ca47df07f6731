"""Per-line instruction counts of one kernel (regex) in an ncu report, top lines + stall samples.
usage: python tools/ncu_kregions.py report.ncu-rep kernel_regex [top_n]"""
import collections, csv, subprocess, sys

rep, kre = sys.argv[1], sys.argv[2]
nl = int(sys.argv[3]) if len(sys.argv) > 3 else 30
src = list(csv.reader(subprocess.run(["/usr/local/cuda/bin/ncu", "-i", rep, "--page", "source", "--csv",
                                      "--print-source", "cuda,sass", "-k", "regex:" + kre],
                                     capture_output=True, text=True).stdout.splitlines()))
h = src[2]
ei, si = h.index("Instructions Executed"), h.index("Warp Stall Sampling (All Samples)")
agg = collections.defaultdict(lambda: [0, 0])
text = {}
line = None
for r in src[3:]:
    if not r or r[0] in ("File Path", "Function Name", "Line No"):
        continue
    if r[0] != "":
        line = int(r[0])
        text[line] = r[1][:95]
    elif len(r) > ei:
        for j, k in enumerate((ei, si)):
            try:
                agg[line][j] += int(r[k] or 0)
            except ValueError:
                pass
ti = sum(v[0] for v in agg.values()) or 1
ts = sum(v[1] for v in agg.values()) or 1
print(f"instructions {ti}  stall samples {ts}")
for l, (n, s) in sorted(agg.items(), key=lambda x: -x[1][1])[:nl]:
    print(f"{l:5d} inst {n / ti * 100:5.1f}% stall {s / ts * 100:5.1f}%  {text.get(l, '')}")
