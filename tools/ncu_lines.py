"""Per-source-line instruction counts of one kernel in an ncu report, grouped into line ranges.
usage: python tools/ncu_lines.py report.ncu-rep [top_n]"""
import collections, csv, subprocess, sys

rep = sys.argv[1]
nl = int(sys.argv[2]) if len(sys.argv) > 2 else 40
src = list(csv.reader(subprocess.run(["/usr/local/cuda/bin/ncu", "-i", rep, "--page", "source", "--csv",
                                      "--print-source", "cuda,sass"], capture_output=True, text=True).stdout.splitlines()))
hh = src[2]
ei = hh.index("Instructions Executed")
agg = collections.defaultdict(int)
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
        text[line] = r[1][:100]
    elif len(r) > ei:
        try:
            agg[line] += int(r[ei] or 0)
        except ValueError:
            pass
ti = sum(agg.values()) or 1
print(f"instructions {ti}")
for l, n in sorted(agg.items(), key=lambda x: -x[1])[:nl]:
    print(f"{l[0][:14]:14s}:{l[1]:5d} {n / ti * 100:5.1f}%  {text.get(l, '')}")
