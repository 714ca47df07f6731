"""Instructions executed per source-line range of an ncu report (source page).
usage: python tools/ncu_regions.py report.ncu-rep name:a-b [name:a-b ...]"""
import collections, csv, subprocess, sys

rep = sys.argv[1]
src = list(csv.reader(subprocess.run(["/usr/local/cuda/bin/ncu", "-i", rep, "--page", "source", "--csv",
                                      "--print-source", "cuda,sass"], capture_output=True, text=True).stdout.splitlines()))
ei = src[2].index("Instructions Executed")
agg = collections.defaultdict(int)
line = None
for r in src[3:]:
    if not r or r[0] in ("File Path", "Function Name", "Line No"):
        continue
    if r[0] != "":
        line = int(r[0])
    elif len(r) > ei:
        try:
            agg[line] += int(r[ei] or 0)
        except ValueError:
            pass
tot = sum(agg.values())
print(f"total {tot}")
for spec in sys.argv[2:]:
    name, ab = spec.split(":")
    a, b = map(int, ab.split("-"))
    v = sum(n for l, n in agg.items() if l is not None and a <= l <= b)
    print(f"{name:12s} {v:12d} {v / tot * 100:5.1f}%")
