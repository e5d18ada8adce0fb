"""Print the SASS instructions with the most warp-stall samples from an ncu report.
usage: python tools/ncu_top_sass.py report.ncu-rep [N] [kernel-index]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True,
                     text=True).stdout
blocks = out.split('"Kernel Name"')
blk = blocks[1] if len(blocks) > 1 else out
lines = blk.split("\n", 1)[1]
rows = list(csv.reader(io.StringIO(lines)))
hdr = rows[0]
iS, iA, iN = hdr.index("Source"), hdr.index("Address"), hdr.index("Warp Stall Sampling (All Samples)")
data = []
for r in rows[1:]:
    if len(r) != len(hdr):
        continue
    try:
        data.append((int(r[iN]), r[iA][-5:], r[iS].strip()))
    except ValueError:
        pass
tot = sum(d[0] for d in data) or 1
for k, (c, a, s) in enumerate(data):
    pass
top = sorted(range(len(data)), key=lambda i: -data[i][0])[:n]
for i in sorted(top):
    c, a, s = data[i]
    print(f"{c / tot * 100:5.1f}% {a} {s}")
print("total samples", tot)
