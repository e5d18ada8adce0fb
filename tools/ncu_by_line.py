"""Warp-stall samples of an ncu report aggregated per CUDA source line.
usage: python tools/ncu_by_line.py report.ncu-rep [N]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
agg, src_text, fname, hdr = {}, {}, None, None
for r in csv.reader(io.StringIO(out)):
    if not r:
        continue
    if r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r[0] == "Line No":
        hdr = r
        continue
    if hdr is None or len(r) < 5:
        continue
    try:
        line = int(r[0])
        samples = int(r[4] or 0)
    except ValueError:
        continue
    key = (fname, line)
    agg[key] = agg.get(key, 0) + samples
    src_text[key] = r[1].strip()
tot = sum(agg.values()) or 1
for key in sorted(agg, key=lambda k: -agg[k])[:n]:
    print(f"{agg[key] / tot * 100:5.1f}% {key[0]}:{key[1]}  {src_text[key][:90]}")
print("total samples", tot)
