"""Aggregate compute-sanitizer racecheck hazards by (kind, first access, second access) source lines."""
import re
import sys
from collections import Counter

pairs = Counter()
kind = None
acc = []
for line in open(sys.argv[1], errors="replace"):
    m = re.search(r"Potential (\w+) hazard", line)
    if m:
        if kind and len(acc) == 2:
            pairs[(kind, acc[0], acc[1])] += 1
        kind, acc = m.group(1), []
        continue
    m = re.search(r"(Read|Write) Thread .* in (\S+:\d+)", line)
    if m and kind:
        acc.append(f"{m.group(1)} {m.group(2)}")
if kind and len(acc) == 2:
    pairs[(kind, acc[0], acc[1])] += 1
for (k, a, b), n in pairs.most_common():
    print(f"{n:9d}  {k}  {a}  <->  {b}")
