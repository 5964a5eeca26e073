#!/usr/bin/env python
"""Per-source-line warp-stall samples from an ncu report (needs -lineinfo + --import-source on).
Usage: ncu_line_stalls.py report.ncu-rep [launch_index] [top]"""
import csv
import io
import subprocess
import sys
from collections import defaultdict

path = sys.argv[1]
launch = int(sys.argv[2]) if len(sys.argv) > 2 else 0
top = int(sys.argv[3]) if len(sys.argv) > 3 else 30
raw = subprocess.run(["ncu", "-i", path, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
secs = [i for i, r in enumerate(rows) if r and r[0] == "File Path"]
# group file sections by launch: a new launch starts when a file repeats
launches, seen = [[]], set()
for i in secs:
    f = rows[i][1]
    if f in seen:
        launches.append([])
        seen = set()
    seen.add(f)
    launches[-1].append(i)
sel = launches[min(launch, len(launches) - 1)]
stats, tot = [], 0
for st in sel:
    end = next((j for j in secs if j > st), len(rows))
    fname = rows[st][1].split("/")[-1]
    hdr = rows[st + 2]
    iS = hdr.index("Warp Stall Sampling (All Samples)")
    for r in rows[st + 3:end]:
        if r and r[0] not in ("", "-") and len(r) > iS:
            try:
                v = int(r[iS] or 0)
            except ValueError:  # source text with embedded quotes breaks the CSV row
                continue
            if v:
                stats.append((v, fname, r[0], r[1].strip()))
                tot += v
print(f"launch {launch}: {len(launches)} launches, {tot} samples")
for v, f, l, s in sorted(stats, reverse=True)[:top]:
    print(f"{100 * v / tot:5.1f}% {f}:{l}: {s[:100]}")
