#!/usr/bin/env python
"""Per-opcode and top-instruction stall attribution from an ncu report's SASS source page."""
import csv
import io
import subprocess
import sys
from collections import defaultdict

path = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
section = int(sys.argv[3]) if len(sys.argv) > 3 else 0  # which profiled launch
raw = subprocess.run(["ncu", "-i", path, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
starts = [i for i, r in enumerate(rows) if r and r[0] == "Address"]
st = starts[min(section, len(starts) - 1)]
end = starts[starts.index(st) + 1] - 1 if starts.index(st) + 1 < len(starts) else len(rows)
h = rows[st]
data = [r for r in rows[st + 1:end] if len(r) == len(h) and r[0] != "Address"]
idx = {n: i for i, n in enumerate(h)}
stalls = [n for n in h if n.startswith("stall_") and "Not Issued" not in n]
T = sum(int(r[idx[s]] or 0) for r in data for s in stalls)
tot = defaultdict(int)
byop = defaultdict(lambda: defaultdict(int))
for r in data:
    toks = r[1].split()
    op = toks[1] if toks and toks[0].startswith("@") and len(toks) > 1 else (toks[0] if toks else "")
    op = op.split(".")[0]
    for s in stalls:
        v = int(r[idx[s]] or 0)
        tot[s] += v
        byop[op][s] += v
print("samples", T)
print(" ".join(f"{k[6:]}={100 * v / T:.1f}%" for k, v in sorted(tot.items(), key=lambda x: -x[1]) if v))
for op, d in sorted(byop.items(), key=lambda x: -sum(x[1].values()))[:14]:
    t = sum(d.values())
    print(f"{op:10s} {100 * t / T:5.1f}%  " + ", ".join(f"{k[6:]}={100 * v / T:.1f}" for k, v in sorted(d.items(), key=lambda x: -x[1])[:5]))
print("--- top non-issue instructions (excluding selected / not_selected)")
scored = []
for r in data:
    v = sum(int(r[idx[s]] or 0) for s in stalls if s not in ("stall_selected", "stall_not_selected"))
    scored.append((v, r[0][-5:], r[1][:60], {s[6:]: int(r[idx[s]] or 0) for s in stalls
                                              if s not in ("stall_selected", "stall_not_selected") and int(r[idx[s]] or 0)}))
for v, a, src, d in sorted(scored, reverse=True)[:top]:
    print(f"{100 * v / T:5.2f}% {a} {src:60s} {d}")
