"""Aggregate an ncu report's per-SASS stall samples by CUDA source line.

usage: python scripts/ncu_lines.py REP.ncu-rep [N]   (needs -lineinfo builds)
"""
import csv
import io
import subprocess
import sys
from collections import defaultdict

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
samples, execd, text = defaultdict(float), defaultdict(float), {}
fname = "?"
hdr = None
for r in rows:
    if len(r) == 2 and r[0] == "File Path":
        fname = r[1].rsplit("/", 1)[-1]
        continue
    if r and r[0] == "Line No":
        hdr = r
        continue
    if hdr is None or len(r) != len(hdr) or not r[0].strip().isdigit():
        continue
    key = (fname, int(r[0]))
    text[key] = r[1].strip()
    try:
        samples[key] += float(r[4].replace(",", "") or 0)
        execd[key] += float(r[7].replace(",", "") or 0)
    except ValueError:
        pass
tot = sum(samples.values()) or 1.0
print(f"total stall samples {tot:.0f}")
for k, v in sorted(samples.items(), key=lambda x: -x[1])[:top]:
    print(f"{k[0]}:{k[1]:<5} {100 * v / tot:6.2f}%  exec {execd[k] / 1e6:9.1f}M  {text[k][:70]}")
