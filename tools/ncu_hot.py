"""Hottest CUDA source lines of an ncu report: warp-stall samples summed per
(file, line) from `ncu -i X --page source --csv --print-source cuda,sass`
(needs -lineinfo builds).

    python tools/ncu_hot.py gpurun_out/p.ncu-rep [top]
"""
import collections
import csv
import io
import os
import subprocess
import sys

path = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
out = subprocess.run(["ncu", "-i", path, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
agg = collections.Counter()
text = {}
fname = "?"
hdr = None
for r in csv.reader(io.StringIO(out)):
    if not r:
        continue
    if r[0] == "File Path":
        fname = os.path.basename(r[1])
        continue
    if r[0] == "Line No":
        hdr = r
        continue
    if hdr is None or len(r) < 5:
        continue
    try:
        v = float(r[4])
    except ValueError:
        continue
    key = (fname, r[0])
    agg[key] += v
    if r[1].strip():
        text[key] = r[1].strip()
tot = sum(agg.values()) or 1
for (f, ln), v in agg.most_common(top):
    print(f"{100 * v / tot:5.1f}%  {f}:{ln:<5} {text.get((f, ln), '')[:100]}")
