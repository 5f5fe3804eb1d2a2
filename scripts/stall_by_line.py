"""Aggregate ncu warp-stall samples of one kernel by CUDA source line.

usage: python scripts/stall_by_line.py <report.ncu-rep> <kernel-regex> <cubin> [top]
Joins `ncu --page source --print-source sass` (per-SASS-instruction samples) with
`nvdisasm -g` line info of the cubin (compile with -lineinfo)."""
import csv
import io
import re
import subprocess
import sys
from collections import defaultdict

rep, kre, cubin = sys.argv[1], sys.argv[2], sys.argv[3]
import os
KSEL = os.environ.get("KSEL", "ILi16EddLi0E")
top = int(sys.argv[4]) if len(sys.argv) > 4 else 30
raw = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass", "-k", f"regex:{kre}"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
hdr_i = next(i for i, r in enumerate(rows) if r and r[0] == "Address")
hdr = rows[hdr_i]
si = hdr.index("Warp Stall Sampling (All Samples)")
samples = []
for r in rows[hdr_i + 1:]:
    if len(r) <= si or not r[0].startswith("0x"):
        if samples:
            break
        continue
    samples.append((int(r[0], 16), float(r[si] or 0), r[1]))
base = samples[0][0]
# function name of the first kernel matching
kname = rows[0][1] if rows and rows[0] and rows[0][0] == "Kernel Name" else ""
dis = subprocess.run(["nvdisasm", "-g", "-c", cubin], capture_output=True, text=True).stdout
# find function section matching the mangled name pattern
funcs = re.split(r"\n\s*\.text\.", dis)
best = None
for f in funcs:
    head = f.split("\n", 1)[0]
    if re.search(kre, head) and (KSEL in head or best is None):
        best = f
        if KSEL in head:
            break
line_of = {}
cur = None
for ln in best.split("\n"):
    m = re.search(r'//## File ".*?/([^/"]+)", line (\d+)', ln)
    if m:
        cur = f"{m.group(1)}:{m.group(2)}"
        continue
    m = re.search(r"/\*([0-9a-f]{4,})\*/", ln)
    if m and cur:
        line_of[int(m.group(1), 16)] = cur
agg = defaultdict(float)
tot = 0.0
for a, v, s in samples:
    off = a - base
    agg[line_of.get(off, "?")] += v
    tot += v
src = {}
for nm in set(k.split(":")[0] for k in agg if k != "?"):
    import glob
    for p in glob.glob(f"/root/repo/**/{nm}", recursive=True):
        src[nm] = open(p).read().split("\n")
for k, v in sorted(agg.items(), key=lambda kv: -kv[1])[:top]:
    text = ""
    if k != "?":
        f, l = k.split(":")
        if f in src and int(l) - 1 < len(src[f]):
            text = src[f][int(l) - 1].strip()[:90]
    print(f"{100 * v / tot:5.1f}%  {k:22s} {text}")
