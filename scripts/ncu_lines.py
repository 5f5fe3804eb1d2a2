"""Per-source-line view of one kernel in an ncu report: warp-stall samples (by
reason) and L2 theoretical sectors, joined from the SASS source page and the
line table of the cubin (build with -lineinfo).  Dev aid.

usage: python scripts/ncu_lines.py <report.ncu-rep> <kernel-regex> <cubin> [mangled-substring] [top]
(extract cubins with `cuobjdump -xelf all libtsmv.so`)"""
import csv
import io
import re
import subprocess
import sys
from collections import defaultdict

rep, kre, cubin = sys.argv[1], sys.argv[2], sys.argv[3]
sel = sys.argv[4] if len(sys.argv) > 4 else ""
top = int(sys.argv[5]) if len(sys.argv) > 5 else 40
raw = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass", "-k", f"regex:{kre}"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
hi = next(i for i, r in enumerate(rows) if r and r[0] == "Address")
h = rows[hi]
col = {n: i for i, n in enumerate(h)}
reasons = [n for n in h if n.startswith("stall_") and "Not Issued" not in n]
ins = []
for r in rows[hi + 1:]:
    if not r or not r[0].startswith("0x"):
        if ins:
            break
        continue
    ins.append(r)
base = int(ins[0][0], 16)
dis = subprocess.run(["nvdisasm", "-g", "-c", cubin], capture_output=True, text=True).stdout
secs = re.split(r"\n\s*\.section\s+\.text\.|\n\s*\.text\.", dis)
best = None
for f in secs:
    head = f.split("\n", 1)[0]
    if re.search(kre, head) and sel in head and (best is None or len(f) > len(best)):
        best = f
assert best is not None, "kernel not found in cubin"
line_of, cur = {}, None
for ln in best.split("\n"):
    m = re.search(r'//## File ".*?/([^/"]+)", line (\d+)', ln)
    if m:
        cur = f"{m.group(1)}:{m.group(2)}"
        continue
    m = re.search(r"/\*([0-9a-f]{4,})\*/", ln)
    if m and cur:
        line_of[int(m.group(1), 16)] = cur
agg = defaultdict(lambda: defaultdict(float))
for r in ins:
    key = line_of.get(int(r[0], 16) - base, "?")
    d = agg[key]
    d["samples"] += float(r[col["Warp Stall Sampling (All Samples)"]] or 0)
    d["l2sect"] += float(r[col["L2 Theoretical Sectors Global"]] or 0)
    d["inst"] += float(r[col["Instructions Executed"]] or 0)
    for rs in reasons:
        d[rs] += float(r[col[rs]] or 0)
tot = sum(d["samples"] for d in agg.values())
totl2 = sum(d["l2sect"] for d in agg.values())
src = {}
import glob
for k in agg:
    if k != "?":
        nm = k.split(":")[0]
        if nm not in src:
            ps = glob.glob(f"/root/repo/**/{nm}", recursive=True)
            src[nm] = open(ps[0]).read().split("\n") if ps else []
print(f"total stall samples {tot:.0f}, L2 theoretical sectors {totl2:.0f}")
for k, d in sorted(agg.items(), key=lambda kv: -kv[1]["samples"])[:top]:
    text = ""
    if k != "?":
        f, l = k.split(":")
        if int(l) - 1 < len(src.get(f, [])):
            text = src[f][int(l) - 1].strip()[:70]
    rs = sorted(((d[r], r[6:]) for r in reasons), reverse=True)[:2]
    rtxt = " ".join(f"{n}:{100 * v / max(d['samples'], 1):.0f}%" for v, n in rs if v)
    print(f"{100 * d['samples'] / tot:5.1f}% {d['l2sect']:9.0f}s {k:20s} {rtxt:28s} {text}")
