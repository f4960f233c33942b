"""Per-source-line instruction counts and stall samples of one kernel from an ncu
source-counter report (scripts/ncu_src.sh), by joining ncu's SASS page with the
line table of `nvdisasm -g` (dev aid).

usage: python scripts/ncu_by_line.py <report.ncu-rep> <lib.so> <mangled kernel name> <norm> [top]
(norm: divide counts by it, e.g. warp-tiles = tiles x 8)
"""
import collections
import csv
import io
import os
import re
import subprocess
import sys
import tempfile

rep, lib, kern, norm = sys.argv[1], sys.argv[2], sys.argv[3], float(sys.argv[4])
top = int(sys.argv[5]) if len(sys.argv) > 5 else 40
raw = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
hi = next(i for i, x in enumerate(rows) if "Source" in x and "Instructions Executed" in x)
H = rows[hi]
A, I, N = H.index("Address"), H.index("Instructions Executed"), H.index("# Samples")
sass = [(int(x[A], 16), int(x[I] or 0), int(x[N] or 0)) for x in rows[hi + 1:] if len(x) > N and x[A].startswith("0x")]
base = sass[0][0]
with tempfile.TemporaryDirectory() as d:
    subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath(lib)], cwd=d, capture_output=True)
    cub = [f for f in os.listdir(d) if f.endswith(".cubin")][0]
    dis = subprocess.run(["nvdisasm", "-g", "-c", os.path.join(d, cub)], capture_output=True, text=True).stdout
lines = dis.splitlines()
start = next(i for i, l in enumerate(lines) if l.startswith(f"{kern}:"))
loc = {}
cur = None
for l in lines[start:]:
    if l.startswith("//---------------------") and loc:
        break
    m = re.search(r'File "(.*)", line (\d+)', l)
    if m:
        cur = (os.path.basename(m.group(1)), int(m.group(2)))
        continue
    m = re.match(r"\s+/\*([0-9a-f]{4,})\*/", l)
    if m:
        loc[int(m.group(1), 16)] = cur
cnt, smp = collections.Counter(), collections.Counter()
for a, n, s in sass:
    k = loc.get(a - base)
    cnt[k] += n
    smp[k] += s
tot, ts = sum(cnt.values()), sum(smp.values()) or 1
print(f"total {tot / norm:.1f} per unit")
src = {}
for (f, ln), n in cnt.most_common(top):
    if f not in src:
        p = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                         "paper_conf_sc_huangdlc24_b200", "csrc", f)
        src[f] = open(p).read().splitlines() if os.path.exists(p) else []
    text = src[f][ln - 1].strip() if ln - 1 < len(src[f]) else ""
    print(f"{n / norm:8.1f} {100 * smp[(f, ln)] / ts:5.1f}%  {f}:{ln}  {text[:80]}")
