"""Per-SASS-instruction execution counts of an ncu report, normalised per warp-tile
(dev aid). usage: python scripts/sass_counts.py <rep> <out.txt> [norm]"""
import csv, io, subprocess, sys
from collections import Counter
rep, outp = sys.argv[1], sys.argv[2]
norm = float(sys.argv[3]) if len(sys.argv) > 3 else 131072.0
txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
r = list(csv.reader(io.StringIO(txt)))
hi = next(i for i, x in enumerate(r) if "Source" in x and "Instructions Executed" in x)
H = r[hi]; S = H.index("Source"); I = H.index("Instructions Executed")
rows = [(int(x[I] or 0), x[S]) for x in r[hi + 1:] if len(x) > I and (x[I] or "0").isdigit()]
tot = sum(a for a, _ in rows)
with open(outp, "w") as f:
    for i, (n, s) in enumerate(rows):
        f.write(f"{i:5d} {n / norm:7.3f} {s}\n")
c = Counter()
for n, s in rows:
    op = s.split()[1] if s.startswith("@") else s.split()[0]
    c[op.split(".")[0]] += n
print(f"total {tot} warp-inst = {tot / norm:.1f} per warp-tile")
for k, v in c.most_common(25):
    print(f"  {k:12s} {v / norm:8.1f} {100 * v / tot:5.1f}%")
