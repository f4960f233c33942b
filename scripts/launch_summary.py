"""Markdown summary of the ncu launch list of the bench command (dev aid):
    python scripts/launch_summary.py gpurun_out/launches_<tag>.csv <out.md> <title>
The first 4 x (warmup + steps) launches are the headline workload's steps (zero_scratch,
minmax, compress, decompress); they are summarised per kernel (count, mean duration,
DRAM bytes per launch, share of the step), plus the totals of every later launch."""
import csv
import sys
from collections import OrderedDict, defaultdict

path, out, title = sys.argv[1], sys.argv[2], sys.argv[3]
rows = list(csv.reader(open(path)))
hi = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
H = rows[hi]
I, K, G, M, V = (H.index(x) for x in ("ID", "Kernel Name", "Grid Size", "Metric Name", "Metric Value"))
launches = OrderedDict()
for r in rows[hi + 1:]:
    if len(r) <= V:
        continue
    d = launches.setdefault(r[I], {"kernel": r[K].split("(")[0].split("<")[0].replace("void ", "").split("::")[-1],
                                   "grid": r[G]})
    d[r[M]] = float(r[V].replace(",", ""))


def unit_ok(d):
    return "gpu__time_duration.sum" in d


L = [d for d in launches.values() if unit_ok(d)]
first = L[:24]  # 3 warm-up + 3 timed steps x (zero_scratch, minmax, compress, decompress)
agg = defaultdict(lambda: {"n": 0, "t": 0.0, "r": 0.0, "w": 0.0, "grid": ""})
for d in first:
    a = agg[d["kernel"]]
    a["n"] += 1
    a["t"] += d["gpu__time_duration.sum"]
    a["r"] += d.get("dram__bytes_read.sum", 0.0)
    a["w"] += d.get("dram__bytes_write.sum", 0.0)
    a["grid"] = d["grid"]
tot = sum(a["t"] for a in agg.values())
with open(out, "w") as f:
    f.write(f"# {title}\n\n")
    f.write("ncu `--metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none` "
            "over `python bench.py --steps 3 --warmup 3 ...` (scripts/profile_r02.sh). Cold-cache, serialised "
            "launches: the per-kernel SHARE of the step is what compares with the bench, not the absolute times. "
            "Headline workload (config 5, 2048^3 f32, REL 1e-4, Outlier): its first 24 launches.\n\n")
    f.write("| kernel | grid | launches | mean ms | DRAM read GB / launch | DRAM write GB / launch | share of step |\n")
    f.write("|---|---|---|---|---|---|---|\n")
    for k, a in sorted(agg.items(), key=lambda kv: -kv[1]["t"]):
        n = a["n"]
        f.write(f"| {k} | {a['grid']} | {n} | {a['t'] / n / 1e6:.4f} | {a['r'] / n / 1e9:.3f} | {a['w'] / n / 1e9:.3f} "
                f"| {a['t'] / tot:.3f} |\n")
    f.write(f"\nAll launches in the list: {len(L)} (the rest: plain-mode, ABS-mode, e2e and the per-config sweep).\n")
print(open(out).read())
