"""Hot spots of an ncu --set full report (--import-source on, -lineinfo build): key
metrics, and CUDA source lines ranked by warp-stall samples with the stall mix.
usage: python scripts/ncu_hot.py <report.ncu-rep> [top]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25


def run(*a):
    return subprocess.run(["ncu", "-i", rep, *a], capture_output=True, text=True).stdout


raw = run("--page", "raw", "--csv")
rows = list(csv.reader(io.StringIO(raw)))
hdr, units, vals = rows[0], rows[1], rows[2]
want = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum", "launch__registers_per_thread",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "dram__throughput.avg.pct_of_peak_sustained_elapsed"]
for w in want:
    if w in hdr:
        i = hdr.index(w)
        print(f"{w:60s} {vals[i]} {units[i]}")
stalls = [(h, vals[i]) for i, h in enumerate(hdr) if h.startswith("smsp__pcsamp_warps_issue_stalled_") and not h.endswith("_not_issued")]
tot = sum(float(v.replace(",", "") or 0) for _, v in stalls)
print("stall mix:", ", ".join(f"{h.split('stalled_')[1]} {100*float(v.replace(',', ''))/tot:.1f}%" for h, v in
                              sorted(stalls, key=lambda x: -float(x[1].replace(',', '') or 0))[:10]))
src = run("--page", "source", "--csv", "--print-source", "cuda,sass")
r = list(csv.reader(io.StringIO(src)))
hi = next(i for i, x in enumerate(r) if x[:2] == ["Line No", "Source"] and "# Samples" in x)
H = r[hi]
N, I = H.index("# Samples"), H.index("Instructions Executed")
from collections import defaultdict
agg = defaultdict(lambda: [0, 0, ""])
text = {}
cur = None
for x in r[hi + 1:]:
    if len(x) <= N:
        continue
    if x[0]:
        cur = x[0]
        text[cur] = x[1].strip()[:100]
    try:
        n = int(x[N] or 0); ins = int(x[I] or 0)
    except ValueError:
        continue
    if cur is not None:
        agg[cur][0] += n
        agg[cur][1] += ins
T = sum(v[0] for v in agg.values()) or 1
TI = sum(v[1] for v in agg.values()) or 1
print(f"total samples {T}, warp-instructions {TI}")
for ln, (n, ins, _) in sorted(agg.items(), key=lambda kv: -kv[1][0])[:top]:
    print(f"{100*n/T:5.1f}% smp {100*ins/TI:5.1f}% ins  L{ln:>5} {text.get(ln, '')}")
