"""Markdown summary of source-level ncu reports (scripts/ncu_src_cfg5.sh): duration,
issue activity, pipe utilisation, stall mix, SASS opcode mix per warp-tile and the SASS
lines with the most stall samples.

usage: python scripts/ncu_src_summary.py <out.md> <title> <report.ncu-rep>:<warp-tiles> ...
(warp-tiles = tiles x 8 producer warps, e.g. 8388608 for config 5)
"""
import csv
import io
import subprocess
import sys
from collections import Counter


def ncu(rep, *a):
    return subprocess.run(["ncu", "-i", rep, *a], capture_output=True, text=True).stdout


def summarize(rep, norm):
    out = []
    rows = list(csv.reader(io.StringIO(ncu(rep, "--page", "raw", "--csv"))))
    hdr, units, vals = rows[0], rows[1], rows[2]
    get = lambda k: vals[hdr.index(k)] if k in hdr else "n/a"
    name = get("Kernel Name")
    out.append(f"### `{name}`\n")
    out.append(f"- duration {get('gpu__time_duration.sum')} {units[hdr.index('gpu__time_duration.sum')]}, "
               f"issue active {get('smsp__issue_active.avg.pct_of_peak_sustained_active')}%, "
               f"warps active {get('sm__warps_active.avg.pct_of_peak_sustained_active')}%, "
               f"{get('launch__registers_per_thread')} regs/thread")
    pipes = [(k.split("__inst_executed_pipe_")[1].split(".")[0], vals[i]) for i, k in enumerate(hdr)
             if k.startswith("sm__inst_executed_pipe_") and k.endswith(".avg.pct_of_peak_sustained_active")]
    pipes = [(p, float(v.replace(",", "") or 0)) for p, v in pipes]
    out.append("- pipe utilisation (% of peak, active cycles): " +
               ", ".join(f"{p} {v:.1f}" for p, v in sorted(pipes, key=lambda x: -x[1]) if v >= 1.0))
    stalls = [(h.split("stalled_")[1], float(vals[i].replace(",", "") or 0)) for i, h in enumerate(hdr)
              if h.startswith("smsp__pcsamp_warps_issue_stalled_") and not h.endswith("_not_issued")]
    tot = sum(v for _, v in stalls) or 1
    out.append("- stall mix (pc samples): " +
               ", ".join(f"{h} {100 * v / tot:.1f}%" for h, v in sorted(stalls, key=lambda x: -x[1])[:8]))
    src = list(csv.reader(io.StringIO(ncu(rep, "--page", "source", "--csv", "--print-source", "sass"))))
    hi = next(i for i, x in enumerate(src) if "Source" in x and "Instructions Executed" in x)
    H = src[hi]
    S, I, N = H.index("Source"), H.index("Instructions Executed"), H.index("# Samples")
    lines = [(int(x[I] or 0), int(x[N] or 0), x[S]) for x in src[hi + 1:]
             if len(x) > N and (x[I] or "0").isdigit() and (x[N] or "0").isdigit()]
    ti = sum(a for a, _, _ in lines)
    ts = sum(b for _, b, _ in lines) or 1
    c = Counter()
    for n, _, s in lines:
        op = s.split()[1] if s.startswith("@") else s.split()[0]
        c[op.split(".")[0]] += n
    out.append(f"- warp-instructions {ti:.4g} = {ti / norm:.1f} per warp-tile; opcode mix per warp-tile: " +
               ", ".join(f"{k} {v / norm:.1f}" for k, v in c.most_common(14)))
    out.append("\nSASS lines with the most stall samples (a barrier's wait is charged to the "
               "instruction after it):\n")
    out.append("| samples | executed / warp-tile | SASS |")
    out.append("|---|---|---|")
    for n, smp, s in sorted(lines, key=lambda t: -t[1])[:12]:
        out.append(f"| {100 * smp / ts:.1f}% | {n / norm:.3f} | `{s.strip()[:70]}` |")
    return "\n".join(out) + "\n"


def main():
    outp, title = sys.argv[1], sys.argv[2]
    parts = [f"# {title}\n"]
    for arg in sys.argv[3:]:
        rep, norm = arg.rsplit(":", 1)
        parts.append(summarize(rep, float(norm)))
    with open(outp, "w") as f:
        f.write("\n".join(parts))
    print(open(outp).read())


if __name__ == "__main__":
    main()
