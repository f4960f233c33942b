"""Summarise ncu captures into profiles/ (tracked): launch list CSV + --set full reports.

usage: python scripts/ncu_summary.py <tag> [--workload-note TEXT]
reads gpurun_out/launches_<tag>.csv and gpurun_out/prof_<kernel>_<tag>.ncu-rep,
writes profiles/<tag>_launches.md, profiles/<tag>_full.md and
profiles/ncu_full_summary.json (per-kernel dram bytes per launch, used by bench.py).
"""
import csv
import io
import json
import os
import subprocess
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "gpurun_out")
PROF = os.path.join(ROOT, "profiles")

KEYS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__warps_active.avg.pct_of_peak_sustained_active",
    "launch__registers_per_thread", "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem",
    "launch__grid_size", "launch__block_size", "smsp__inst_executed.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
]
STALLS = "smsp__pcsamp_warps_issue_stalled_"


def kernel_short(name):
    for k in ("decompress_kernel", "compress_kernel", "minmax_kernel", "container_index_kernel"):
        if k in name:
            return k
    return name[:40]


def launches(tag):
    p = os.path.join(OUT, f"launches_{tag}.csv")
    if not os.path.exists(p):
        return None
    lines = open(p).read().splitlines()
    start = next(i for i, l in enumerate(lines) if l.startswith('"ID"'))
    rows = list(csv.DictReader(io.StringIO("\n".join(lines[start:]))))
    per = defaultdict(lambda: defaultdict(list))
    for r in rows:
        k = kernel_short(r["Kernel Name"])
        v = float(r["Metric Value"].replace(",", ""))
        per[k][r["Metric Name"]].append((r["ID"], v))
    return per


def full(tag, kernel):
    p = os.path.join(OUT, f"prof_{kernel}_{tag}.ncu-rep")
    if not os.path.exists(p):
        return None
    txt = subprocess.check_output(["ncu", "-i", p, "--page", "raw", "--csv"], text=True, stderr=subprocess.DEVNULL)
    rows = list(csv.reader(io.StringIO(txt)))
    h, u, v = rows[0], rows[1], rows[2]
    d = {}
    for k, un, val in zip(h, u, v):
        if k in KEYS or (k.startswith(STALLS) and not k.endswith("not_issued")):
            try:
                x = float(val.replace(",", ""))
            except ValueError:
                continue
            # normalise units to bytes / ns
            scale = {"Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12, "byte": 1,
                     "us": 1e3, "ms": 1e6, "ns": 1, "s": 1e9}.get(un, 1)
            d[k] = x * scale
    return d


def main():
    tag = sys.argv[1]
    note = sys.argv[sys.argv.index("--workload-note") + 1] if "--workload-note" in sys.argv else ""
    os.makedirs(PROF, exist_ok=True)
    summary = {}
    per = launches(tag)
    if per:
        md = [f"# ncu launch list — {tag}", "", note, "",
              "`ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none`",
              "over `python bench.py --steps 3 --warmup 3 --no-plain --e2e-steps 1` (config 5, 2048^3 f32, REL 1e-4, Outlier).",
              "Cold-cache, serialised: compare each kernel's SHARE of the step with bench.py's phase_ms, not absolutes.", "",
              "| kernel | launches | mean time (ms) | share of our kernels | DRAM read / launch (GB) | DRAM write / launch (GB) |",
              "|---|---|---|---|---|---|"]
        tot = sum(sum(v for _, v in m["gpu__time_duration.sum"]) for m in per.values())
        for k, m in per.items():
            ts = [v for _, v in m["gpu__time_duration.sum"]]
            rd = [v for _, v in m.get("dram__bytes_read.sum", [])]
            wr = [v for _, v in m.get("dram__bytes_write.sum", [])]
            md.append(f"| {k} | {len(ts)} | {sum(ts)/len(ts)/1e6:.3f} | {sum(ts)/tot:.1%} | "
                      f"{(sum(rd)/len(rd) if rd else 0)/1e9:.3f} | {(sum(wr)/len(wr) if wr else 0)/1e9:.3f} |")
            summary.setdefault(k, {})["launch_list_cfg5"] = {
                "mean_ms": sum(ts) / len(ts) / 1e6, "share": sum(ts) / tot,
                "dram_read_per_launch": sum(rd) / len(rd) if rd else None,
                "dram_write_per_launch": sum(wr) / len(wr) if wr else None}
            if rd and wr:
                summary[k]["dram_bytes_per_launch"] = sum(rd) / len(rd) + sum(wr) / len(wr)
        open(os.path.join(PROF, f"{tag}_launches.md"), "w").write("\n".join(md) + "\n")
    md = [f"# ncu --set full — {tag}", "", "Captured on config 3b (512^3 f32 NYX-like, REL 1e-4, Outlier) via",
          "`ncu --set full --clock-control none --import-source on -k regex:^<kernel> -s 3 -c 1 python bench.py --config cfg3b ...`.", ""]
    for k in ("compress_kernel", "decompress_kernel", "minmax_kernel"):
        d = full(tag, k)
        if not d:
            continue
        t = d.get("gpu__time_duration.sum", 0)
        rb, wb = d.get("dram__bytes_read.sum", 0), d.get("dram__bytes_write.sum", 0)
        md += [f"## {k}", "",
               f"- duration {t/1e3:.1f} us; DRAM read {rb/1e6:.1f} MB, write {wb/1e6:.1f} MB "
               f"-> {(rb+wb)/t:.0f} GB/s",
               f"- issue active {d.get('smsp__issue_active.avg.pct_of_peak_sustained_active', 0):.1f}%, warps active "
               f"{d.get('sm__warps_active.avg.pct_of_peak_sustained_active', 0):.1f}%, "
               f"{d.get('launch__registers_per_thread', 0):.0f} regs/thread, grid {d.get('launch__grid_size', 0):.0f} x "
               f"{d.get('launch__block_size', 0):.0f}, occupancy limit regs {d.get('launch__occupancy_limit_registers', 0):.0f} / "
               f"smem {d.get('launch__occupancy_limit_shared_mem', 0):.0f} CTAs/SM",
               f"- warp-instructions executed {d.get('smsp__inst_executed.sum', 0):.3e}; smem bank conflicts "
               f"{d.get('l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum', 0):.3e}"]
        st = sorted(((kk[len(STALLS):], v) for kk, v in d.items() if kk.startswith(STALLS)), key=lambda x: -x[1])
        tot = sum(v for _, v in st) or 1
        md.append("- top stall reasons (pc samples): " + ", ".join(f"{n} {v/tot:.0%}" for n, v in st[:6]))
        md.append("")
        summary.setdefault(k, {})["full_cfg3b"] = {kk: d[kk] for kk in d if not kk.startswith(STALLS)}
    open(os.path.join(PROF, f"{tag}_full.md"), "w").write("\n".join(md) + "\n")
    json.dump(summary, open(os.path.join(PROF, "ncu_full_summary.json"), "w"), indent=1)
    print(open(os.path.join(PROF, f"{tag}_launches.md")).read() if per else "", "\n".join(md))


if __name__ == "__main__":
    main()
