"""DRAM traffic per launch of the three hot-path kernels on each BASELINE config and
encoding mode, from one `ncu --set full` capture each (run on the GPU box):

    python scripts/ncu_traffic.py gpurun_out/ncu_traffic_<tag>.json cfg3b:outlier cfg4a:plain ...

Writes {"<cfg>/<enc>/<kernel>": {"dram_bytes": read + write, "dram_read": .., "dram_write": ..,
"duration_ns": .., "source": "ncu --set full ..."}}; bench.py reads the committed copy
(profiles/ncu_traffic.json) for `roofline.traffic`. Config 5 (96 GiB working set) is
captured with the metrics-only launch list instead (kernel replay of the full set is
impractical): scripts/gpu_profile.sh list.
"""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KERNELS = ("minmax_kernel", "compress_kernel", "decompress_kernel")


def capture(cfg, enc):
    sys.path.insert(0, ROOT)
    from synthetic import CONFIGS

    per_round = "3" if CONFIGS[cfg].eb_mode == "rel" else "2"  # ABS has no min/max launch
    rep = os.path.join("/tmp", f"traffic_{cfg}_{enc}")  # reports stay off gpurun_out (64 MiB cap)
    # prof_one: (prepare = memset + minmax, compress, decompress) x 3; skip the first round
    cmd = ["ncu", "--set", "full", "--clock-control", "none", "--kernel-name-base", "function",
           "-k", "regex:^(minmax_kernel|compress_kernel|decompress_kernel)", "-s", per_round, "-c", per_round,
           "-o", rep, "-f", sys.executable, os.path.join(ROOT, "scripts", "prof_one.py"), cfg, enc, "3"]
    subprocess.run(cmd, check=True, stdout=subprocess.DEVNULL, stderr=subprocess.STDOUT, timeout=900)
    raw = subprocess.run(["ncu", "-i", rep + ".ncu-rep", "--page", "raw", "--csv", "--print-units", "base"],
                         capture_output=True,
                         text=True, check=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, data = rows[0], rows[2:]
    res = {}
    for r in data:
        name = r[hdr.index("Kernel Name")]
        # demangled or base names: test the longer name first (it contains the shorter)
        k = next((k for k in ("decompress_kernel", "compress_kernel", "minmax_kernel") if k in name), None)
        if k is None:
            continue
        f = lambda m: float(r[hdr.index(m)].replace(",", ""))  # noqa: E731
        rd, wr = f("dram__bytes_read.sum"), f("dram__bytes_write.sum")
        res[f"{cfg}/{enc}/{k}"] = {"dram_bytes": rd + wr, "dram_read": rd, "dram_write": wr,
                                   "duration_ns": f("gpu__time_duration.sum"),
                                   "source": "ncu --set full --clock-control none, one launch (2nd round)"}
    os.remove(rep + ".ncu-rep")
    return res


def main():
    out = sys.argv[1]
    res = {}
    for item in sys.argv[2:]:
        cfg, enc = item.split(":")
        try:
            res.update(capture(cfg, enc))
        except Exception as e:  # keep the others
            print(f"{item}: {e}", file=sys.stderr)
        print(item, "done", flush=True)
    with open(out, "w") as f:
        json.dump(res, f, indent=1, sort_keys=True)


if __name__ == "__main__":
    main()
