#!/usr/bin/env python
"""Benchmark of the cuSZp2 hot path on B200 (BASELINE.json metric).

Workload (default): BASELINE config 5 — the 2048^3 f32 NYX-shaped synthetic
field (32 GiB), REL 1e-4, Outlier-FLE, slab-sharded across the ranks (strong
scaling: the field is fixed, each of N ranks owns 2^33/N values). One step =
one pass of the whole hot path: REL resolve (memset + device min/max) →
fused compression kernel → [N>1: NCCL all-gather of the per-rank compressed
sizes + container index kernel] → fused decompression kernel.

value = round-trip throughput: uncompressed bytes of the whole field ÷ (max
over ranks of the device time of compress + decompress), GB/s. comp_gbs and
decomp_gbs give the two directions separately (same clock).

Launch: python bench.py [--gpus N --steps K --warmup W] (torchrun for N>1);
        python bench.py --impl reference  → the CPU oracle on host cores.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import subprocess
import sys
import threading
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from synthetic import CONFIGS, make_field  # noqa: E402

METRIC = "comp/decomp end-to-end GB/s per B200 & at 2/4/8 GPUs; CR and PSNR at REL 1e-4"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="cfg5")
    ap.add_argument("--enc", default="outlier", choices=["plain", "outlier"])
    ap.add_argument("--eb", type=float, default=None)
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--e2e-max-gib", type=float, default=32.0,
                    help="cap on the per-rank slab used for the host-buffer e2e leg (pinned host "
                         "memory per rank is ~2x this plus the stream)")
    ap.add_argument("--cpu-sample-log2", type=int, default=28,
                    help="values in the oracle cpu_baseline sample (2^k)")
    ap.add_argument("--no-plain", action="store_true", help="skip the secondary Plain-mode pass")
    ap.add_argument("--no-configs", action="store_true",
                    help="skip the per-config sweep (BASELINE configs 1-4, both modes, both directions)")
    ap.add_argument("--config-steps", type=int, default=20, help="timed steps per sweep entry")
    ap.add_argument("--launcher-selftest", action="store_true",
                    help="(tests) start the ranks like a real run, join a gloo group, report the world and exit")
    ap.add_argument("--rel-scope", default="rank", choices=["rank", "global"],
                    help="REL range per rank's slab (default; no extra collective) or of the whole "
                         "field (one 16-byte NCCL all-reduce of (min, -max); SURVEY 8(e))")
    return ap.parse_args()


# ----------------------------------------------------------------- helpers

def dist_env():
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


def load_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            p = json.load(f)
        return float(p["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


class ClockSampler:
    """nvidia-smi clocks + throttle reasons during the timed region."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index: int, period_ms: int = 50):
        self.gpu = gpu_index
        self.period_ms = period_ms
        self.proc = None
        self.raw = []

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", f"--id={self.gpu}", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                 "-lms", str(self.period_ms)], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
            # nvidia-smi takes a few hundred ms to start: wait for its first sample, so
            # the timed region (often < 1 s) is covered, and keep only samples taken
            # between entry and exit
            deadline = time.monotonic() + 5.0
            while not self.raw and time.monotonic() < deadline and self.proc.poll() is None:
                time.sleep(0.01)
        except Exception:
            self.proc = None
        self.t_in = time.monotonic()
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.raw.append((time.monotonic(), line.strip()))

    def __exit__(self, *a):
        self.t_out = time.monotonic()
        if self.proc:
            time.sleep(0.06)  # the sample in flight at exit still belongs to the region
            self.proc.terminate()
            try:
                self.proc.wait(timeout=2)
            except Exception:
                self.proc.kill()

    @property
    def lines(self):
        t_out = getattr(self, "t_out", float("inf")) + 0.06
        return [l for t, l in self.raw if self.t_in <= t <= t_out]

    def window(self, t0, t1):
        """summary() of the samples taken in [t0, t1] (time.monotonic())."""
        return self.summary([l for t, l in self.raw if t0 <= t <= t1 + 0.06])

    def summary(self, lines=None):
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for l in (self.lines if lines is None else lines):
            f = [x.strip() for x in l.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                mx = float(f[2])
            except ValueError:
                continue
            for nm, v in zip(names, f[5:9]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"], "samples": 0}
        return {"sm_mhz": float(np.median(sm)), "sm_max_mhz": mx, "reasons": sorted(reasons),
                "samples": len(sm)}


def traffic_from_profiles(kernel_key: str, cfg: str = "cfg5", enc: str = "outlier"):
    """dram read+write bytes per launch of `kernel_key` on (cfg, enc), from the
    committed ncu --set full captures (profiles/ncu_traffic.json, written by
    scripts/ncu_traffic.py); None when no capture of that workload is committed."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return d.get(f"{cfg}/{enc}/{kernel_key}", {}).get("dram_bytes")
    except Exception:
        return None


def workload_config(args, spec, lam, world, n_total, values_per_rank):
    """The `config` object of both arms (the reference arm times a sample of it)."""
    return {"workload": f"{args.config}: {spec.name} {spec.dtype} field, REL {lam:g}, "
                        f"{args.enc}-FLE, slab-sharded over {world} rank(s)",
            "n_values": n_total, "values_per_rank": values_per_rank, "eb_mode": spec.eb_mode,
            "eb": lam, "enc_mode": args.enc,
            "l2": "inputs larger than L2 (field >> 126 MB); no flush needed",
            "rel_scope": args.rel_scope,
            "parallelism": f"slab x{world}, NCCL all-gather of compressed sizes"
                           + (" + all-reduce of the value range"
                              if args.rel_scope == "global" and spec.eb_mode == "rel" else "")}


# ----------------------------------------------------------------- reference arm (CPU oracle)

def run_reference(args):
    rank, world, _ = dist_env()
    if rank != 0:
        return 0
    if "WORLD_SIZE" not in os.environ:
        world = args.gpus  # the same workload description as our arm at --gpus N
    import oracle

    spec = CONFIGS[args.config]
    lam = args.eb if args.eb is not None else spec.ebs[-1]
    enc = oracle.OUTLIER if args.enc == "outlier" else oracle.PLAIN
    ebm = oracle.REL if spec.eb_mode == "rel" else oracle.ABS
    torch.set_num_threads(os.cpu_count() or 1)
    sample = 1 << 24
    x = make_field(args.config, "cpu", 0, sample).numpy()
    w = x.itemsize
    for _ in range(args.warmup):
        s, _ = oracle.compress(x, lam, ebm, enc)
        oracle.decompress(s, x.size, x.dtype)
    tc = td = 0.0
    for _ in range(args.steps):
        t0 = time.perf_counter()
        s, rc = oracle.compress(x, lam, ebm, enc)
        t1 = time.perf_counter()
        y, rc2 = oracle.decompress(s, x.size, x.dtype)
        t2 = time.perf_counter()
        tc += t1 - t0
        td += t2 - t1
    gb = x.nbytes * args.steps / 1e9
    value = gb / (tc + td)
    desc = (f"first 2^24 values ({x.nbytes/2**20:.0f} MiB) of the {spec.name} field per step, "
            f"single-threaded C oracle, REL {lam:g} {args.enc}")
    line = {
        "impl": "reference", "metric": METRIC, "value": round(value, 4), "unit": "GB/s",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": round((tc + td) / args.steps * 1e3, 3), "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "f32" if w == 4 else "f64",
        "data": "synthetic",
        # rank 0's slab size, computed here (this arm loads nothing of the product)
        "config": workload_config(args, spec, lam, world, spec.n,
                                  min(spec.n, -(-(-(-spec.n // world)) // 32) * 32)),
        "reference_sample_values": sample,
        "comp_gbs": round(gb / tc, 4), "decomp_gbs": round(gb / td, 4),
        "cr": round(x.nbytes / s.size, 3),
        "cpu_baseline": {"value": round(value, 4), "unit": "GB/s", "cores": 1, "kind": "oracle",
                         "sample": desc},
        "e2e": {"value": round(value, 4), "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


# ----------------------------------------------------------------- our arm

def relaunch_under_torchrun(args) -> int:
    """`python bench.py --gpus N` without a torchrun environment: start the N ranks
    ourselves (one process per GPU, NCCL over 127.0.0.1) with the same arguments and
    return their exit code; rank 0 prints the JSON line."""
    import socket

    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__), *sys.argv[1:]]
    env = dict(os.environ, BENCH_SELF_LAUNCHED="1")
    return subprocess.call(cmd, env=env)


def launcher_selftest(args) -> int:
    """The multi-rank plumbing of a real run without GPUs (tests/test_bench_launch.py):
    every rank joins a gloo group over the torchrun environment and all-gathers its
    rank; rank 0 prints what the group saw."""
    import torch.distributed as dist

    rank, world, local = dist_env()
    dist.init_process_group("gloo")
    got = [None] * world
    dist.all_gather_object(got, {"rank": rank, "local_rank": local, "pid": os.getpid()})
    t = torch.tensor([float(rank + 1)])
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    if rank == 0:
        print(json.dumps({"n_gpus": world, "gpus_arg": args.gpus, "ranks": got, "max_over_ranks": t.item(),
                          "self_launched": os.environ.get("BENCH_SELF_LAUNCHED") == "1"}), flush=True)
    dist.destroy_process_group()
    return 0


def main():
    args = parse()
    if args.gpus < 1:
        raise SystemExit("--gpus must be >= 1")
    if args.launcher_selftest:
        if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
            return relaunch_under_torchrun(args)
        return launcher_selftest(args)
    if args.impl == "reference":
        return run_reference(args)  # rank 0 only; needs no process group
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        return relaunch_under_torchrun(args)

    import paper_conf_sc_huangdlc24_b200 as cz
    from paper_conf_sc_huangdlc24_b200.multi import reduce_range, slab

    rank, world, local = dist_env()
    if world != args.gpus and world > 1:
        print(f"warning: WORLD_SIZE={world} != --gpus {args.gpus}", file=sys.stderr)
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    dist = None
    if world > 1:
        import torch.distributed as dist

        dist.init_process_group("nccl", device_id=dev)

    spec = CONFIGS[args.config]
    lam = args.eb if args.eb is not None else spec.ebs[-1]
    n_total = spec.n
    s0, cnt = slab(n_total, world, rank)
    w = spec.itemsize
    dtype = spec.dtype

    x = make_field(args.config, dev, start=s0, count=cnt)
    bound = cz.compress_bound(cnt, dtype)
    out = torch.empty(bound, dtype=torch.uint8, device=dev)
    nbytes = torch.zeros(1, dtype=torch.int64, device=dev)
    y = torch.empty_like(x)
    sizes = torch.zeros(world, dtype=torch.int64, device=dev)
    offsets = torch.zeros(world + 1, dtype=torch.int64, device=dev)
    stream = torch.cuda.current_stream(dev)

    glob = args.rel_scope == "global" and spec.eb_mode == "rel"
    rng_work = torch.empty(8, dtype=torch.float64, device=dev)

    def step(evs=None, enc=args.enc):
        if evs:
            evs[0].record(stream)
        if glob:  # value range -> 16-byte all-reduce -> eb_abs from the global range
            cz.value_range(x, work=rng_work, stream=stream)
            cz.compress_prepare_range(x, lam, reduce_range(rng_work), out, stream=stream)
        else:
            cz.compress_prepare(x, lam, spec.eb_mode, out, stream=stream)
        if evs:
            evs[1].record(stream)
        cz.compress_encode(x, lam, spec.eb_mode, enc, out, nbytes, stream=stream, prepared=True)
        if evs:
            evs[2].record(stream)
        if world > 1:
            dist.all_gather_into_tensor(sizes, nbytes)
            cz.container_index(sizes, out=offsets, stream=stream)
        if evs:
            evs[3].record(stream)
        cz.decompress(out, cnt, dtype, out=y, stream=stream)
        if evs:
            evs[4].record(stream)

    for _ in range(max(3, args.warmup)):
        step()
    torch.cuda.synchronize()

    evs = [[torch.cuda.Event(enable_timing=True) for _ in range(5)] for _ in range(args.steps)]
    t_start, t_end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    if dist:
        dist.barrier()
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        t_start.record(stream)
        for k in range(args.steps):
            step(evs[k])
        t_end.record(stream)
        torch.cuda.synchronize()
    if dist:
        dist.barrier()
    total_ms = t_start.elapsed_time(t_end)
    ph = np.array([[e[i].elapsed_time(e[i + 1]) for i in range(4)] for e in evs])  # ms
    prep_ms, enc_ms, gather_ms, dec_ms = ph.mean(axis=0)
    comp_ms = prep_ms + enc_ms + gather_ms
    stream_bytes = int(nbytes.item())
    # per-step spread (median and min next to the mean), this rank
    comp_steps, dec_steps = ph[:, 0] + ph[:, 1] + ph[:, 2], ph[:, 3]
    spread = {"comp_ms_median": round(float(np.median(comp_steps)), 4), "comp_ms_min": round(float(comp_steps.min()), 4),
              "decomp_ms_median": round(float(np.median(dec_steps)), 4), "decomp_ms_min": round(float(dec_steps.min()), 4)}

    # max over ranks of every timing (device clocks), sum of stream bytes
    vec = torch.tensor([total_ms, comp_ms, dec_ms, prep_ms, enc_ms, gather_ms], dtype=torch.float64, device=dev)
    sb = torch.tensor([stream_bytes], dtype=torch.int64, device=dev)
    if dist:
        dist.all_reduce(vec, op=dist.ReduceOp.MAX)
        dist.all_reduce(sb, op=dist.ReduceOp.SUM)
    total_ms, comp_ms, dec_ms, prep_ms, enc_ms, gather_ms = vec.tolist()
    stream_total = int(sb.item())

    # CR + PSNR of the whole field (after the timed region; PSNR per reading R-16)
    hdr = cz.read_header(out)
    mse_sum = torch.zeros(1, dtype=torch.float64, device=dev)
    mn = torch.full((1,), float("inf"), dtype=torch.float64, device=dev)
    mx = torch.full((1,), -float("inf"), dtype=torch.float64, device=dev)
    for c0 in range(0, cnt, 1 << 28):
        xs, ys = x[c0:c0 + (1 << 28)].double(), y[c0:c0 + (1 << 28)].double()
        mse_sum += ((xs - ys) ** 2).sum()
        mn = torch.minimum(mn, xs.min().view(1))
        mx = torch.maximum(mx, xs.max().view(1))
        del xs, ys
    if dist:
        dist.all_reduce(mse_sum)
        dist.all_reduce(mn, op=dist.ReduceOp.MIN)
        dist.all_reduce(mx, op=dist.ReduceOp.MAX)
    mse = float(mse_sum.item()) / n_total
    rng_v = float(mx.item() - mn.item())
    psnr = 20 * math.log10(rng_v) - 10 * math.log10(mse) if mse > 0 else float("inf")

    gb_field = n_total * w / 1e9
    value = gb_field / ((comp_ms + dec_ms) * 1e-3)
    comp_gbs = gb_field / (comp_ms * 1e-3)
    decomp_gbs = gb_field / (dec_ms * 1e-3)

    # roofline of the dominant kernel (per rank, algorithmic bytes / avg duration)
    peak, peak_src = load_peaks()
    slab_bytes = cnt * w
    enc_bytes = slab_bytes + stream_bytes           # read field, write stream
    dec_bytes = stream_bytes + slab_bytes           # read stream, write field
    kern = {
        "compress_kernel": {"ms": enc_ms, "bytes": enc_bytes},
        "decompress_kernel": {"ms": dec_ms, "bytes": dec_bytes},
        "minmax_kernel": {"ms": prep_ms, "bytes": slab_bytes},
    }
    for k, v in kern.items():
        v["gbs"] = v["bytes"] / (v["ms"] * 1e-3) / 1e9
        v["frac"] = v["gbs"] / peak
    dom = max(("compress_kernel", "decompress_kernel"), key=lambda k: kern[k]["ms"])
    roof = {"bound": "hbm", "kernel": dom, "achieved": round(kern[dom]["gbs"], 1), "peak": peak,
            "unit": "GB/s", "frac": round(kern[dom]["frac"], 4),
            "traffic": traffic_from_profiles(dom, args.config, args.enc), "peak_source": peak_src,
            "algorithmic_bytes_per_launch": kern[dom]["bytes"],
            "kernels": {k: {"ms": round(v["ms"], 4), "gbs": round(v["gbs"], 1), "frac": round(v["frac"], 4)}
                        for k, v in kern.items()}}
    clocks = clk.summary()

    # secondary: Plain mode (both encoding modes are part of config 5)
    plain = None
    if not args.no_plain and args.enc != "plain":
        for _ in range(2):
            step(enc="plain")
        pe = [[torch.cuda.Event(enable_timing=True) for _ in range(5)] for _ in range(3)]
        for k in range(3):
            step(pe[k], enc="plain")
        torch.cuda.synchronize()
        pp = np.array([[e[i].elapsed_time(e[i + 1]) for i in range(4)] for e in pe]).mean(axis=0)
        pv = torch.tensor([pp[0] + pp[1] + pp[2], pp[3]], dtype=torch.float64, device=dev)
        pbytes = torch.tensor([int(nbytes.item())], dtype=torch.int64, device=dev)
        if dist:
            dist.all_reduce(pv, op=dist.ReduceOp.MAX)
            dist.all_reduce(pbytes)
        plain = {"comp_gbs": round(gb_field / (pv[0].item() * 1e-3), 1),
                 "decomp_gbs": round(gb_field / (pv[1].item() * 1e-3), 1),
                 "cr": round(n_total * w / int(pbytes.item()), 3)}
        step()  # leave the main-mode stream in `out`
        torch.cuda.synchronize()

    # ABS mode with eb = the REL run's eb_abs: the same quantization without the
    # min/max pass, so the cost of REL's extra read is visible
    abs_mode = None
    if spec.eb_mode == "rel":
        eb_abs = cz.read_header(out)["eb_abs"]
        ae = [[torch.cuda.Event(enable_timing=True) for _ in range(2)] for _ in range(4)]
        for k in range(6):
            if k >= 2:
                ae[k - 2][0].record(stream)
            cz.compress(x, eb_abs, "abs", args.enc, out=out, out_bytes=nbytes, stream=stream)
            if k >= 2:
                ae[k - 2][1].record(stream)
        torch.cuda.synchronize()
        av = torch.tensor([float(np.mean([e[0].elapsed_time(e[1]) for e in ae]))], dtype=torch.float64, device=dev)
        if dist:
            dist.all_reduce(av, op=dist.ReduceOp.MAX)
        abs_mode = {"comp_gbs": round(gb_field / (av.item() * 1e-3), 1), "eb": "eb_abs of the REL run (per rank)",
                    "note": "memset + compress kernel; REL adds the min/max read (phase_ms.prepare_minmax)"}
        step()  # leave the main-mode stream in `out`
        torch.cuda.synchronize()

    # every other BASELINE config, N=1 only (configs 1-4 are single-GPU configs)
    sweep = None
    if world == 1 and not args.no_configs:
        with ClockSampler(local, period_ms=10) as sclk:
            rows = run_config_sweep(args, cz, dev, stream, peak, sclk)
        sweep = {"clocks": sclk.summary(), "entries": rows,
                 "note": "per entry: kernel-only roofline fractions (algorithmic bytes = field + stream) and "
                         "whole-direction GB/s (compress incl. the REL min/max pass), CUDA events on the "
                         "launching stream, L2 flushed before every timed direction; clocks per entry are "
                         "the nvidia-smi samples (10 ms) that fell inside it, the sweep's are above"}

    # cpu_baseline: the oracle as it stands, on a bounded sample, rank 0 at N=1 only
    cpu = cpu_mt = None
    if rank == 0 and world == 1:
        cpu = run_cpu_baseline(args, x, lam, spec)
        cpu_mt = run_cpu_baseline_all_cores(args, x, lam, spec)

    # e2e through the host-buffer C-ABI calls (pinned host memory, copies timed)
    e2e = run_e2e(args, cz, x, y, out, dev, stream, lam, spec, dist, world, n_total, w)

    if rank == 0:
        line = {
            "metric": METRIC, "value": round(value, 2), "unit": "GB/s", "n_gpus": world,
            "steps": args.steps, "warmup": max(3, args.warmup),
            "ms_per_step": round(total_ms / args.steps, 4), "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None,
            "dtype": "f32" if w == 4 else "f64", "data": "synthetic",
            "config": workload_config(args, spec, lam, world, n_total, cnt),
            "comp_gbs": round(comp_gbs, 1), "decomp_gbs": round(decomp_gbs, 1),
            "cr": round(n_total * w / stream_total, 3), "psnr_db": round(psnr, 3),
            "eb_abs_rank0": hdr["eb_abs"],
            "phase_ms": {"prepare_minmax": round(prep_ms, 4), "compress_kernel": round(enc_ms, 4),
                         "allgather_index": round(gather_ms, 4), "decompress_kernel": round(dec_ms, 4)},
            "step_spread_rank0": spread,
            "abs_mode": abs_mode,
            "roofline": roof,
            "cpu_baseline": cpu,
            "cpu_baseline_all_cores": cpu_mt,
            "e2e": e2e,
            "clocks": clocks,
            # our kernels per step: prepare = zero_scratch (+ minmax for REL; global REL: minmax +
            # zero_scratch + eb_from_range), compress, decompress (+ container index at N > 1)
            "gpu_launches": args.steps * ((3 if glob else (2 if spec.eb_mode == "rel" else 1)) + 2
                                          + (1 if world > 1 else 0)),
            "plain_mode": plain,
            "configs": sweep,
        }
        print(json.dumps(line), flush=True)
    if dist:
        dist.barrier()
        dist.destroy_process_group()
    return 0


SWEEP = ("cfg1", "cfg2", "cfg3a", "cfg3b", "cfg4a", "cfg4b")


def field_quality(x, y, eb_abs, chunk=1 << 27):
    """PSNR (R-16), max|x - x'| / eb_abs, values outside BASELINE's strict slack
    eb(1+2^-20) (f32) / eb(1+2^-40) (f64), and the R-10 bound on every value."""
    f32 = x.dtype == torch.float32
    slack, rnd = (1 + 2.0 ** -20, 2.0 ** -21) if f32 else (1 + 2.0 ** -40, 2.0 ** -50)
    mse = 0.0
    mx_err = 0.0
    strict = 0
    ok = True
    mn, mxv = math.inf, -math.inf
    for c in range(0, x.numel(), chunk):
        a, b = x[c:c + chunk].double(), y[c:c + chunk].double()
        e = (a - b).abs()
        mse += float((e * e).sum())
        mx_err = max(mx_err, float(e.max()))
        strict += int((e > eb_abs * slack).sum())
        ok &= bool((e <= eb_abs * slack + rnd * torch.maximum(a.abs(), b.abs())).all())
        mn, mxv = min(mn, float(a.min())), max(mxv, float(a.max()))
    mse /= x.numel()
    psnr = 20 * math.log10(mxv - mn) - 10 * math.log10(mse) if mse > 0 and mxv > mn else float("inf")
    return {"psnr_db": round(psnr, 3), "max_err_over_eb": round(mx_err / eb_abs, 6),
            "strict_slack_violations": strict, "bound_ok": ok}


def run_config_sweep(args, cz, dev, stream, peak, clk):
    """Every other BASELINE config on one GPU (BASELINE.md "Output"):
    config x REL bound x encoding mode, both directions, device-timed with CUDA events
    on the launching stream, L2 flushed (a 256 MiB write) before every timed
    direction, since configs 1-3a fit in the 126 MB L2, and a device spin before each
    step so that host launch latency never shows up between the events."""
    rows = []
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    for cfg in SWEEP:
        spec = CONFIGS[cfg]
        x = make_field(cfg, dev)
        n, w = x.numel(), x.element_size()
        out = torch.empty(cz.compress_bound(n, x.dtype), dtype=torch.uint8, device=dev)
        nbytes = torch.zeros(1, dtype=torch.int64, device=dev)
        y = torch.empty_like(x)
        for eb in spec.ebs:
            for enc in ("plain", "outlier"):
                K = args.config_steps
                ev = [[torch.cuda.Event(enable_timing=True) for _ in range(5)] for _ in range(K)]
                for k in range(3 + K):  # 3 untimed warm-up steps
                    e = ev[k - 3] if k >= 3 else None
                    flush.zero_()
                    # ~0.2 ms device spin: the host enqueues the whole step before the GPU
                    # reaches e[0], so the events time the kernels back to back, not the
                    # host's launch latency (which exceeds a small config's kernel time)
                    torch.cuda._sleep(400_000)
                    if e: e[0].record(stream)
                    cz.compress_prepare(x, eb, spec.eb_mode, out, stream=stream)
                    if e: e[1].record(stream)
                    cz.compress_encode(x, eb, spec.eb_mode, enc, out, nbytes, stream=stream, prepared=True)
                    if e: e[2].record(stream)
                    flush.zero_()
                    if e: e[3].record(stream)
                    cz.decompress(out, n, x.dtype, out=y, stream=stream)
                    if e: e[4].record(stream)
                    if k == 2:
                        torch.cuda.synchronize()
                        t0 = time.monotonic()
                torch.cuda.synchronize()
                t1 = time.monotonic()
                ph = np.array([[e[0].elapsed_time(e[1]), e[1].elapsed_time(e[2]), e[3].elapsed_time(e[4])]
                               for e in ev])
                prep, enc_ms, dec_ms = ph.mean(axis=0)
                total = int(nbytes.item())
                eb_abs = cz.read_header(out, stream)["eb_abs"]
                gb = n * w / 1e9
                kb = n * w + total  # algorithmic bytes of either kernel: field + stream
                q = field_quality(x, y, eb_abs)
                rows.append({
                    "config": cfg, "field": spec.name, "n": n, "dtype": "f32" if w == 4 else "f64",
                    "eb_mode": spec.eb_mode, "eb": eb, "eb_abs": eb_abs, "enc_mode": enc,
                    "cr": round(n * w / total, 3), **q,
                    "comp_gbs": round(gb / ((prep + enc_ms) * 1e-3), 1),
                    "decomp_gbs": round(gb / (dec_ms * 1e-3), 1),
                    "prepare_ms": round(prep, 4), "compress_kernel_ms": round(enc_ms, 4),
                    "decompress_kernel_ms": round(dec_ms, 4),
                    "roofline": {
                        "bound": "hbm", "peak": peak, "unit": "GB/s",
                        "compress_kernel": {"achieved": round(kb / (enc_ms * 1e-3) / 1e9, 1),
                                            "frac": round(kb / (enc_ms * 1e-3) / 1e9 / peak, 4),
                                            "algorithmic_bytes": kb,
                                            "traffic": traffic_from_profiles("compress_kernel", cfg, enc)},
                        "decompress_kernel": {"achieved": round(kb / (dec_ms * 1e-3) / 1e9, 1),
                                              "frac": round(kb / (dec_ms * 1e-3) / 1e9 / peak, 4),
                                              "algorithmic_bytes": kb,
                                              "traffic": traffic_from_profiles("decompress_kernel", cfg, enc)},
                    },
                    "steps": K, "clocks": clk.window(t0, t1),
                })
        del x, out, y
        torch.cuda.empty_cache()
    return rows


def run_e2e(args, cz, x, y, out, dev, stream, lam, spec, dist, world, n_total, w):
    """Same metric through cszp2_compress_host / cszp2_decompress_host: every
    step copies its input from pinned host memory and its result back. Reuses
    the device buffers of the main run (x's contents are consumed)."""
    cap = int(args.e2e_max_gib * 2**30 // w) // 32 * 32
    m = min(x.numel(), cap)
    h_in = torch.empty(m, dtype=x.dtype, pin_memory=True)
    h_in.copy_(x[:m])
    # the stream's size, from one device compression of the same values (deterministic),
    # sizes the pinned stream buffer (the compress bound would pin ~the input size again)
    nb_dev = torch.zeros(1, dtype=torch.int64, device=dev)
    cz.compress(x[:m], lam, spec.eb_mode, args.enc, out=out, out_bytes=nb_dev, stream=stream)
    torch.cuda.synchronize()
    d_in, d_out, d_y = y[:m], out, x[:m]  # work buffers (caller-owned, FORMAT.md-sized)
    h_out = torch.empty(int(nb_dev.item()) + (1 << 16), dtype=torch.uint8, pin_memory=True)
    h_y = torch.empty(m, dtype=x.dtype, pin_memory=True)
    st = torch.zeros(1, dtype=torch.int32, device=dev)
    nbytes = cz.compress_host(h_in, lam, spec.eb_mode, args.enc, d_in, d_out, h_out, stream)  # warm-up
    cz.decompress_host(h_out, nbytes, d_out, d_y, h_y, status=st, stream=stream)
    tc = td = 0.0
    for _ in range(args.e2e_steps):
        if dist:
            dist.barrier()
        torch.cuda.synchronize()
        e0, e1, e2 = (torch.cuda.Event(enable_timing=True) for _ in range(3))
        e0.record(stream)
        nbytes = cz.compress_host(h_in, lam, spec.eb_mode, args.enc, d_in, d_out, h_out, stream)
        e1.record(stream)
        cz.decompress_host(h_out, nbytes, d_out, d_y, h_y, status=st, stream=stream)
        e2.record(stream)
        torch.cuda.synchronize()
        tc += e0.elapsed_time(e1)
        td += e1.elapsed_time(e2)
    v = torch.tensor([tc / args.e2e_steps, td / args.e2e_steps], dtype=torch.float64, device=dev)
    mm = torch.tensor([m], dtype=torch.int64, device=dev)
    if dist:
        dist.all_reduce(v, op=dist.ReduceOp.MAX)
        dist.all_reduce(mm)
    tcm, tdm = v.tolist()
    gb = int(mm.item()) * w / 1e9
    # sanity: the host result honours the bound on a prefix (full parity is in tests/)
    k = min(m, 1 << 22)
    eb_abs = cz.read_header(d_out, stream)["eb_abs"]
    a, b = h_in[:k].double(), h_y[:k].double()
    okb = bool(((a - b).abs() <= eb_abs * (1 + 2.0 ** -20) + 2.0 ** -21 * torch.maximum(a.abs(), b.abs())).all())
    res = {"value": round(gb / ((tcm + tdm) * 1e-3), 2), "unit": "GB/s",
           "comp_gbs": round(gb / (tcm * 1e-3), 2), "decomp_gbs": round(gb / (tdm * 1e-3), 2),
           "h2d_bytes_per_step": m * w + nbytes, "d2h_bytes_per_step": nbytes + m * w,
           "values_per_rank": m, "status_ok": int(st.item()) == 0, "bound_ok_prefix": okb,
           "api": "cszp2_compress_host + cszp2_decompress_host (pinned host buffers)"}
    if m < x.numel():
        res["sample"] = f"first {m} values of each rank's slab (--e2e-max-gib {args.e2e_max_gib})"
    del h_in, h_out, h_y
    return res


def cpu_model():
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return None


def run_cpu_baseline(args, x, lam, spec):
    import oracle

    m = min(x.numel(), 1 << args.cpu_sample_log2)
    xs = x[:m].cpu().numpy()
    ebm = oracle.REL if spec.eb_mode == "rel" else oracle.ABS
    enc = oracle.OUTLIER if args.enc == "outlier" else oracle.PLAIN
    # pinned to one core for the single-threaded run, restored afterwards
    try:
        aff = os.sched_getaffinity(0)
        os.sched_setaffinity(0, {max(aff)})
    except (AttributeError, OSError):
        aff = None
    try:
        t0 = time.perf_counter()
        s, rc = oracle.compress(xs, lam, ebm, enc)
        t1 = time.perf_counter()
        yh, rc2 = oracle.decompress(s, m, xs.dtype)
        t2 = time.perf_counter()
    finally:
        if aff:
            os.sched_setaffinity(0, aff)
    gb = xs.nbytes / 1e9
    return {"value": round(gb / (t2 - t0), 4), "unit": "GB/s", "cores": 1, "kind": "oracle",
            "cpu": cpu_model(), "pinned": aff is not None,
            "comp_gbs": round(gb / (t1 - t0), 4), "decomp_gbs": round(gb / (t2 - t1), 4),
            "seconds": round(t2 - t0, 2),
            "sample": f"first {m} values ({xs.nbytes / 2**30:.2f} GiB) of the rank-0 slab, one "
                      f"compress + decompress, single-threaded C oracle (REL range of the sample)"}


def run_cpu_baseline_all_cores(args, x, lam, spec):
    """SURVEY §8(d)'s second CPU baseline: the same oracle over block-aligned chunks of
    the same sample on every host core (ctypes releases the GIL; one thread per core):
    the REL range of the sample (one oracle pass), then per-chunk compress and
    decompress in parallel. Chunk streams are separate (no serial concatenation)."""
    import concurrent.futures as cf

    import oracle

    m = min(x.numel(), 1 << args.cpu_sample_log2)
    xs = x[:m].cpu().numpy()
    cores = os.cpu_count() or 1
    enc = oracle.OUTLIER if args.enc == "outlier" else oracle.PLAIN
    ebm = oracle.REL if spec.eb_mode == "rel" else oracle.ABS
    step = -(-m // cores)
    step = -(-step // 8192) * 8192
    chunks = [xs[i:i + step] for i in range(0, m, step)]
    with cf.ThreadPoolExecutor(max_workers=cores) as ex:
        t0 = time.perf_counter()
        eb_abs = oracle.resolve_eb(xs, lam, ebm)
        streams = list(ex.map(lambda c: oracle.compress(c, eb_abs, oracle.ABS, enc)[0], chunks))
        t1 = time.perf_counter()
        list(ex.map(lambda a: oracle.decompress(a[0], a[1].size, a[1].dtype), zip(streams, chunks)))
        t2 = time.perf_counter()
    gb = xs.nbytes / 1e9
    return {"value": round(gb / (t2 - t0), 4), "unit": "GB/s", "cores": min(cores, len(chunks)),
            "kind": "oracle", "cpu": cpu_model(), "comp_gbs": round(gb / (t1 - t0), 4), "decomp_gbs": round(gb / (t2 - t1), 4),
            "seconds": round(t2 - t0, 2),
            "sample": f"the cpu_baseline sample in {len(chunks)} block-aligned chunks, one oracle "
                      f"thread per core (REL range by one serial oracle pass)"}


if __name__ == "__main__":
    sys.exit(main())
