"""Table VI analog: 1D (L=32) vs 2D 8x8 / 3D 4x4x4 Lorenzo (L=64) on the
2D/3D-shaped configs — compression ratio and device-timed kernel throughput, Outlier
mode, REL 1e-4. Writes one JSON object per (config, predictor) to stdout: whole
compression (REL min/max + kernel) and decompression GB/s of uncompressed data, and
kernel-only roofline fractions (compression re-run in ABS mode at the resolved eb_abs,
so only the stream-header zeroing precedes the kernel; algorithmic bytes = field +
stream; peak = MEASURED_PEAKS.json hbm_gbs), with the nvidia-smi clocks of each entry."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import time  # noqa: E402

import paper_conf_sc_huangdlc24_b200 as cz  # noqa: E402
from bench import ClockSampler, load_peaks  # noqa: E402
from synthetic import CONFIGS, make_field  # noqa: E402


def timeit(fn, reps=10):
    for _ in range(3):
        fn()
    s, e = torch.cuda.Event(True), torch.cuda.Event(True)
    torch.cuda.synchronize()
    s.record()
    for _ in range(reps):
        fn()
    e.record()
    torch.cuda.synchronize()
    return s.elapsed_time(e) / reps * 1e-3


def main(cfgs):
    peak = load_peaks()[0]
    clk = ClockSampler(torch.cuda.current_device(), period_ms=10).__enter__()
    for cfg in cfgs:
        spec = CONFIGS[cfg]
        x = make_field(cfg, "cuda").view(spec.shape)
        n, w = x.numel(), x.element_size()
        lam = spec.ebs[-1]
        GB = n * w / 1e9
        for pred in ("1d", f"{x.dim()}d"):
            if pred == "1d":
                xf = x.view(-1)
                out = torch.empty(cz.compress_bound(n, x.dtype), dtype=torch.uint8, device="cuda")
                nb = torch.zeros(1, dtype=torch.int64, device="cuda")
                y = torch.empty_like(xf)
                comp = lambda: cz.compress(xf, lam, "rel", "outlier", out=out, out_bytes=nb)  # noqa: E731
                dec = lambda: cz.decompress(out, n, x.dtype, out=y)  # noqa: E731
            else:
                out = torch.empty(cz.compress_bound_nd(x.shape, x.dtype), dtype=torch.uint8, device="cuda")
                nb = torch.zeros(1, dtype=torch.int64, device="cuda")
                y = torch.empty_like(x)
                comp = lambda: cz.compress_nd(x, lam, "rel", "outlier", out=out, out_bytes=nb)  # noqa: E731
                dec = lambda: cz.decompress_nd(out, x.shape, x.dtype, out=y)  # noqa: E731
            comp()
            torch.cuda.synchronize()
            total = int(nb.item())
            eb_abs = cz.read_header(out)["eb_abs"]
            if pred == "1d":
                kern = lambda: cz.compress(xf, eb_abs, "abs", "outlier", out=out, out_bytes=nb)  # noqa: E731
            else:
                kern = lambda: cz.compress_nd(x, eb_abs, "abs", "outlier", out=out, out_bytes=nb)  # noqa: E731
            t0 = time.monotonic()
            tc, td, tk = timeit(comp), timeit(dec), timeit(kern)
            t1 = time.monotonic()
            kb = n * w + total
            dec()
            err = (y.view(-1).double() - x.view(-1).double()).abs().max().item()
            rng = (x.max() - x.min()).item()
            print(json.dumps({"config": cfg, "shape": list(spec.shape), "predictor": pred,
                              "cr": round(n * w / total, 3), "comp_GBps": round(GB / tc, 1),
                              "decomp_GBps": round(GB / td, 1),
                              "compress_kernel_frac": round(kb / tk / 1e9 / peak, 3),
                              "decompress_kernel_frac": round(kb / td / 1e9 / peak, 3), "peak_GBps": peak,
                              "max_err_over_range": err / rng, "clocks": clk.window(t0, t1)}),
                  flush=True)
            del out, y
        del x
        torch.cuda.empty_cache()
    clk.__exit__()


if __name__ == "__main__":
    main(sys.argv[1:] or ["cfg2", "cfg3a", "cfg3b"])
