"""NEXT rows measured on B200: (#2) decoupled lookback vs plain chained scan
(the paper's Fig 17 comparison), TMA vs per-thread vector vs scalar
loads (the §VI-E memory ablation), persisted tile index vs the paper's
decompression-side lookback (R-14), and (#1) random-access decompression
(P:345-356). Prints one JSON object; timings with CUDA events after warm-up."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sc_huangdlc24_b200 as cz
from synthetic import CONFIGS, make_field


def timeit(fn, reps=10):
    for _ in range(3):
        fn()
    s, e = torch.cuda.Event(True), torch.cuda.Event(True)
    torch.cuda.synchronize(); s.record()
    for _ in range(reps):
        fn()
    e.record(); torch.cuda.synchronize()
    return s.elapsed_time(e) / reps * 1e-3


res = {}
for cfg in sys.argv[1:] or ["cfg3b", "cfg5"]:
    spec = CONFIGS[cfg]
    x = make_field(cfg, "cuda"); n = x.numel(); w = x.element_size()
    out = torch.empty(cz.compress_bound(n, x.dtype), dtype=torch.uint8, device="cuda")
    nb = torch.zeros(1, dtype=torch.int64, device="cuda")
    lam = spec.ebs[-1]
    r = {}
    t_prep = timeit(lambda: cz.compress_prepare(x, lam, spec.eb_mode, out))
    for name, flags in (("decoupled_lookback", 0), ("chained_scan", cz.FLAG_CHAINED_SCAN),
                        ("load_vec16_per_thread", cz.FLAG_LOAD_VEC), ("load_scalar_per_thread", cz.FLAG_LOAD_SCALAR)):
        def run():
            cz.compress_prepare(x, lam, spec.eb_mode, out)
            cz.compress_encode_ex(x, lam, spec.eb_mode, "outlier", out, nb, flags=flags)
        t = timeit(run, 5) - t_prep
        torch.cuda.synchronize()
        total = int(nb.item())
        r[name] = {"compress_kernel_ms": round(t * 1e3, 4), "gbs_uncompressed": round(n * w / t / 1e9, 1),
                   "roofline_gbs": round((n * w + total) / t / 1e9, 1)}
    r["lookback_speedup"] = round(r["chained_scan"]["compress_kernel_ms"] / r["decoupled_lookback"]["compress_kernel_ms"], 2)
    r["tma_vs_vec_speedup"] = round(r["load_vec16_per_thread"]["compress_kernel_ms"] / r["decoupled_lookback"]["compress_kernel_ms"], 2)
    r["tma_vs_scalar_speedup"] = round(r["load_scalar_per_thread"]["compress_kernel_ms"] / r["decoupled_lookback"]["compress_kernel_ms"], 2)
    # random access on the Outlier stream
    cz.compress(x, lam, spec.eb_mode, "outlier", out=out, out_bytes=nb)
    y = torch.empty(1 << 20, dtype=x.dtype, device="cuda")
    ra = {}
    for count in (32, 8192, 1 << 20):
        first = (n // 2) // 32 * 32 + 7
        t = timeit(lambda: cz.decompress_range(out, n, first, count, x.dtype, out=y[:count]), 50)
        ra[f"{count}_values"] = {"us": round(t * 1e6, 2), "gbs": round(count * w / t / 1e9, 2)}
    yfull = torch.empty_like(x)
    t = timeit(lambda: cz.decompress(out, n, x.dtype, out=yfull), 5)
    ra["full_decompress_gbs"] = round(n * w / t / 1e9, 1)
    scr = torch.empty(int(cz._lib.cszp2_decompress_scratch_bytes(n)), dtype=torch.uint8, device="cuda")
    t_lb = timeit(lambda: cz.decompress_tilewise(out, n, x.dtype, cz.LOCATE_LOOKBACK, out=yfull, scratch=scr), 5)
    t_ix = timeit(lambda: cz.decompress_tilewise(out, n, x.dtype, cz.LOCATE_INDEX, out=yfull, scratch=scr), 5)
    r["decompress_locate"] = {
        "persisted_index_persistent_kernel_gbs": ra["full_decompress_gbs"],
        "persisted_index_cta_per_tile_gbs": round(n * w / t_ix / 1e9, 1),
        "decompression_lookback_cta_per_tile_gbs": round(n * w / t_lb / 1e9, 1)}
    r["random_access"] = ra
    res[cfg] = r
    del x, out, yfull; torch.cuda.empty_cache()
print(json.dumps(res))
