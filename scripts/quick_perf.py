"""Quick device-timed throughput of the three kernels on a config (dev aid)."""
import sys, os, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sc_huangdlc24_b200 as cz
from synthetic import CONFIGS, make_field

def timeit(fn, reps=10):
    for _ in range(3): fn()
    s, e = torch.cuda.Event(True), torch.cuda.Event(True)
    torch.cuda.synchronize(); s.record()
    for _ in range(reps): fn()
    e.record(); torch.cuda.synchronize()
    return s.elapsed_time(e) / reps * 1e-3

for cfg in sys.argv[1:]:
    spec = CONFIGS[cfg]
    x = make_field(cfg, "cuda")
    n = x.numel(); w = x.element_size()
    out = torch.empty(cz.compress_bound(n, x.dtype), dtype=torch.uint8, device="cuda")
    nb = torch.zeros(1, dtype=torch.int64, device="cuda")
    y = torch.empty_like(x)
    lam = spec.ebs[-1]
    for enc in ("plain", "outlier"):
        cz.compress(x, lam, spec.eb_mode, enc, out=out, out_bytes=nb)
        torch.cuda.synchronize()
        total = int(nb.item()); cr = n * w / total
        t_prep = timeit(lambda: cz.compress_prepare(x, lam, spec.eb_mode, out))
        def pe():
            cz.compress_prepare(x, lam, spec.eb_mode, out)
            cz.compress_encode(x, lam, spec.eb_mode, enc, out, nb)
        t_enc = timeit(pe) - t_prep  # encode needs a fresh ticket from prepare
        t_all = timeit(lambda: cz.compress(x, lam, spec.eb_mode, enc, out=out, out_bytes=nb))
        t_dec = timeit(lambda: cz.decompress(out, n, x.dtype, out=y))
        GB = n * w / 1e9
        print(f"{cfg} {enc:8s} CR={cr:6.2f} prep={t_prep*1e6:8.1f}us enc={t_enc*1e6:8.1f}us "
              f"comp_e2e={GB/t_all:7.1f}GB/s enc_only={GB/t_enc:7.1f}GB/s "
              f"enc_roof={(n*w+total)/t_enc/1e9:7.1f}GB/s dec={GB/t_dec:7.1f}GB/s dec_roof={(n*w+total)/t_dec/1e9:7.1f}GB/s", flush=True)
    del x, out, y; torch.cuda.empty_cache()
