"""A/B device timing of several builds of libcszp2.so (dev aid, not a bench line).

usage: python scripts/ab_libs.py cfg5,cfg3b,cfg4a lib_a.so lib_b.so ...
Each lib runs in its own process (CSZP2_LIB); per config and encoding mode it prints
the compress-kernel (encode only, CUDA events around each launch) and
decompress-kernel times, alternating libs over two rounds to expose box noise.
"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CHILD = r"""
import sys, os, json
sys.path.insert(0, os.environ["ROOT"])
import torch
import paper_conf_sc_huangdlc24_b200 as cz
from synthetic import CONFIGS, make_field
res = {}
for cfg in sys.argv[1].split(","):
    name, _, lg = cfg.partition("@")  # cfg5@24: the first 2^24 values of cfg5's field (L2-resident)
    spec = CONFIGS[name]
    x = make_field(name, "cuda", count=(1 << int(lg)) if lg else None)
    n, w = x.numel(), x.element_size()
    out = torch.empty(cz.compress_bound(n, x.dtype), dtype=torch.uint8, device="cuda")
    nb = torch.zeros(1, dtype=torch.int64, device="cuda")
    y = torch.empty_like(x)
    lam = spec.ebs[-1]
    for enc in ("outlier", "plain"):
        te, td, tp = [], [], []
        for it in range(8):
            s0, e0 = torch.cuda.Event(True), torch.cuda.Event(True)
            s0.record(); cz.compress_prepare(x, lam, spec.eb_mode, out); e0.record()
            s, e = torch.cuda.Event(True), torch.cuda.Event(True)
            s.record(); cz.compress_encode(x, lam, spec.eb_mode, enc, out, nb); e.record()
            s2, e2 = torch.cuda.Event(True), torch.cuda.Event(True)
            s2.record(); cz.decompress(out, n, x.dtype, out=y); e2.record()
            torch.cuda.synchronize()
            if it >= 3:
                te.append(s.elapsed_time(e)); td.append(s2.elapsed_time(e2)); tp.append(s0.elapsed_time(e0))
        tot = int(nb.item())
        te.sort(); td.sort(); tp.sort()
        res[f"{cfg}/{enc}"] = dict(prep_gbs=round(n * w / tp[len(tp)//2] / 1e6, 1), cr=round(n * w / tot, 2), enc_ms=te[len(te)//2], dec_ms=td[len(td)//2],
                                   enc_gbs=round((n * w + tot) / te[len(te)//2] / 1e6, 1),
                                   dec_gbs=round((n * w + tot) / td[len(td)//2] / 1e6, 1))
    del x, out, y
    torch.cuda.empty_cache()
print("RESULT " + json.dumps(res))
"""


def main():
    cfgs, libs = sys.argv[1], sys.argv[2:]
    allres = {lib: [] for lib in libs}
    for rnd in range(2):
        for lib in libs:
            env = dict(os.environ, CSZP2_LIB=os.path.abspath(lib), ROOT=ROOT)
            p = subprocess.run([sys.executable, "-c", CHILD, cfgs], env=env, capture_output=True, text=True)
            line = [l for l in p.stdout.splitlines() if l.startswith("RESULT ")]
            if not line:
                print(lib, "FAILED", p.stderr[-2000:])
                continue
            r = json.loads(line[0][7:])
            allres[lib].append(r)
            for k, v in r.items():
                print(f"round {rnd} {os.path.basename(lib):24s} {k:14s} CR {v['cr']:6.2f} enc {v['enc_ms']:8.3f} ms "
                      f"({v['enc_gbs']:7.1f} GB/s alg)  dec {v['dec_ms']:8.3f} ms ({v['dec_gbs']:7.1f} GB/s alg)", flush=True)
    json.dump(allres, open(os.path.join(ROOT, "gpurun_out", "ab_libs.json"), "w"), indent=1)


if __name__ == "__main__":
    main()
