"""A/B device timing of the nD (2D/3D Lorenzo) kernels across libcszp2 builds (dev aid).
usage: python scripts/ab_nd.py cfg3b,cfg2 lib_a.so lib_b.so ...  (each lib in its own
process via CSZP2_LIB, two alternating rounds)"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CHILD = r"""
import sys, os, json
sys.path.insert(0, os.environ["ROOT"])
import torch, numpy as np
import paper_conf_sc_huangdlc24_b200 as cz
from synthetic import CONFIGS, make_field
res = {}
for cfg in sys.argv[1].split(","):
    spec = CONFIGS[cfg]
    x = make_field(cfg, "cuda").view(spec.shape)
    n, w = x.numel(), x.element_size()
    out = torch.empty(cz.compress_bound_nd(x.shape, x.dtype), dtype=torch.uint8, device="cuda")
    nb = torch.zeros(1, dtype=torch.int64, device="cuda")
    y = torch.empty_like(x)
    for enc in ("outlier", "plain"):
        tc, td = [], []
        for it in range(10):
            a, b, c = (torch.cuda.Event(True) for _ in range(3))
            a.record(); cz.compress_nd(x, 1e-4, "rel", enc, out=out, out_bytes=nb); b.record()
            cz.decompress_nd(out, x.shape, x.dtype, out=y); c.record()
            torch.cuda.synchronize()
            if it >= 3:
                tc.append(a.elapsed_time(b)); td.append(b.elapsed_time(c))
        tot = int(nb.item())
        res[f"{cfg}/{enc}"] = dict(cr=round(n * w / tot, 2), comp_ms=float(np.median(tc)), dec_ms=float(np.median(td)),
                                   comp_gbs=round(n * w / np.median(tc) / 1e6, 1), dec_gbs=round(n * w / np.median(td) / 1e6, 1))
    del x, out, y; torch.cuda.empty_cache()
print("RESULT " + json.dumps(res))
"""
cfgs, libs = sys.argv[1], sys.argv[2:]
allres = {l: [] for l in libs}
for rnd in range(2):
    for l in (libs if rnd == 0 else libs[::-1]):
        env = dict(os.environ, CSZP2_LIB=os.path.abspath(l), ROOT=ROOT)
        out = subprocess.run([sys.executable, "-c", CHILD, cfgs], capture_output=True, text=True, env=env)
        line = [x for x in out.stdout.splitlines() if x.startswith("RESULT ")]
        if not line:
            print(l, out.stderr[-2000:]); continue
        allres[l].append(json.loads(line[0][7:]))
for key in allres[libs[0]][0]:
    for l in libs:
        rs = [r[key] for r in allres[l]]
        cm = min(r["comp_ms"] for r in rs); dm = min(r["dec_ms"] for r in rs)
        print(f"{key:16s} {os.path.basename(l):12s} CR {rs[0]['cr']:6.2f} comp {cm:8.4f} ms  dec {dm:8.4f} ms  "
              f"(whole compress incl. REL: {rs[0]['comp_gbs']:7.1f} GB/s)", flush=True)
