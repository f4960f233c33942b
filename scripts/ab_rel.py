"""A/B of the REL compression pipeline (min/max pass + compress kernel) across library
builds, L2 flushed (256 MiB write) before each step, CUDA events (dev aid).
usage: python scripts/ab_rel.py cfg3a,cfg4a lib_a.so lib_b.so ..."""
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
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for cfg in sys.argv[1].split(","):
    spec = CONFIGS[cfg]
    x = make_field(cfg, "cuda")
    n, w = x.numel(), x.element_size()
    out = torch.empty(cz.compress_bound(n, x.dtype), dtype=torch.uint8, device="cuda")
    nb = torch.zeros(1, dtype=torch.int64, device="cuda")
    lam = spec.ebs[-1]
    for enc in ("outlier", "plain"):
        tp, te = [], []
        for it in range(12):
            flush.zero_(); torch.cuda._sleep(400_000)
            a, b, c = (torch.cuda.Event(True) for _ in range(3))
            a.record(); cz.compress_prepare(x, lam, spec.eb_mode, out); b.record()
            cz.compress_encode(x, lam, spec.eb_mode, enc, out, nb, prepared=True); c.record()
            torch.cuda.synchronize()
            if it >= 3:
                tp.append(a.elapsed_time(b)); te.append(b.elapsed_time(c))
        tp.sort(); te.sort()
        tot = int(nb.item())
        res[f"{cfg}/{enc}"] = dict(prep=tp[len(tp)//2], enc=te[len(te)//2], frac=(n*w+tot)/(te[len(te)//2]*1e-3)/6531e9)
    del x, out
    torch.cuda.empty_cache()
print("RESULT " + json.dumps(res))
"""
cfgs, libs = sys.argv[1], sys.argv[2:]
allres = {l: [] for l in libs}
for rnd in range(2):
    for l in (libs if rnd == 0 else libs[::-1]):
        env = dict(os.environ, CSZP2_LIB=os.path.abspath(l), ROOT=ROOT)
        p = subprocess.run([sys.executable, "-c", CHILD, cfgs], capture_output=True, text=True, env=env)
        line = [x for x in p.stdout.splitlines() if x.startswith("RESULT ")]
        if not line:
            print(l, p.stderr[-1500:]); continue
        allres[l].append(json.loads(line[0][7:]))
for key in allres[libs[0]][0]:
    for l in libs:
        rs = [r[key] for r in allres[l]]
        print(f"{key:16s} {os.path.basename(l):12s} prep {min(r['prep'] for r in rs):8.4f} ms  "
              f"enc {min(r['enc'] for r in rs):8.4f} ms  kernel frac {max(r['frac'] for r in rs):.3f}", flush=True)
