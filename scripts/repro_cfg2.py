import sys, os, time
sys.path.insert(0, "/root/repo")
import torch, numpy as np
import paper_conf_sc_huangdlc24_b200 as cz
from synthetic import make_field
x = make_field("cfg2", "cuda")
for enc in ("plain", "outlier"):
    for eb in (1e-2, 1e-3, 1e-4):
        t0 = time.time()
        out, nb = cz.compress(x, eb, "rel", enc)
        torch.cuda.synchronize()
        print(enc, eb, int(nb.item()), f"{time.time()-t0:.3f}s", flush=True)
