import sys, os
sys.path.insert(0, os.getcwd())
import torch
import paper_conf_sc_huangdlc24_b200 as cz
from synthetic import CONFIGS, make_field
cfg = sys.argv[1]
spec = CONFIGS[cfg]
x = make_field(cfg, "cuda").view(spec.shape)
out = torch.empty(cz.compress_bound_nd(x.shape, x.dtype), dtype=torch.uint8, device="cuda")
nb = torch.zeros(1, dtype=torch.int64, device="cuda")
y = torch.empty_like(x)
for _ in range(3):
    cz.compress_nd(x, 1e-4, "rel", "outlier", out=out, out_bytes=nb)
    cz.decompress_nd(out, x.shape, x.dtype, out=y)
torch.cuda.synchronize()
print("ok", int(nb.item()))
