"""Run compress (prepare+encode) and decompress a few times on one config (for ncu)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sc_huangdlc24_b200 as cz
from synthetic import CONFIGS, make_field
cfg = sys.argv[1] if len(sys.argv) > 1 else "cfg3b"
enc = sys.argv[2] if len(sys.argv) > 2 else "outlier"
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
spec = CONFIGS[cfg]
x = make_field(cfg, "cuda")
out = torch.empty(cz.compress_bound(x.numel(), x.dtype), dtype=torch.uint8, device="cuda")
nb = torch.zeros(1, dtype=torch.int64, device="cuda")
y = torch.empty_like(x)
for _ in range(reps):
    cz.compress(x, spec.ebs[-1], spec.eb_mode, enc, out=out, out_bytes=nb)
    cz.decompress(out, x.numel(), x.dtype, out=y)
torch.cuda.synchronize()
print("done", int(nb.item()))
