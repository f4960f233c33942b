"""Run the nD (2D/3D Lorenzo) compressor and decompressor a few times on one config (for ncu)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_sc_huangdlc24_b200 as cz  # noqa: E402
from synthetic import CONFIGS, make_field  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "cfg3b"
enc = sys.argv[2] if len(sys.argv) > 2 else "outlier"
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
spec = CONFIGS[cfg]
x = make_field(cfg, "cuda").view(spec.shape)
out = torch.empty(cz.compress_bound_nd(x.shape, x.dtype), dtype=torch.uint8, device="cuda")
nb = torch.zeros(1, dtype=torch.int64, device="cuda")
y = torch.empty_like(x)
for _ in range(reps):
    cz.compress_nd(x, spec.ebs[-1], spec.eb_mode, enc, out=out, out_bytes=nb)
    cz.decompress_nd(out, x.shape, x.dtype, out=y)
torch.cuda.synchronize()
print("done", int(nb.item()))
