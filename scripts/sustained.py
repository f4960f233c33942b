"""Sustained compress-kernel loop on one config with nvidia-smi clocks/power sampling (dev aid).
usage: CSZP2_LIB=... python scripts/sustained.py cfg5 [seconds]"""
import sys, os, subprocess, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sc_huangdlc24_b200 as cz
from synthetic import CONFIGS, make_field
cfg = sys.argv[1]; secs = float(sys.argv[2]) if len(sys.argv) > 2 else 3.0
spec = CONFIGS[cfg]
x = make_field(cfg, "cuda"); n = x.numel()
out = torch.empty(cz.compress_bound(n, x.dtype), dtype=torch.uint8, device="cuda")
nb = torch.zeros(1, dtype=torch.int64, device="cuda")
lam = spec.ebs[-1]
cz.compress_prepare(x, lam, spec.eb_mode, out); torch.cuda.synchronize()
smi = subprocess.Popen(["nvidia-smi", "--query-gpu=clocks.sm,clocks.mem,power.draw,clocks_throttle_reasons.active",
                        "--format=csv,noheader", "-lms", "200"], stdout=subprocess.PIPE, text=True)
t0 = time.time(); times = []
while time.time() - t0 < secs:
    cz.compress_prepare(x, lam, spec.eb_mode, out)
    s, e = torch.cuda.Event(True), torch.cuda.Event(True)
    s.record(); cz.compress_encode(x, lam, spec.eb_mode, "outlier", out, nb); e.record()
    torch.cuda.synchronize(); times.append(s.elapsed_time(e))
smi.terminate(); lines = smi.stdout.read().strip().splitlines()
times.sort()
print(os.path.basename(os.environ.get("CSZP2_LIB", "inplace")), cfg, "iters", len(times), "enc ms min/med/max %.3f %.3f %.3f" % (times[0], times[len(times)//2], times[-1]))
for l in lines[::max(1, len(lines)//8)]: print("   smi:", l)
