"""One-off calibration of synthetic noise amplitudes.

Prints the Outlier/Plain-mode CR of each config's field (or a contiguous slab of
it) at REL 1e-4 using the CPU oracle. Paper targets (Table III):
CESM 14.97, HACC 4.84, NYX 24.12.
"""
import sys, os, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle
from synthetic import CONFIGS, make_field
from dataclasses import replace

def cr(name, count=None, **params):
    spec = CONFIGS[name]
    if params:
        spec = replace(spec, params={**spec.params, **params})
    x = make_field(spec, "cpu", 0, count).numpy()
    out = {}
    for mode, m in (("O", oracle.OUTLIER), ("P", oracle.PLAIN)):
        s, rc = oracle.compress(x, 1e-4, oracle.REL, m)
        out[mode] = x.nbytes / s.size
    return out

if __name__ == "__main__":
    torch.set_num_threads(8)
    args = sys.argv[1:]
    name = args[0]; count = int(float(args[1])) if len(args) > 1 and args[1] != "-" else None
    kv = {a.split("=")[0]: float(a.split("=")[1]) for a in args[2:]}
    t = time.time(); print(name, kv, cr(name, count, **kv), f"{time.time()-t:.1f}s")
