"""Dev aid: 1D compression kernel time with the lookback window forced 32 / 256 wide
(FLAG_LB_NARROW / FLAG_LB_WIDE) on leading slabs of config 5 of 2^k values."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_sc_huangdlc24_b200 as cz  # noqa: E402
from synthetic import CONFIGS, make_field  # noqa: E402

for lg in [int(a) for a in sys.argv[1:]] or [28, 29, 30, 31]:
    n = 1 << lg
    x = make_field("cfg5", "cuda", count=n)
    out = torch.empty(cz.compress_bound(n, x.dtype), dtype=torch.uint8, device="cuda")
    nb = torch.zeros(1, dtype=torch.int64, device="cuda")
    for enc in ("outlier", "plain"):
        res = {}
        for rnd in range(2):
            for name, fl in (("narrow", cz.FLAG_LB_NARROW), ("wide", cz.FLAG_LB_WIDE)):
                ts = []
                for it in range(6):
                    cz.compress_prepare(x, 1e-4, "rel", out)
                    s, e = torch.cuda.Event(True), torch.cuda.Event(True)
                    s.record()
                    cz.compress_encode_ex(x, 1e-4, "rel", enc, out, nb, flags=fl | cz.FLAG_PREPARED)
                    e.record()
                    torch.cuda.synchronize()
                    if it >= 2:
                        ts.append(s.elapsed_time(e))
                res.setdefault(name, []).append(min(ts))
        tiles = n // 8192
        print(f"2^{lg} values ({tiles} tiles) {enc:8s} narrow {min(res['narrow']):.3f} ms  wide {min(res['wide']):.3f} ms",
              flush=True)
    del x, out
    torch.cuda.empty_cache()
