"""Interleaved A/B of several builds of libcszp2.so in ONE process (dev aid): every
library is loaded with its own ctypes handle, and the timed launches alternate
library by library inside each repetition, so clock/power drift over the run hits
all builds alike. Prints the median compress-kernel and decompress-kernel time per
build (CUDA events around each launch; `prep` = cszp2_compress_prepare, i.e.
the REL min/max pass for REL configs) and the ratio to the first build.

usage: python scripts/ab_interleave.py cfg5[,cfg3b...] lib_a.so lib_b.so ... [--reps N]
"""
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from synthetic import CONFIGS, make_field  # noqa: E402

vp, u64, i32, dbl = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int, ctypes.c_double


def load(path):
    L = ctypes.CDLL(os.path.abspath(path), mode=ctypes.RTLD_LOCAL)
    L.cszp2_compress_bound.restype = u64
    L.cszp2_compress_bound.argtypes = [u64, i32]
    L.cszp2_compress_prepare.argtypes = [vp, u64, i32, dbl, i32, vp, vp]
    L.cszp2_compress_encode.argtypes = [vp, u64, i32, dbl, i32, i32, vp, vp, vp]
    L.cszp2_compress_encode_ex.argtypes = [vp, u64, i32, dbl, i32, i32, vp, vp, ctypes.c_uint, vp]
    L.cszp2_decompress.argtypes = [vp, vp, u64, i32, vp, vp]
    return L


def main():
    args = [a for a in sys.argv[1:] if not a.startswith("--")]
    reps = 12
    if "--reps" in sys.argv:
        reps = int(sys.argv[sys.argv.index("--reps") + 1])
        args = [a for a in args if a != str(reps)]
    cfgs, libs = args[0].split(","), args[1:]
    Ls = [load(p) for p in libs]
    st = torch.cuda.current_stream()
    sp = vp(st.cuda_stream)
    for cfg in cfgs:
        spec = CONFIGS[cfg]
        x = make_field(cfg, "cuda")
        n, w = x.numel(), x.element_size()
        dt = 0 if w == 4 else 1
        lam = spec.ebs[-1]
        ebm = 1 if spec.eb_mode == "rel" else 0
        out = torch.empty(int(Ls[0].cszp2_compress_bound(n, dt)), dtype=torch.uint8, device="cuda")
        nb = torch.zeros(1, dtype=torch.int64, device="cuda")
        y = torch.empty_like(x)
        for enc, encname in ((1, "outlier"), (0, "plain")):
            te = [[] for _ in Ls]
            td = [[] for _ in Ls]
            tp = [[] for _ in Ls]
            for r in range(reps + 2):
                for k, L in enumerate(Ls):
                    ep = torch.cuda.Event(enable_timing=True)
                    ep.record(st)
                    L.cszp2_compress_prepare(vp(x.data_ptr()), n, dt, lam, ebm, vp(out.data_ptr()), sp)
                    e0, e1, e2 = (torch.cuda.Event(enable_timing=True) for _ in range(3))
                    e0.record(st)
                    # the kernel alone (FLAG_PREPARED: prepare zeroed the index); builds that
                    # predate the flag reject it (ARG) and zero the index in prepare anyway
                    if L.cszp2_compress_encode_ex(vp(x.data_ptr()), n, dt, lam, ebm, enc, vp(out.data_ptr()),
                                                  vp(nb.data_ptr()), 8, sp) == 1:
                        L.cszp2_compress_encode(vp(x.data_ptr()), n, dt, lam, ebm, enc, vp(out.data_ptr()),
                                                vp(nb.data_ptr()), sp)
                    e1.record(st)
                    L.cszp2_decompress(vp(out.data_ptr()), vp(y.data_ptr()), n, dt, None, sp)
                    e2.record(st)
                    torch.cuda.synchronize()
                    if r >= 2:
                        te[k].append(e0.elapsed_time(e1))
                        td[k].append(e1.elapsed_time(e2))
                        tp[k].append(ep.elapsed_time(e0))
            me = [float(np.median(v)) for v in te]
            md = [float(np.median(v)) for v in td]
            mp = [float(np.median(v)) for v in tp]
            for k, p in enumerate(libs):
                print(f"{cfg:6s} {encname:8s} {os.path.basename(p):14s} enc {me[k]:8.4f} ms ({me[0] / me[k]:6.4f}x)"
                      f"  dec {md[k]:8.4f} ms ({md[0] / md[k]:6.4f}x)"
                      f"  prep {mp[k]:8.4f} ms ({mp[0] / mp[k]:6.4f}x)", flush=True)
        del x, out, y
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
