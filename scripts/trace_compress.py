"""Per-tile timeline of the compression kernel (debug build libcszp2_trace.so)."""
import sys, os, ctypes
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from synthetic import CONFIGS, make_field
lib = ctypes.CDLL(os.environ.get("CSZP2_TRACE_LIB", os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "paper_conf_sc_huangdlc24_b200", "libcszp2_trace.so")))
vp, u64, i32, dbl = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int, ctypes.c_double
lib.cszp2_compress.argtypes = [vp, u64, i32, dbl, i32, i32, vp, vp, vp]
lib.cszp2_compress_bound.argtypes = [u64, i32]; lib.cszp2_compress_bound.restype = u64
lib.cszp2_debug_set_trace.argtypes = [vp]
for arg in sys.argv[1:]:
    cfg, _, mode = arg.partition(":")
    enc = 0 if mode == "plain" else 1
    spec = CONFIGS[cfg]
    x = make_field(cfg, "cuda"); n = x.numel()
    T = -(-(-(-n // 32)) // 256)
    out = torch.empty(lib.cszp2_compress_bound(n, 0), dtype=torch.uint8, device="cuda")
    tr = torch.zeros(T * 16, dtype=torch.int64, device="cuda")
    lib.cszp2_debug_set_trace(ctypes.c_void_p(tr.data_ptr()))
    st = torch.cuda.current_stream().cuda_stream
    for rep in range(3):
        tr.zero_()
        lib.cszp2_compress(ctypes.c_void_p(x.data_ptr()), n, 0, spec.ebs[-1], 1, enc, ctypes.c_void_p(out.data_ptr()), None, ctypes.c_void_p(st))
        torch.cuda.synchronize()
    a = tr.view(T, 16).cpu().numpy().astype(np.int64)
    t0 = a[:, 0][a[:, 0] > 0].min()
    a[:, :5] -= t0
    a[:, 6] -= t0
    a[:, 8] -= t0
    a[:, 9] -= t0
    claim, data, pub, res, staged, polls, rstart = [a[:, i] for i in range(7)]
    moves = np.zeros_like(polls)
    print(f"== {cfg}: T={T} span={(res.max())/1e3:.1f}us rate={T/(res.max()/1e3):.1f} tiles/us")
    copied_ = a[:, 9]
    print(f"ramp/tail: first data {data[data>0].min()/1e3:.2f}us, first pubA {pub.min()/1e3:.2f}us, "
          f"1st-wave (first 444 tiles) resolved by {np.max(res[:min(T,444)])/1e3:.2f}us, "
          f"10%/50%/90%/100% of tiles resolved at " + "/".join(f"{np.percentile(res, p)/1e3:.2f}" for p in (10, 50, 90, 100))
          + f"us, last copy {copied_.max()/1e3:.2f}us, last claim {claim.max()/1e3:.2f}us")
    def q(v): return " ".join(f"{np.percentile(v,p):7.2f}" for p in (5,25,50,75,95,99))
    print("pct                5      25      50      75      95      99  (us)")
    print("claim->data   ", q((data-claim)/1e3))
    print("data->pubA    ", q((pub-data)/1e3))
    print("pubA->staged  ", q((staged-pub)/1e3))
    print("pubA->resolved", q((res[1:]-pub[1:])/1e3))
    print("staged->rstart", q((rstart[1:]-staged[1:])/1e3))
    print("rstart->resolved", q((res[1:]-rstart[1:])/1e3))
    issued, copied = a[:, 8], a[:, 9]
    print("rstart->issued", q((issued[1:]-rstart[1:])/1e3))
    print("issued->resolved", q((res[1:]-issued[1:])/1e3))
    print("resolved->copied", q((copied[1:]-res[1:])/1e3))
    print("claim->resolved", q((res[1:]-claim[1:])/1e3))
    windows = 1 + (polls >> 32)
    polls = polls & 0xFFFFFFFF
    print("polls mean", polls.mean(), "max", polls.max(), "windows mean", windows.mean(), "pct", q(windows))
    # distance from a tile to the previous tile of the same CTA (slot 7 = CTA id)
    cta_ = a[:, 7]
    o = np.lexsort((np.arange(T), cta_))
    same = cta_[o][1:] == cta_[o][:-1]
    dist = (o[1:] - o[:-1])[same]
    print("distance to the same CTA's previous tile", q(dist))
    # frontier: resolved time vs tile index; claim order vs time
    order = np.argsort(claim)
    print("claims per us (median over 10us windows):", np.median(np.diff(np.searchsorted(np.sort(claim), np.arange(0, claim.max(), 10000))))/10)
    # lag between claim of tile t and resolve of tile t: grows?
    for frac in (0.1, 0.3, 0.5, 0.7, 0.9):
        i = int(frac * T); sl = slice(i, i + 200)
        print(f" tiles@{frac:.1f}: claim->res {np.median(res[sl]-claim[sl])/1e3:7.2f}us  claim-gap to prev tile claim {np.median(np.diff(claim[sl]))/1e3:6.3f}us  polls {polls[sl].mean():.2f}")
    del x, out, tr; torch.cuda.empty_cache()
    # per-CTA timelines (slot 7 = CTA id)
    cta = a[:, 7]
    per = []
    waits = []; comp = []; stg = []
    for c in np.unique(cta)[:300]:
        idx = np.where(cta == c)[0]
        idx = idx[np.argsort(data[idx])]
        if len(idx) < 3: continue
        d, p_, s_ = data[idx], pub[idx], staged[idx]
        per.append(np.median(np.diff(d)))
        waits.append(np.median(d[1:] - s_[:-1])); comp.append(np.median(p_ - d)); stg.append(np.median(s_ - p_))
    print(f"per-CTA period {np.median(per)/1e3:.2f}us  staged->next data {np.median(waits)/1e3:.2f}us  compute {np.median(comp)/1e3:.2f}us  staging {np.median(stg)/1e3:.2f}us")
    w = np.array([x for x in waits])
    print("staged->next data pct", q(w/1e3))
    # tails: per CTA, consecutive data arrivals; where do the long gaps come from?
    gaps = []; parts = []
    for c in np.unique(cta):
        idx = np.where(cta == c)[0]
        idx = idx[np.argsort(data[idx])]
        if len(idx) < 3: continue
        g = np.diff(data[idx])
        gaps.append(g)
        # for tile k+1: claim(k+1) - data(k), data(k+1) - claim(k+1), staged(k) - data(k)
        parts.append(np.stack([g, claim[idx][1:] - data[idx][:-1], data[idx][1:] - claim[idx][1:],
                               staged[idx][:-1] - data[idx][:-1]], 1))
    G = np.concatenate(gaps); Pm = np.concatenate(parts)
    print(f"period mean {G.mean()/1e3:.3f}us median {np.median(G)/1e3:.3f}us  pct", q(G/1e3))
    big = Pm[:, 0] > 2 * np.median(G)
    print(f"long gaps (>2x median): {big.mean()*100:.2f}% of tiles, {Pm[big,0].sum()/G.sum()*100:.1f}% of time; "
          f"mean [gap, data->claim(next), claim->data(next), data->staged] = {np.round(Pm[big].mean(0)/1e3, 2)} us")
    print(f"all tiles mean [gap, data->claim(next), claim->data(next), data->staged] = {np.round(Pm.mean(0)/1e3, 2)} us")
