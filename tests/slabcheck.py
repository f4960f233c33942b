"""Whole-stream parity of a GPU stream too large for one oracle call (tests only).

SURVEY §8(d)'s streaming check for config 5 (and the > 4 GiB stream test): the
field is cut into tile-aligned slabs, each slab is run through the CPU oracle on
host threads (ctypes releases the GIL), and every byte the oracle's slab stream
implies for the whole stream is compared with the GPU stream:

* block offset bytes of the slab (FORMAT.md §2 region [O, O+nb));
* the slab's payload byte range [D + e0, D + e1), e0/e1 = the GPU tile index at the
  slab's edges — block payloads are position independent (prediction
  restarts every block), so they are the oracle slab stream's payload region;
* the GPU tile index of the slab = e0 + the oracle slab stream's own index (the
  serial prefix of P:192 restarted at the slab), flags included;
* the decompressed values of the slab, bit for bit, against the oracle's
  decompression of its slab stream.

Together with the header fields and the zero pads, which the caller checks, this
covers every byte of the stream. The oracle runs with ABS and the stream's own
eb_abs, which gives the same quantization as REL with that eb_abs (FORMAT.md
§6.2: both derive inv and s from eb_abs alone); the REL eb_abs itself is checked
by the caller against the oracle's resolve_eb.
"""
from __future__ import annotations

import concurrent.futures as cf
import os
import threading

import numpy as np
import torch

import oracle
from tests import streamparse as sp

TILE = 256 * 32  # values per tile (FORMAT.md §1)


def host_workers() -> int:
    try:
        return max(1, len(os.sched_getaffinity(0)))
    except AttributeError:  # pragma: no cover
        return os.cpu_count() or 1


def rel_eb_abs(x: torch.Tensor, lam: float, chunk: int = 1 << 28) -> float:
    """The oracle's REL eb_abs of a field too large for one host copy: the exact
    (min, max) over host slabs (numpy reductions; min/max are order independent),
    then oracle_resolve_eb of the two-value array (min, max), i.e. the oracle's own
    λ·(max − min) arithmetic (R-15)."""
    mn, mx = np.inf, -np.inf
    for s in range(0, x.numel(), chunk):
        xs = x[s:s + chunk].cpu().numpy()
        ok = xs[~np.isnan(xs)]
        if ok.size:
            mn = min(mn, float(ok.min()))
            mx = max(mx, float(ok.max()))
    ends = np.array([mn, mx], dtype=np.float32 if x.dtype == torch.float32 else np.float64)
    return oracle.resolve_eb(ends, lam, oracle.REL)


def slab_parity(x: torch.Tensor, out: torch.Tensor, y: torch.Tensor, enc: int, eb_abs: float,
                slab_tiles: int = 4096, workers: int | None = None) -> dict:
    """Compare the GPU stream `out` (and decompressed `y`) of the 1D field `x`
    slab by slab with the oracle. Raises AssertionError on the first mismatch.
    Returns a summary (payload bytes, slabs, workers)."""
    n = x.numel()
    nb, T, O, D = sp.geometry(n)
    iv = np.uint32 if x.dtype == torch.float32 else np.uint64
    h = sp.header(out[:64].cpu().numpy())
    assert h["n"] == n and h["status"] == 0
    index = out[64:64 + 8 * T].cpu().numpy().view("<u8")
    assert np.all((index >> np.uint64(62)) == 2), "tile index flags"
    incl = (index & np.uint64((1 << 62) - 1)).astype(np.uint64)
    assert np.all(np.diff(incl.astype(np.int64)) >= 0)
    assert (int(incl[-1]) if T else 0) == h["payload_bytes"]
    workers = workers or min(32, host_workers())
    sem = threading.Semaphore(2 * workers)  # bounds host memory in flight
    errors = []

    def check(t0, t1, xs, ys, obytes, payload, rel_incl):
        try:
            ref, rc = oracle.compress(xs, eb_abs, oracle.ABS, enc)
            assert rc == oracle.OK, f"oracle rc {rc} on tiles [{t0},{t1})"
            rnb, rT, rO, rD = sp.geometry(xs.size)
            ridx = ref[64:64 + 8 * rT].view("<u8")
            np.testing.assert_array_equal(ridx & np.uint64((1 << 62) - 1), rel_incl,
                                          err_msg=f"tile index, tiles [{t0},{t1})")
            np.testing.assert_array_equal(ridx >> np.uint64(62), np.full(rT, 2, np.uint64))
            np.testing.assert_array_equal(obytes, ref[rO:rO + rnb], err_msg=f"offset bytes, tiles [{t0},{t1})")
            rpb = sp.header(ref)["payload_bytes"]
            assert payload.size == rpb, f"payload size {payload.size} != {rpb}, tiles [{t0},{t1})"
            np.testing.assert_array_equal(payload, ref[rD:rD + rpb], err_msg=f"payload, tiles [{t0},{t1})")
            yr, rc = oracle.decompress(ref, xs.size, xs.dtype)
            assert rc == oracle.OK
            np.testing.assert_array_equal(ys.view(iv), yr.view(iv), err_msg=f"values, tiles [{t0},{t1})")
        except AssertionError as e:  # pragma: no cover - reported below
            errors.append(e)
        finally:
            sem.release()

    slabs = 0
    with cf.ThreadPoolExecutor(max_workers=workers) as ex:
        futs = []
        for t0 in range(0, T, slab_tiles):
            if errors:
                break
            t1 = min(T, t0 + slab_tiles)
            v0, v1 = t0 * TILE, min(n, t1 * TILE)
            b0, b1 = t0 * 256, min(nb, t1 * 256)
            e0 = int(incl[t0 - 1]) if t0 else 0
            e1 = int(incl[t1 - 1])
            sem.acquire()
            xs = x[v0:v1].cpu().numpy()
            ys = y[v0:v1].cpu().numpy()
            obytes = out[O + b0:O + b1].cpu().numpy()
            payload = out[D + e0:D + e1].cpu().numpy()
            rel = incl[t0:t1] - np.uint64(e0)
            futs.append(ex.submit(check, t0, t1, xs, ys, obytes, payload, rel))
            slabs += 1
        for f in futs:
            f.result()
    if errors:
        raise errors[0]
    # pads: after the index, after the offset bytes, after the payload (FORMAT.md §2)
    pb = h["payload_bytes"]
    assert h["total_bytes"] == sp.roundup16(D + pb)
    assert not out[64 + 8 * T:O].any().item()
    assert not out[O + nb:D].any().item()
    assert not out[D + pb:h["total_bytes"]].any().item()
    return {"payload_bytes": pb, "slabs": slabs, "workers": workers, "tiles": T}
