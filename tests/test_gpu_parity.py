"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Bar (BASELINE.json north_star): the compressed stream is byte-identical to the
oracle's (whole stream, d_out pre-poisoned with 0xAA), the decompressed values
bit-identical. At full config sizes, sampled tiles are compared byte for byte
and properties that hold at any size (error bound, header, REL range) are
checked on every element.
"""
import math

import numpy as np
import pytest
import torch

from tests import streamparse as sp

pytestmark = pytest.mark.gpu

cuda = pytest.importorskip("torch").cuda
if not cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import oracle  # noqa: E402
import paper_conf_sc_huangdlc24_b200 as cz  # noqa: E402
from synthetic import CONFIGS, make_field  # noqa: E402

DEV = torch.device("cuda:0")
ENC = {"plain": oracle.PLAIN, "outlier": oracle.OUTLIER}
EBM = {"abs": oracle.ABS, "rel": oracle.REL}


def gpu_compress(x: torch.Tensor, eb, eb_mode, enc):
    out = torch.full((cz.compress_bound(x.numel(), x.dtype),), 0xAA, dtype=torch.uint8, device=DEV)
    nb = torch.zeros(1, dtype=torch.int64, device=DEV)
    cz.compress(x, eb, eb_mode, enc, out=out, out_bytes=nb)
    torch.cuda.synchronize()
    total = int(nb.item())
    return out, total


def check_roundtrip(xh: np.ndarray, eb, eb_mode, enc, compare_stream=True):
    x = torch.from_numpy(xh).to(DEV)
    out, total = gpu_compress(x, eb, eb_mode, enc)
    ref, rc = oracle.compress(xh, eb, EBM[eb_mode], ENC[enc])
    got = out[:total].cpu().numpy()
    h = sp.header(got)
    assert total == ref.size == h["total_bytes"]
    if rc == oracle.ERR_RANGE:
        assert h["status"] == 3
        np.testing.assert_array_equal(got[:64], ref[:64])  # parity covers the header only
        st = torch.zeros(1, dtype=torch.int32, device=DEV)
        cz.decompress(out, xh.size, x.dtype, status=st)
        torch.cuda.synchronize()
        assert int(st.item()) == 3
        return None
    assert rc == oracle.OK
    if compare_stream:
        if not np.array_equal(got, ref):
            bad = np.nonzero(got != ref)[0]
            raise AssertionError(f"stream differs at {bad.size} bytes, first {bad[:8]} (total {total})")
    st = torch.zeros(1, dtype=torch.int32, device=DEV)
    y = torch.full_like(x, float("nan"))
    cz.decompress(out, xh.size, x.dtype, out=y, status=st)
    torch.cuda.synchronize()
    assert int(st.item()) == 0
    yr, rc = oracle.decompress(ref, xh.size, xh.dtype)
    assert rc == oracle.OK
    iv = np.uint32 if xh.dtype == np.float32 else np.uint64
    np.testing.assert_array_equal(y.cpu().numpy().view(iv), yr.view(iv))
    _error_bound_all(x, y, sp.header(got)["eb_abs"])  # R-10 on every value
    return got


SIZES = [0, 1, 31, 32, 33, 1000, 8192, 8192 * 3 + 32 * 5 + 11, 100003]


@pytest.mark.parametrize("n", SIZES)
@pytest.mark.parametrize("enc", ["plain", "outlier"])
@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_small_sizes_rel(n, enc, dtype):
    rng = np.random.default_rng(n + 17)
    xh = (np.cumsum(rng.standard_normal(n)) * 0.3 + 10).astype(dtype)
    check_roundtrip(xh, 1e-3, "rel", enc)


@pytest.mark.parametrize("eb", [0.5, 1e-1, 1e-3, 1e-6])
@pytest.mark.parametrize("enc", ["plain", "outlier"])
def test_abs_bounds_noise(eb, enc):
    """Random noise: every fixed length up to ~24 bits appears."""
    rng = np.random.default_rng(int(1 / eb))
    xh = (rng.standard_normal(40000) * rng.choice([1e-3, 1.0, 100.0], 40000)).astype(np.float32)
    check_roundtrip(xh, eb, "abs", enc)


def test_ties_round_half_even():
    xh = (np.arange(-5000, 5000) + 0.5).astype(np.float32)
    got = check_roundtrip(xh, 0.5, "abs", "plain")
    np.testing.assert_array_equal(sp.parse(got)["q"], np.rint(xh).astype(np.int64))


@pytest.mark.parametrize("enc", ["plain", "outlier"])
def test_special_fields(enc):
    n = 8192 * 2 + 77
    check_roundtrip(np.zeros(n, np.float32), 1e-4, "abs", enc)            # zero blocks
    check_roundtrip(np.full(n, 5.0, np.float32), 0.5, "abs", enc)         # constant
    check_roundtrip(np.full(n, -3.25, np.float64), 1e-2, "rel", enc)      # zero range
    alt = np.where(np.arange(n) % 2 == 0, 1073741760.0, -1073741760.0).astype(np.float32)
    check_roundtrip(alt, 0.5, "abs", enc)                                 # fl = 31 everywhere
    xh = np.zeros(n, np.float32)
    xh[::97] = 1000.0                                                     # sparse spikes
    check_roundtrip(xh, 1e-3, "abs", enc)


@pytest.mark.parametrize("enc", ["plain", "outlier"])
def test_unchecked_quantizer_boundary(enc):
    """f32 blocks whose differences sit at the unchecked quantizer's cut-off (fl_p 17 vs
    18, i.e. |q| up to 32 (2^17 - 1) = 2^22 - 32 on the fast side) and ties near 2^21:
    both sides of the cut must give the oracle's bytes (kernels.cuh FAST_FL_MAX)."""
    rng = np.random.default_rng(2024)
    nblk = 600
    lim = np.array([2**16, 2**17 - 1, 2**17, 2**17 + 1, 2**18])[rng.integers(0, 5, nblk)]
    steps = rng.integers(-1, 2, (nblk, 32)) * lim[:, None]          # steps of 0, ±lim
    steps[::7] = np.abs(steps[::7])                                   # monotone ramps to ~2^22
    steps[::11] = lim[::11, None]                                     # exactly 32 lim
    q = np.cumsum(steps, axis=1).reshape(-1).astype(np.float64)
    xh = q.astype(np.float32)
    xh[::13] += 0.5                                                   # ties, even and odd
    check_roundtrip(xh, 0.5, "abs", enc)
    near = (2.0**21 + np.arange(-4000, 4000) + 0.5).astype(np.float32)  # ties near 2^21
    check_roundtrip(near, 0.5, "abs", enc)
    big = np.float32(2.0**22) + np.arange(-3000, 3000).astype(np.float32)  # |q| around 2^22
    check_roundtrip(big, 0.5, "abs", enc)
    check_roundtrip(-big, 0.5, "abs", enc)


def test_range_status_header_parity():
    xh = np.linspace(0, 1, 10000).astype(np.float32)
    xh[5000] = 3e9
    check_roundtrip(xh, 0.5, "abs", "outlier")
    xh[5000] = np.nan
    check_roundtrip(xh, 0.5, "abs", "plain")
    xh = np.array([1.0, np.inf, 2.0] * 100, np.float32)
    check_roundtrip(xh, 1e-3, "rel", "plain")  # infinite range -> RANGE


@pytest.mark.parametrize("cfg", ["cfg1", "cfg2"])
@pytest.mark.parametrize("enc", ["plain", "outlier"])
def test_configs_small_full_stream(cfg, enc):
    """BASELINE configs 1 and 2 at full size: whole-stream byte parity."""
    spec = CONFIGS[cfg]
    xh = make_field(cfg, DEV).cpu().numpy()
    for eb in spec.ebs:
        check_roundtrip(xh, eb, spec.eb_mode, enc)


def test_decompress_rejects_corrupt_streams():
    rng = np.random.default_rng(0)
    x = torch.from_numpy(np.cumsum(rng.standard_normal(50000)).astype(np.float32)).to(DEV)
    out, total = gpu_compress(x, 1e-2, "abs", "outlier")

    def status(buf, n=x.numel(), dtype=torch.float32):
        st = torch.zeros(1, dtype=torch.int32, device=DEV)
        cz.decompress(buf, n, dtype, status=st)
        torch.cuda.synchronize()
        return int(st.item())

    assert status(out) == 0
    bad = out.clone(); bad[0] ^= 1
    assert status(bad) == 4
    assert status(out, x.numel() + 1) == 4
    assert status(out, x.numel(), torch.float64) == 4
    nb, T, O, D = sp.geometry(x.numel())
    bad = out.clone(); bad[O + 3] = 0x60  # reserved bits
    assert status(bad) == 4
    bad = out.clone(); bad[64 + 8 * 2 + 7] = 0  # index flag cleared
    assert status(bad) == 4


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_random_access_ranges(dtype):
    """NEXT #1, random access: any value range decodes to exactly the
    oracle's values, touching only the tiles that cover it."""
    rng = np.random.default_rng(21)
    n = 8192 * 5 + 32 * 3 + 13
    xh = (np.cumsum(rng.standard_normal(n)) * 0.7).astype(dtype)
    x = torch.from_numpy(xh).to(DEV)
    out, total = gpu_compress(x, 1e-3, "rel", "outlier")
    ref, _ = oracle.compress(xh, 1e-3, oracle.REL, oracle.OUTLIER)
    yr, _ = oracle.decompress(ref, n, dtype)
    iv = np.uint32 if dtype == np.float32 else np.uint64
    cases = [(0, 1), (0, 32), (5, 27), (31, 2), (8191, 2), (8190, 8200), (n - 13, 13), (n - 1, 1), (0, n),
             (12345, 1000)] + [(int(a), int(rng.integers(1, 5000))) for a in rng.integers(0, n - 5000, 6)]
    for first, count in cases:
        st = torch.zeros(1, dtype=torch.int32, device=DEV)
        y = cz.decompress_range(out, n, first, count, x.dtype, status=st)
        torch.cuda.synchronize()
        assert int(st.item()) == 0
        np.testing.assert_array_equal(y.cpu().numpy().view(iv), yr[first:first + count].view(iv))
    with pytest.raises(cz.CszpError):
        cz.decompress_range(out, n, n - 1, 2, x.dtype)


@pytest.mark.parametrize("enc", ["plain", "outlier"])
def test_chained_scan_ablation_same_stream(enc):
    """NEXT #2: the chained-scan ablation must emit the identical stream."""
    rng = np.random.default_rng(4)
    xh = np.cumsum(rng.standard_normal(8192 * 40 + 77)).astype(np.float32)
    x = torch.from_numpy(xh).to(DEV)
    a, ta = gpu_compress(x, 1e-3, "rel", enc)
    b = torch.full_like(a, 0x55)
    nb = torch.zeros(1, dtype=torch.int64, device=DEV)
    cz.compress_prepare(x, 1e-3, "rel", b)
    cz.compress_encode_ex(x, 1e-3, "rel", enc, b, nb, flags=cz.FLAG_CHAINED_SCAN)
    torch.cuda.synchronize()
    assert int(nb.item()) == ta
    assert torch.equal(a[:ta], b[:ta])


def test_container_index():
    sizes = torch.tensor([100, 0, 37, 5], dtype=torch.int64, device=DEV)
    off = cz.container_index(sizes)
    assert off.cpu().tolist() == [0, 100, 100, 137, 142]


def test_host_buffer_api():
    rng = np.random.default_rng(9)
    xh = np.cumsum(rng.standard_normal(70001)).astype(np.float32)
    h_in = torch.from_numpy(xh).pin_memory()
    d_in = torch.empty(xh.size, dtype=torch.float32, device=DEV)
    d_out = torch.empty(cz.compress_bound(xh.size), dtype=torch.uint8, device=DEV)
    h_out = torch.empty(cz.compress_bound(xh.size), dtype=torch.uint8).pin_memory()
    nbytes = cz.compress_host(h_in, 1e-3, "rel", "outlier", d_in, d_out, h_out)
    ref, _ = oracle.compress(xh, 1e-3, oracle.REL, oracle.OUTLIER)
    np.testing.assert_array_equal(h_out[:nbytes].numpy(), ref)
    h_y = torch.empty(xh.size, dtype=torch.float32).pin_memory()
    st = torch.zeros(1, dtype=torch.int32, device=DEV)
    cz.decompress_host(h_out, nbytes, d_out, d_in, h_y, status=st)
    yr, _ = oracle.decompress(ref, xh.size)
    np.testing.assert_array_equal(h_y.numpy().view(np.uint32), yr.view(np.uint32))


# ---------------------------------------------------------------- full-size configs

def _error_bound_all(x, y, eb_abs, chunk=1 << 28):
    """R-10 bound on every element; also returns the number of values
    outside BASELINE's strict eb(1+2^-20) / eb(1+2^-40) slack (a diagnostic)."""
    strict = 0
    for s in range(0, x.numel(), chunk):
        xd, yd = x[s:s + chunk].double(), y[s:s + chunk].double()
        err = (xd - yd).abs()
        mag = torch.maximum(xd.abs(), yd.abs())
        if x.dtype == torch.float32:
            slack, rnd = 1 + 2.0 ** -20, 2.0 ** -21
        else:
            slack, rnd = 1 + 2.0 ** -40, 2.0 ** -50
        assert bool((err <= eb_abs * slack + rnd * mag).all())
        strict += int((err > eb_abs * slack).sum().item())
        del xd, yd, err, mag
    return strict


@pytest.mark.slow
@pytest.mark.parametrize("enc", ["plain", "outlier"])
@pytest.mark.parametrize("cfg", ["cfg3a", "cfg3b", "cfg4a", "cfg4b"])
def test_full_size_configs_whole_stream(cfg, enc):
    """BASELINE configs 3a, 3b, 4a, 4b at full size, both encoding modes: the whole
    GPU stream equals the oracle's byte for byte (d_out poisoned with 0xAA), the
    decompressed field equals the oracle's bit for bit, and REL's eb_abs is
    λ·(max − min) of torch's own reduction."""
    spec = CONFIGS[cfg]
    x = make_field(cfg, DEV)
    lam = spec.ebs[-1]
    got = check_roundtrip(x.cpu().numpy(), lam, spec.eb_mode, enc)
    assert got is not None
    h = sp.header(got)
    assert h["status"] == 0
    assert h["eb_abs"] == lam * float(x.max().double() - x.min().double())


def _big_roundtrip(x, eb, eb_mode, enc, eb_abs_expect=None, slab_tiles=4096):
    """GPU compress + decompress of a field too large for one oracle call, then
    tests/slabcheck.py's streaming whole-stream parity against the oracle."""
    from tests import slabcheck

    n = x.numel()
    out = torch.full((cz.compress_bound(n, x.dtype),), 0xAA, dtype=torch.uint8, device=DEV)
    nb = torch.zeros(1, dtype=torch.int64, device=DEV)
    cz.compress(x, eb, eb_mode, enc, out=out, out_bytes=nb)
    torch.cuda.synchronize()
    total = int(nb.item())
    h = cz.read_header(out)
    assert h["status"] == 0 and h["total_bytes"] == total and h["n"] == n
    assert h["eb_mode"] == EBM[eb_mode] and h["enc_mode"] == ENC[enc] and h["eb"] == eb
    if eb_abs_expect is not None:
        assert h["eb_abs"] == eb_abs_expect
    st = torch.zeros(1, dtype=torch.int32, device=DEV)
    y = torch.empty_like(x)
    cz.decompress(out, n, x.dtype, out=y, status=st)
    torch.cuda.synchronize()
    assert int(st.item()) == 0
    r = slabcheck.slab_parity(x, out[:total], y, ENC[enc], h["eb_abs"], slab_tiles=slab_tiles)
    strict = _error_bound_all(x, y, h["eb_abs"])
    return out, y, total, h, r, strict


@pytest.mark.slow
@pytest.mark.parametrize("enc", ["outlier", "plain"])
def test_config5_whole_stream_streamed(enc):
    """Config 5 (2048^3 f32 = 32 GiB) on one B200, both modes: every byte of the GPU
    stream and every decompressed value against the oracle, slab by slab
    (SURVEY §8(d) streaming check); REL eb_abs against the oracle's resolve of the
    field's exact range."""
    from tests import slabcheck

    free, _ = torch.cuda.mem_get_info()
    if free < 110 * 2**30:
        pytest.skip("needs ~110 GiB free device memory")
    x = make_field("cfg5", DEV)
    eb_expect = slabcheck.rel_eb_abs(x, 1e-4)
    out, y, total, h, r, strict = _big_roundtrip(x, 1e-4, "rel", enc, eb_expect)
    assert r["tiles"] == 1 << 20
    del out, y, x
    torch.cuda.empty_cache()


@pytest.mark.slow
def test_stream_larger_than_4gib():
    """A stream past 2^32 bytes (64-bit sizes and offsets everywhere;
    P:113 a single unified array): 2^31 + 8192·3 + 77 f32 noise values at a tiny ABS
    bound (fl ~ 27, ~7.6 GB of stream). Whole-stream streamed parity, tile index
    values above 2^32, and random access to values whose payload lies past 4 GiB."""
    free, _ = torch.cuda.mem_get_info()
    if free < 40 * 2**30:
        pytest.skip("needs ~40 GiB free device memory")
    n = (1 << 31) + 8192 * 3 + 77
    g = torch.Generator(device=DEV)
    g.manual_seed(0xC52000F0)
    x = torch.randn(n, generator=g, device=DEV, dtype=torch.float32).mul_(1000.0)
    out, y, total, h, r, strict = _big_roundtrip(x, 1e-5, "abs", "outlier")
    assert total > (1 << 32) + (1 << 30)
    nb, T, O, D = sp.geometry(n)
    idx = out[64:64 + 8 * T].cpu().numpy().view("<u8") & np.uint64((1 << 62) - 1)
    far = int(np.searchsorted(idx, np.uint64(1 << 32)))  # first tile ending past 4 GiB
    assert far < T - 2
    iv = np.uint32
    for first, count in [(far * 8192 + 5, 30000), (n - 100, 100), ((far + 7) * 8192 - 3, 9)]:
        st = torch.zeros(1, dtype=torch.int32, device=DEV)
        v = cz.decompress_range(out, n, first, count, x.dtype, status=st)
        torch.cuda.synchronize()
        assert int(st.item()) == 0
        np.testing.assert_array_equal(v.cpu().numpy().view(iv), y[first:first + count].cpu().numpy().view(iv))
    del out, y, x
    torch.cuda.empty_cache()


@pytest.mark.parametrize("flags", [2, 4, 3, 5])
@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_load_ablation_same_stream(flags, dtype):
    """NEXT #2: per-thread vector / scalar loads (± chained scan) give the product stream."""
    n = 7 * 8192 + 32 * 9 + 13
    xh = make_field("cfg2", DEV, 0, n).cpu().numpy().astype(dtype)
    x = torch.from_numpy(xh).to(DEV)
    ref, rc = oracle.compress(xh, 1e-4, oracle.REL, oracle.OUTLIER)
    out = torch.full((cz.compress_bound(n, x.dtype),), 0xAA, dtype=torch.uint8, device=DEV)
    nb = torch.zeros(1, dtype=torch.int64, device=DEV)
    cz.compress_prepare(x, 1e-4, "rel", out)
    cz.compress_encode_ex(x, 1e-4, "rel", "outlier", out, nb, flags=flags)
    torch.cuda.synchronize()
    assert int(nb.item()) == ref.size
    np.testing.assert_array_equal(out[: ref.size].cpu().numpy(), ref)


@pytest.mark.parametrize("locate", [0, 1])
@pytest.mark.parametrize("n", [0, 1, 8192, 5 * 8192 + 32 * 3 + 7])
@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_decompress_tilewise_ablation(n, dtype, locate):
    """NEXT #2: the paper-style decompression-side lookback decodes the same values."""
    xh = make_field("cfg2", DEV, 0, max(n, 1)).cpu().numpy().astype(dtype)[:n]
    ref, rc = oracle.compress(xh, 1e-4, oracle.REL, oracle.OUTLIER)
    yr, rc = oracle.decompress(ref, n, dtype)
    cmp = torch.from_numpy(ref).to(DEV)
    st = torch.zeros(1, dtype=torch.int32, device=DEV)
    y = cz.decompress_tilewise(cmp, n, torch.float32 if dtype == np.float32 else torch.float64, locate=locate,
                               status=st)
    torch.cuda.synchronize()
    assert int(st.item()) == 0
    iv = np.uint32 if dtype == np.float32 else np.uint64
    np.testing.assert_array_equal(y.cpu().numpy().view(iv), yr.view(iv))


@pytest.mark.parametrize("seed", range(24))
def test_randomized_parity(seed):
    """Seeded random mixtures (smooth + noise + spikes + ±0 / denormals / huge values,
    random n, eb mode, bound and encoding): whole-stream bytes and decompressed bits
    equal the oracle's. Covers both sides of the unchecked-quantizer cut (fl_p 17/18)
    and of the F2I fallback (|t| >= 2^22) inside one field."""
    rng = np.random.default_rng(1000 + seed)
    dtype = np.float32 if seed % 3 else np.float64
    n = int(rng.integers(1, 5 * 8192 + 97))
    i = np.arange(n)
    base = np.sin(i / rng.uniform(5, 500)) * rng.uniform(0.1, 1e4)
    noise = rng.standard_normal(n) * rng.choice([0.0, 1e-3, 1.0, 1e2])
    x = base + noise
    eb_mode = "rel" if seed % 2 else "abs"
    eb = float(rng.choice([1e-2, 1e-3, 1e-4, 1e-5])) if eb_mode == "rel" else float(rng.choice([1e-3, 0.05, 2.0]))
    # spikes in units of 2·eb (ABS) or of the smooth part's scale (REL): around the
    # F2I cut (|q| ~ 2^22), deep in F2I territory (2^26), and a RANGE hit in 1 seed of 8
    unit = 2 * eb if eb_mode == "abs" else np.abs(base).max() + 1.0
    big = [2**22 - 0.5, 2**22 + 0.5, -(2**22 + 1.5), 2**26 + 3, 3e5] if eb_mode == "abs" else [1e3, -5e2, 37.0]
    if seed % 8 == 7:
        big.append(2**31 if eb_mode == "abs" else np.inf)
    k = rng.integers(0, n, max(1, n // 200))
    x[k] = rng.choice([0.0, -0.0, 1e-40, -1e-40] + [b * unit for b in big], size=k.size)
    xh = x.astype(dtype)
    check_roundtrip(xh, eb, eb_mode, "outlier" if seed % 4 < 2 else "plain")


def test_c_abi_rejects_invalid_arguments():
    """include/cszp2.h error behaviour: every entry point returns CSZP2_ERR_ARG (and
    touches nothing) for null / misaligned pointers, unknown dtype / modes / flags,
    non-positive or non-finite bounds and oversized n."""
    import ctypes

    L = cz._lib
    x = torch.zeros(4096, dtype=torch.float32, device=DEV)
    out = torch.zeros(cz.compress_bound(4096) + 64, dtype=torch.uint8, device=DEV)
    nb = torch.zeros(1, dtype=torch.int64, device=DEV)
    p = lambda t, off=0: ctypes.c_void_p(t.data_ptr() + off)  # noqa: E731
    s = ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)
    E = cz.ERR_ARG
    assert L.cszp2_compress(None, 10, 0, 1e-3, 0, 0, p(out), p(nb), s) == E          # null input
    assert L.cszp2_compress(p(x), 10, 0, 1e-3, 0, 0, None, p(nb), s) == E            # null output
    assert L.cszp2_compress(p(x), 10, 2, 1e-3, 0, 0, p(out), p(nb), s) == E          # dtype
    assert L.cszp2_compress(p(x), 10, 0, 1e-3, 2, 0, p(out), p(nb), s) == E          # eb_mode
    assert L.cszp2_compress(p(x), 10, 0, 1e-3, 0, 2, p(out), p(nb), s) == E          # enc_mode
    for eb in (0.0, -1.0, float("nan"), float("inf")):
        assert L.cszp2_compress(p(x), 10, 0, eb, 0, 0, p(out), p(nb), s) == E        # bound
    assert L.cszp2_compress(p(x, 4), 10, 0, 1e-3, 0, 0, p(out), p(nb), s) == E       # misaligned in
    assert L.cszp2_compress(p(x), 10, 0, 1e-3, 0, 0, p(out, 8), p(nb), s) == E       # misaligned out
    assert L.cszp2_compress(p(x), (1 << 35) + 1, 0, 1e-3, 0, 0, p(out), p(nb), s) == E  # n too large
    assert L.cszp2_compress_encode_ex(p(x), 10, 0, 1e-3, 0, 0, p(out), p(nb), 64, s) == E  # flags
    assert L.cszp2_compress_encode_ex(p(x), 10, 0, 1e-3, 0, 0, p(out), p(nb), 6, s) == E  # vec+scalar
    assert L.cszp2_decompress(None, p(x), 10, 0, None, s) == E
    assert L.cszp2_decompress(p(out), p(x, 4), 10, 0, None, s) == E
    assert L.cszp2_decompress(p(out), p(x), 10, 3, None, s) == E
    assert L.cszp2_value_range(p(x), 10, 0, None, s) == E
    assert L.cszp2_value_range(p(x), 10, 0, p(out, 8), s) == E
    assert L.cszp2_compress_prepare_range(p(x), 10, 0, 1e-3, None, p(out), s) == E
    assert L.cszp2_compress_prepare_range(p(x), 10, 0, 1e-3, p(out, 8), p(out), s) == E
    assert L.cszp2_compress_prepare_range(p(x), 10, 0, 0.0, p(nb), p(out), s) == E
    assert L.cszp2_decompress_nd(p(out), p(x), 2 ** 12, 2 ** 12, 2 ** 12, 3, 0, None, s) == E  # > 2^35 values
    assert L.cszp2_compress_nd(p(x), 2 ** 12, 2 ** 12, 2 ** 12, 3, 0, 1e-3, 0, 0, p(out), p(nb), s) == E
    torch.cuda.synchronize()
    assert int(nb.item()) == 0 and int(out.sum().item()) == 0  # nothing was written


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
@pytest.mark.parametrize("enc", ["plain", "outlier"])
def test_incompressible_many_tiles(dtype, enc):
    """More tiles than resident compression CTAs with near-incompressible payloads
    (noise at a tiny ABS bound: fl ~ 25-30, most of the 32 KiB staging ring per tile),
    so tiles are claimed after staging, the resolver falls behind and producers wait
    for ring room: whole-stream parity with the oracle."""
    rng = np.random.default_rng(31 if dtype == np.float32 else 32)
    n = (1 << 23) + 32 * 77 + 5
    xh = (rng.standard_normal(n) * 1e3).astype(dtype)
    got = check_roundtrip(xh, 1e-5, "abs", enc)
    assert got is not None and got.size > 0.4 * xh.nbytes  # near-incompressible (f64: ~0.45)


@pytest.mark.parametrize("eb_mode", ["abs", "rel"])
def test_encode_repeated_on_one_buffer(eb_mode):
    """cszp2_compress_encode re-zeroes its lookback descriptors and ticket, so encoding
    again into the same d_out (after one prepare, or with another mode) gives the
    oracle's stream every time (include/cszp2.h)."""
    rng = np.random.default_rng(77)
    xh = np.cumsum(rng.standard_normal(8192 * 30 + 45)).astype(np.float32)
    x = torch.from_numpy(xh).to(DEV)
    out = torch.full((cz.compress_bound(x.numel()),), 0xAA, dtype=torch.uint8, device=DEV)
    nb = torch.zeros(1, dtype=torch.int64, device=DEV)
    cz.compress_prepare(x, 1e-3, eb_mode, out)
    for enc in ("outlier", "outlier", "plain", "outlier"):
        cz.compress_encode(x, 1e-3, eb_mode, enc, out, nb)
        torch.cuda.synchronize()
        ref, rc = oracle.compress(xh, 1e-3, EBM[eb_mode], ENC[enc])
        assert rc == oracle.OK and int(nb.item()) == ref.size
        np.testing.assert_array_equal(out[:ref.size].cpu().numpy(), ref)


def test_binding_validates_buffers():
    """The ctypes binding refuses buffers the kernels would overrun or misread
    (ADVICE r1): short / wrongly typed stream buffers, output tensors of the wrong
    length, dtype or layout, status / size words of the wrong type."""
    x = torch.randn(10000, device=DEV)
    bound = cz.compress_bound(x.numel())
    good = torch.empty(bound, dtype=torch.uint8, device=DEV)
    nb = torch.zeros(1, dtype=torch.int64, device=DEV)
    bad_calls = [
        lambda: cz.compress(x, 1e-3, out=torch.empty(bound - 1, dtype=torch.uint8, device=DEV)),
        lambda: cz.compress(x, 1e-3, out=torch.empty(bound // 4 + 1, dtype=torch.int32, device=DEV)),
        lambda: cz.compress(x, 1e-3, out=good, out_bytes=torch.zeros(1, dtype=torch.int32, device=DEV)),
        lambda: cz.compress(x.to(torch.float16), 1e-3),
        lambda: cz.compress_encode(x[::2], 1e-3, "abs", "plain", good, nb),
        lambda: cz.compress_prepare(x, 1e-3, "rel", good[:100]),
        lambda: cz.decompress(good, x.numel(), out=torch.empty(x.numel() - 1, device=DEV)),
        lambda: cz.decompress(good, x.numel(), out=torch.empty(2 * x.numel(), device=DEV)[::2]),
        lambda: cz.decompress(good, x.numel(), status=torch.zeros(1, dtype=torch.int64, device=DEV)),
        lambda: cz.decompress_range(good, x.numel(), 0, 10, out=torch.empty(9, device=DEV)),
        lambda: cz.container_index(nb, out=torch.empty(1, dtype=torch.int64, device=DEV)),
    ]
    for c in bad_calls:
        with pytest.raises(ValueError):
            c()


@pytest.mark.parametrize("eb_mode", ["abs", "rel"])
def test_encode_prepared_flag(eb_mode):
    """FLAG_PREPARED (include/cszp2.h): after a prepare, encode may skip re-zeroing the
    tile index — the stream is the oracle's; cszp2_compress uses exactly this pair."""
    rng = np.random.default_rng(78)
    xh = np.cumsum(rng.standard_normal(8192 * 20 + 45)).astype(np.float32)
    x = torch.from_numpy(xh).to(DEV)
    out = torch.full((cz.compress_bound(x.numel()),), 0xAA, dtype=torch.uint8, device=DEV)
    nb = torch.zeros(1, dtype=torch.int64, device=DEV)
    for enc in ("outlier", "plain"):
        cz.compress_prepare(x, 1e-3, eb_mode, out)
        cz.compress_encode(x, 1e-3, eb_mode, enc, out, nb, prepared=True)
        torch.cuda.synchronize()
        ref, rc = oracle.compress(xh, 1e-3, EBM[eb_mode], ENC[enc])
        assert rc == oracle.OK and int(nb.item()) == ref.size
        np.testing.assert_array_equal(out[:ref.size].cpu().numpy(), ref)


@pytest.mark.slow
@pytest.mark.parametrize("cfg,enc", [("cfg3b", "outlier"), ("cfg4a", "plain")])
def test_repeated_runs_are_deterministic(cfg, enc):
    """The decoupled lookback, the dynamic tile tickets and the staging ring are
    concurrent; the stream they produce must not depend on the schedule. 25 encodes of
    a full-size config (with the L2 flushed in between, so the schedules differ) give
    the same bytes every time (compared on the device), and the first equals the oracle."""
    spec = CONFIGS[cfg]
    x = make_field(cfg, DEV)
    lam = spec.ebs[-1]
    out = torch.empty(cz.compress_bound(x.numel(), x.dtype), dtype=torch.uint8, device=DEV)
    nb = torch.zeros(1, dtype=torch.int64, device=DEV)
    cz.compress(x, lam, spec.eb_mode, enc, out=out, out_bytes=nb)
    torch.cuda.synchronize()
    total = int(nb.item())
    first = out[:total].clone()
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=DEV)
    for _ in range(25):
        flush.zero_()
        out.fill_(0xAA)
        cz.compress(x, lam, spec.eb_mode, enc, out=out, out_bytes=nb)
        torch.cuda.synchronize()
        assert int(nb.item()) == total
        assert torch.equal(out[:total], first)
    ref, rc = oracle.compress(x.cpu().numpy(), lam, EBM[spec.eb_mode], ENC[enc])
    assert rc == oracle.OK
    np.testing.assert_array_equal(first.cpu().numpy(), ref)


@pytest.mark.parametrize("flags", [16, 32])
@pytest.mark.parametrize("enc", ["plain", "outlier"])
@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_lookback_window_width_same_stream(flags, enc, dtype):
    """The lookback's first window is 32 predecessors below 2^16 tiles and 256 from there on (a
    speed choice, kernels.cuh LB_NARROW_TILES); forcing either width (FLAG_LB_WIDE /
    FLAG_LB_NARROW) on a field of ~1700 tiles — several per CTA, lookbacks across many
    windows — gives the oracle's stream byte for byte."""
    n = 1700 * 8192 + 32 * 5 + 9
    xh = make_field("cfg4a", DEV, 0, n).cpu().numpy().astype(dtype)
    x = torch.from_numpy(xh).to(DEV)
    ref, rc = oracle.compress(xh, 1e-4, oracle.REL, oracle.OUTLIER if enc == "outlier" else oracle.PLAIN)
    assert rc == oracle.OK
    out = torch.full((cz.compress_bound(n, x.dtype),), 0xAA, dtype=torch.uint8, device=DEV)
    nb = torch.zeros(1, dtype=torch.int64, device=DEV)
    cz.compress_prepare(x, 1e-4, "rel", out)
    cz.compress_encode_ex(x, 1e-4, "rel", enc, out, nb, flags=flags)
    torch.cuda.synchronize()
    assert int(nb.item()) == ref.size
    np.testing.assert_array_equal(out[: ref.size].cpu().numpy(), ref)
    with pytest.raises(cz.CszpError):
        cz.compress_encode_ex(x, 1e-4, "rel", enc, out, nb, flags=48)
