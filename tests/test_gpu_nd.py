"""GPU parity for the multi-dimensional Lorenzo layouts (
P:365-388, Table VI; FORMAT.md §7): 2D 8x8 and 3D 4x4x4 blocks through
cszp2_compress_nd / cszp2_decompress_nd against oracle.compress_nd /
oracle.decompress_nd — whole stream byte-identical (output pre-poisoned with
0xAA), reconstruction bit-identical."""
import numpy as np
import pytest
import torch

pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import oracle  # noqa: E402
import paper_conf_sc_huangdlc24_b200 as cz  # noqa: E402

DEV = torch.device("cuda:0")
ENC = {"plain": oracle.PLAIN, "outlier": oracle.OUTLIER}
EBM = {"abs": oracle.ABS, "rel": oracle.REL}


def smooth_field(shape, seed, dtype, noise=1e-3):
    """Seeded smooth field + small noise (the structure of the paper's 2D/3D
    datasets: correlated along every axis)."""
    rng = np.random.default_rng(seed)
    axes = np.meshgrid(*[np.linspace(0, 3, s) for s in shape], indexing="ij")
    f = np.ones(shape)
    for k, a in enumerate(axes):
        f = f * np.sin(a * (1.3 + 0.4 * k) + k) + 0.3 * np.cos(2.1 * a)
    f = f + noise * rng.standard_normal(shape)
    return f.astype(dtype)


def gpu_nd(xh, eb, eb_mode, enc):
    x = torch.from_numpy(xh).to(DEV)
    out = torch.full((cz.compress_bound_nd(xh.shape, x.dtype),), 0xAA, dtype=torch.uint8, device=DEV)
    nb = torch.zeros(1, dtype=torch.int64, device=DEV)
    cz.compress_nd(x, eb, eb_mode, enc, out=out, out_bytes=nb)
    torch.cuda.synchronize()
    return x, out, int(nb.item())


def check_nd(xh, eb, eb_mode, enc):
    x, out, total = gpu_nd(xh, eb, eb_mode, enc)
    ref, rc = oracle.compress_nd(xh, eb, EBM[eb_mode], ENC[enc])
    got = out[:total].cpu().numpy()
    assert total == ref.size
    st = torch.zeros(1, dtype=torch.int32, device=DEV)
    if rc == oracle.ERR_RANGE:
        np.testing.assert_array_equal(got[:64], ref[:64])
        cz.decompress_nd(out, xh.shape, x.dtype, status=st)
        torch.cuda.synchronize()
        assert int(st.item()) == 3
        return got
    assert rc == oracle.OK
    if not np.array_equal(got, ref):
        bad = np.nonzero(got != ref)[0]
        raise AssertionError(f"stream differs at {bad.size} bytes, first {bad[:8]} (total {total})")
    y = torch.full_like(x, float("nan"))
    cz.decompress_nd(out, xh.shape, x.dtype, out=y, status=st)
    torch.cuda.synchronize()
    assert int(st.item()) == 0
    yr, rc = oracle.decompress_nd(ref, xh.shape, xh.dtype)
    assert rc == oracle.OK
    iv = np.uint32 if xh.dtype == np.float32 else np.uint64
    np.testing.assert_array_equal(y.cpu().numpy().view(iv), yr.view(iv))
    return got


SHAPES = [(8, 8), (37, 53), (1, 200), (300, 301), (0, 5),
          (4, 4, 4), (9, 10, 11), (5, 17, 3), (33, 70, 65), (1, 1, 1)]


@pytest.mark.parametrize("shape", SHAPES)
@pytest.mark.parametrize("enc", ["plain", "outlier"])
@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_nd_parity_rel(shape, enc, dtype):
    xh = smooth_field(shape, sum(shape) + 3, dtype)
    check_nd(xh, 1e-4, "rel", enc)


@pytest.mark.parametrize("shape", [(300, 301), (33, 70, 65)])
@pytest.mark.parametrize("eb", [0.5, 1e-2, 1e-6])
def test_nd_parity_abs_noise(shape, eb):
    rng = np.random.default_rng(7)
    xh = rng.standard_normal(shape).astype(np.float32)
    check_nd(xh, eb, "abs", "outlier")


@pytest.mark.parametrize("ndim", [2, 3])
def test_nd_range_status(ndim):
    shape = (40, 40) if ndim == 2 else (12, 12, 12)
    xh = smooth_field(shape, 1, np.float32)
    xh.flat[777] = 1e30  # |x/2eb| beyond the predictor's limit
    got = check_nd(xh, 1e-3, "abs", "outlier")
    assert got[9] == 3


def test_nd_and_1d_streams_are_not_interchangeable():
    xh = smooth_field((64, 64), 5, np.float32)
    x, out, total = gpu_nd(xh, 1e-3, "abs", "outlier")
    st = torch.zeros(1, dtype=torch.int32, device=DEV)
    cz.decompress(out, xh.size, torch.float32, status=st)
    torch.cuda.synchronize()
    assert int(st.item()) == 4
    s1, _ = cz.compress(x.view(-1), 1e-3, "abs", "outlier")
    st.zero_()
    cz.decompress_nd(s1, xh.shape, torch.float32, status=st)
    torch.cuda.synchronize()
    assert int(st.item()) == 4
    st.zero_()  # wrong extents
    cz.decompress_nd(out, (32, 128), torch.float32, status=st)
    torch.cuda.synchronize()
    assert int(st.item()) == 4


def test_nd_bad_arguments():
    x = torch.zeros(4, 4, 4, device=DEV)
    out = torch.empty(cz.compress_bound_nd((4, 4, 4)), dtype=torch.uint8, device=DEV)
    rc = cz._lib.cszp2_compress_nd(cz._ptr(x), 4, 4, 4, 2, 0, 1e-3, 0, 1, cz._ptr(out), None,
                                   cz._stream(None))  # ndim 2 with nz != 1
    assert rc == cz.ERR_ARG
    assert cz._lib.cszp2_compress_bound_nd(4, 4, 4, 4, 0) == 0
    assert cz._lib.cszp2_compress_bound_nd(1 << 32, 1, 1, 2, 0) == 0


@pytest.mark.parametrize("ndim", [2, 3])
def test_nd_error_bound_and_ratio_vs_1d(ndim):
    """Table VI analog: on a smooth field the nD predictor beats the 1D one
    in compression ratio; both honour the bound."""
    shape = (512, 512) if ndim == 2 else (64, 64, 64)
    xh = smooth_field(shape, 11, np.float32, noise=0.0)
    x, out, total = gpu_nd(xh, 1e-4, "rel", "outlier")
    y = cz.decompress_nd(out, xh.shape, torch.float32)
    s1, n1 = cz.compress(x.view(-1), 1e-4, "rel", "outlier")
    torch.cuda.synchronize()
    eb_abs = float(np.frombuffer(out[32:40].cpu().numpy().tobytes(), dtype=np.float64)[0])
    err = (y.double() - x.double()).abs().max().item()
    assert err <= eb_abs * (1 + 1e-6) + 1e-7 * float(x.abs().max())
    assert total < int(n1.item())


@pytest.mark.parametrize("kind", ["smooth", "incompressible"])
def test_nd_persistent_multi_tile_per_cta(kind):
    """Fields with more tiles than resident compression CTAs (1024 tiles of 4x4x4 blocks,
    2 CTAs/SM), so every CTA defers lookbacks across several tiles; the incompressible
    one (~60 KB per tile payload) forces the ring-full path (resolve the deferred tile
    before staging). Whole streams and values must equal the oracle's."""
    shape = (256, 256, 256)
    if kind == "smooth":
        xh = smooth_field(shape, 11, np.float32, noise=1e-2)
        check_nd(xh, 1e-4, "rel", "outlier")
    else:
        rng = np.random.default_rng(12)
        xh = (rng.standard_normal(shape) * 100.0).astype(np.float32)
        check_nd(xh, 1e-5, "abs", "plain")


@pytest.mark.parametrize("shape", [(9, 10, 128), (5, 17, 384), (3, 33, 256), (4, 4, 128), (64, 64, 512)])
@pytest.mark.parametrize("enc", ["plain", "outlier"])
def test_nd3_wide_rows_parity(shape, enc):
    """3D f32 fields with long rows (x a multiple of 128, so every warp's 32 blocks are
    one run of a block row), y/z extents that are not multiples of 4, partial last tiles,
    many tiles per CTA, and an incompressible field (ring-full path)."""
    xh = smooth_field(shape, sum(shape) + 5, np.float32, noise=1e-2)
    check_nd(xh, 1e-4, "rel", enc)
    rng = np.random.default_rng(sum(shape))
    xn = (rng.standard_normal(shape) * 100.0).astype(np.float32)  # incompressible: direct path
    check_nd(xn, 1e-5, "abs", enc)


@pytest.mark.parametrize("shape", [(96, 136), (12, 40, 68)])
@pytest.mark.parametrize("enc", ["plain", "outlier"])
@pytest.mark.parametrize("sigma_q", [2.0 ** 11, 2.0 ** 12.5, 2.0 ** 13.5])
def test_nd_certificate_boundary(shape, enc, sigma_q):
    """f32 nD compression quantizes with the unchecked magic-add patterns and redoes a
    block with F2I when its residuals reach |d| >= 2^15 (kernels_nd.cuh, ND_FAST_FL_MAX):
    noise scaled so that the blocks' fixed lengths straddle 15/16/17 must still give the
    oracle's stream byte for byte."""
    rng = np.random.default_rng(int(sigma_q) + len(shape))
    eb = 1e-3
    xh = (rng.standard_normal(shape) * sigma_q * 2 * eb).astype(np.float32)
    check_nd(xh, eb, "abs", enc)


@pytest.mark.parametrize("ndim", [2, 3])
@pytest.mark.parametrize("offset_q", [2.0 ** 20, 2.0 ** 21.5, 2.0 ** 22, 2.0 ** 23.5])
def test_nd_large_q_small_residuals(ndim, offset_q):
    """Smooth fields riding on a large offset: |q| from 2^20 to 2^23.5 (around the 2^22
    edge of the fast quantizer's binade) with small in-block residuals except at each
    block's corner, Outlier and Plain: streams and values equal the oracle's."""
    shape = (64, 72) if ndim == 2 else (16, 20, 24)
    eb = 1e-4
    xh = (smooth_field(shape, 3, np.float64, noise=1e-4) + offset_q * 2 * eb).astype(np.float32)
    for enc in ("plain", "outlier"):
        check_nd(xh, eb, "abs", enc)


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_nd_decompress_rejects_corrupt_streams(dtype):
    """FORMAT errors inside a multi-tile 3D stream (an offset byte with reserved bits, an
    offset byte whose size no longer sums to the tile's index range, a cleared index
    flag) in the first and in a later tile: status FORMAT (4), and the decompressor
    returns (its payload prefetch in flight is drained, no hang)."""
    shape = (64, 64, 96)  # 6144 blocks = 24 tiles, several per persistent CTA
    xh = smooth_field(shape, 9, dtype, noise=1e-2)
    x, out, total = gpu_nd(xh, 1e-4, "rel", "outlier")
    nb = (64 // 4) * (64 // 4) * (96 // 4)
    T = -(-nb // 256)
    O = (64 + 8 * T + 15) // 16 * 16

    def status(buf):
        st = torch.zeros(1, dtype=torch.int32, device=DEV)
        cz.decompress_nd(buf, shape, x.dtype, status=st)
        torch.cuda.synchronize()
        return int(st.item())

    assert status(out) == 0
    for b in (3, 256 * 17 + 5):
        bad = out.clone()
        bad[O + b] = 0x60  # Plain block with the reserved bits set
        assert status(bad) == 4
        bad = out.clone()
        bad[O + b] = (int(out[O + b].item()) & 0xE0) | ((int(out[O + b].item()) + 1) & 31)  # size changes
        assert status(bad) == 4
    for t in (0, 13):
        bad = out.clone()
        bad[64 + 8 * t + 7] = 0  # descriptor flag cleared
        assert status(bad) == 4


@pytest.mark.parametrize("flags", [cz.FLAG_LB_WIDE, cz.FLAG_LB_NARROW])
@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_nd_lookback_window_width_same_stream(flags, dtype):
    """The nD compressor is instantiated for 32- and 256-wide first lookback windows
    (32 below 2^16 tiles, kernels.cuh); forcing either on a 1024-tile field gives the
    oracle's stream, so the 256-wide one is covered without an 8 GiB field."""
    shape = (256, 256, 256)
    xh = smooth_field(shape, 13, dtype, noise=1e-2)
    x = torch.from_numpy(xh).to(DEV)
    ref, rc = oracle.compress_nd(xh, 1e-4, oracle.REL, oracle.OUTLIER)
    assert rc == oracle.OK
    out = torch.full((cz.compress_bound_nd(xh.shape, x.dtype),), 0xAA, dtype=torch.uint8, device=DEV)
    nb = torch.zeros(1, dtype=torch.int64, device=DEV)
    cz.compress_nd(x, 1e-4, "rel", "outlier", out=out, out_bytes=nb, flags=flags)
    torch.cuda.synchronize()
    assert int(nb.item()) == ref.size
    np.testing.assert_array_equal(out[: ref.size].cpu().numpy(), ref)
    with pytest.raises(cz.CszpError):
        cz.compress_nd(x, 1e-4, "rel", "outlier", out=out, out_bytes=nb, flags=cz.FLAG_LB_WIDE | cz.FLAG_LB_NARROW)


@pytest.mark.parametrize("shape,dtype", [((256, 1024), np.float32), ((96, 1000), np.float64),
                                         ((24, 64, 128), np.float64), ((20, 40, 96), np.float64)])
@pytest.mark.parametrize("offset16", [False, True])
def test_nd_256bit_paths(shape, dtype, offset16):
    """Rows of whole 32-byte vectors (2D: 8 values x w, 3D f64: 4 doubles) are gathered and
    stored with 256-bit accesses when the field base and the row pitch are 32-byte aligned
    (g.vec32); a base that is only 16-byte aligned takes the 16-byte path. Multi-tile
    fields, both bases: streams and values equal the oracle's."""
    xh = smooth_field(shape, sum(shape), dtype, noise=1e-2)
    w = np.dtype(dtype).itemsize
    pad = 16 // w if offset16 else 0
    flat = torch.empty(xh.size + pad + 16, dtype=torch.float32 if w == 4 else torch.float64, device=DEV)
    x = flat[pad: pad + xh.size].view(shape)
    x.copy_(torch.from_numpy(xh))
    assert (x.data_ptr() % 32 == 16) == offset16
    ref, rc = oracle.compress_nd(xh, 1e-4, oracle.REL, oracle.OUTLIER)
    assert rc == oracle.OK
    out = torch.full((cz.compress_bound_nd(xh.shape, x.dtype),), 0xAA, dtype=torch.uint8, device=DEV)
    nb = torch.zeros(1, dtype=torch.int64, device=DEV)
    cz.compress_nd(x, 1e-4, "rel", "outlier", out=out, out_bytes=nb)
    torch.cuda.synchronize()
    assert int(nb.item()) == ref.size
    np.testing.assert_array_equal(out[: ref.size].cpu().numpy(), ref)
    yflat = torch.full_like(flat, float("nan"))
    y = yflat[pad: pad + xh.size].view(shape)
    st = torch.zeros(1, dtype=torch.int32, device=DEV)
    cz.decompress_nd(out, shape, x.dtype, out=y, status=st)
    torch.cuda.synchronize()
    assert int(st.item()) == 0
    yr, rc = oracle.decompress_nd(ref, shape, dtype)
    iv = np.uint32 if w == 4 else np.uint64
    np.testing.assert_array_equal(y.cpu().numpy().view(iv), yr.view(iv))
    assert torch.isnan(yflat[:pad]).all() and torch.isnan(yflat[pad + xh.size:]).all()  # nothing outside
