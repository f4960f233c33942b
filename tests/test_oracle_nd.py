"""Pins of the oracle's multi-dimensional Lorenzo path (NEXT #3; P:365-388,
FORMAT.md §7) against closed forms and an independent numpy inverse."""
import numpy as np
import pytest

from tests import streamparse as sp


def _nd_residual_blocks(s):
    """numpy reader: per-block residuals (nb, 64) of an nD stream."""
    h = sp.header(s)
    nb_hdr = None
    buf = np.asarray(s, np.uint8)
    nx = int.from_bytes(bytes(buf[56:60]), "little")
    ny = int.from_bytes(bytes(buf[60:64]), "little")
    pred = int(buf[12])
    b = 8 if pred == 1 else 4
    nz = h["n"] // (nx * ny)
    nbx, nby = -(-nx // b), -(-ny // b)
    nbz = 1 if pred == 1 else -(-nz // b)
    nb = nbx * nby * nbz
    T = -(-nb // 256)
    O = sp.roundup16(64 + 8 * T)
    D = sp.roundup16(O + nb)
    offs = buf[O:O + nb]
    sizes = np.array([sp.block_size(int(o), 64) for o in offs])
    starts = np.concatenate([[0], np.cumsum(sizes)])
    d = np.stack([sp.decode_block(int(offs[k]), buf[D + starts[k]:D + starts[k + 1]], 64) for k in range(nb)])
    return d, (nx, ny, nz, nbx, nby, nbz, b, pred)


def _numpy_inverse(d, geo):
    """Lorenzo inverse as cumulative sums (an independent formulation of FORMAT.md §7:
    the residual is the block-local mixed difference, so q is its multi-axis cumsum)."""
    nx, ny, nz, nbx, nby, nbz, b, pred = geo
    if pred == 1:
        blocks = d.reshape(nby, nbx, 8, 8).cumsum(-1).cumsum(-2)
        full = blocks.transpose(0, 2, 1, 3).reshape(nby * 8, nbx * 8)
        return full[:ny, :nx]
    blocks = d.reshape(nbz, nby, nbx, 4, 4, 4).cumsum(-1).cumsum(-2).cumsum(-3)
    full = blocks.transpose(0, 3, 1, 4, 2, 5).reshape(nbz * 4, nby * 4, nbx * 4)
    return full[:nz, :ny, :nx]


def test_2d_linear_field_closed_form(orc):
    """A linear integer field a + bx + cy is predicted exactly inside a block: residual
    a+bX+cY at the corner, b on the first row, c on the first column, 0 elsewhere."""
    y, x = np.mgrid[0:19, 0:27]
    f = (3 + 2 * x + 5 * y).astype(np.float32)
    s, rc = orc.compress_nd(f, 0.5, orc.ABS, orc.PLAIN)
    assert rc == orc.OK
    d, geo = _nd_residual_blocks(s)
    nx, ny, nz, nbx, nby, nbz, b, pred = geo
    for k in range(d.shape[0]):
        by_, bx_ = divmod(k, nbx)
        blk = d[k].reshape(8, 8)
        X0, Y0 = 8 * bx_, 8 * by_
        assert blk[0, 0] == 3 + 2 * X0 + 5 * Y0
        rows = min(8, ny - Y0)
        cols = min(8, nx - X0)
        assert np.all(blk[0, 1:cols] == 2) and np.all(blk[1:rows, 0] == 5)
        assert not blk[1:rows, 1:cols].any()
        assert not blk[rows:, :].any() and not blk[:, cols:].any()  # outside the field: 0


def test_3d_trilinear_mixed_term(orc):
    """3D Lorenzo annihilates everything but the xyz term: q = 1 + x + y + z + 7xyz gives
    interior residual 7 (the triple mixed difference)."""
    z, y, x = np.mgrid[0:8, 0:8, 0:8]
    f = (1 + x + y + z + 7 * x * y * z).astype(np.float64)
    s, rc = orc.compress_nd(f, 0.5, orc.ABS, orc.OUTLIER)
    assert rc == orc.OK
    d, geo = _nd_residual_blocks(s)
    for k in range(d.shape[0]):
        blk = d[k].reshape(4, 4, 4)
        assert np.all(blk[1:, 1:, 1:] == 7)


@pytest.mark.parametrize("shape", [(37, 53), (8, 8), (1, 200), (9, 10, 11), (4, 4, 4), (5, 17, 3)])
@pytest.mark.parametrize("enc", [0, 1])
def test_nd_roundtrip_numpy_inverse_and_bound(orc, shape, enc):
    rng = np.random.default_rng(len(shape) * 100 + enc)
    f = rng.standard_normal(shape)
    for ax in range(len(shape)):
        f = f.cumsum(ax)
    f = f.astype(np.float32)
    s, rc = orc.compress_nd(f, 1e-3, orc.REL, enc)
    assert rc == orc.OK
    g, rc = orc.decompress_nd(s, shape)
    assert rc == orc.OK
    eb = sp.header(s)["eb_abs"]
    err = np.abs(f.astype(np.float64) - g)
    assert np.all(err <= eb * (1 + 2 ** -20) + 2 ** -21 * np.maximum(np.abs(f), np.abs(g)))
    d, geo = _nd_residual_blocks(s)
    q = _numpy_inverse(d, geo)
    inv = np.float32(1.0 / (2.0 * eb))
    np.testing.assert_array_equal(q, np.rint(f * inv).astype(np.int64))


def test_nd_range_limit(orc):
    """2D residuals reach 4 max|q|: the stricter limit 2^28-16 (f32) applies."""
    ok = np.full((8, 8), 268435440.0, np.float32)
    assert orc.compress_nd(ok, 0.5, orc.ABS, orc.PLAIN)[1] == orc.OK
    bad = np.full((8, 8), 268435456.0, np.float32)
    assert orc.compress_nd(bad, 0.5, orc.ABS, orc.PLAIN)[1] == orc.ERR_RANGE
    bad3 = np.full((4, 4, 4), 134217728.0, np.float32)
    assert orc.compress_nd(bad3, 0.5, orc.ABS, orc.PLAIN)[1] == orc.ERR_RANGE


def test_1d_decoder_rejects_nd_stream(orc):
    f = np.ones((16, 16), np.float32)
    s, _ = orc.compress_nd(f, 1e-2, orc.ABS, orc.PLAIN)
    assert orc.decompress(s, 256)[1] == orc.ERR_FORMAT
