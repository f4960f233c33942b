"""Pins of the CPU oracle against what the paper and mathematics fix (not gpu).

Each test names the passage (P:n = PAPER.md line) or the closed form it checks.
None of them re-derives an expected value by calling the oracle on the same
input through another entry point only; expected values come from the paper,
hand-worked fixtures (tests/golden/), numpy library routines, closed forms or
the independent numpy stream reader (tests/streamparse.py).
"""
import math
import os

import numpy as np
import pytest

from tests import streamparse as sp

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "worked_blocks.txt")


def _records():
    recs, cur = [], {}
    for line in open(GOLDEN):
        line = line.rstrip("\n")
        if line.startswith("#"):
            continue
        if not line.strip():
            if cur:
                recs.append(cur)
            cur = {}
            continue
        k, _, v = line.partition(":")
        cur[k.strip()] = v.strip()
    if cur:
        recs.append(cur)
    return recs


RECORDS = _records()


# ---------------------------------------------------------------- ❶ quantization

def test_paper_running_example_quantization(orc):
    """P:122 (Fig 5): eb = 0.1, 1.12 -> 6, reconstructed 6 x 2eb = 1.2, |1.12 - 1.2| < eb."""
    x = np.array([1.12], dtype=np.float32)
    q, rc = orc.quantize(x, 0.1)
    assert rc == orc.OK and q[0] == 6
    xr = orc.dequantize(q, 0.1)
    assert xr[0] == np.float32(1.2)
    assert abs(float(x[0]) - float(xr[0])) < 0.1


def test_eb_half_is_textbook_round_half_even(orc):
    """eb = 0.5 makes inv = s = 1, so q must be numpy's rint (ties to even):
    pins the rounding function (reading R-1) against a library routine."""
    rng = np.random.default_rng(1)
    x = np.concatenate([
        rng.uniform(-1e6, 1e6, 20000),
        np.arange(-50, 50) + 0.5,          # exact ties
        rng.integers(-1000, 1000, 500) + 0.5,
    ]).astype(np.float32)
    q, rc = orc.quantize(x, 0.5)
    assert rc == orc.OK
    np.testing.assert_array_equal(q, np.rint(x).astype(np.int32))
    xd = x.astype(np.float64)
    qd, rc = orc.quantize(xd, 0.5)
    np.testing.assert_array_equal(qd, np.rint(xd).astype(np.int32))


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
@pytest.mark.parametrize("eb", [1e-1, 1e-3, 3.7e-5])
def test_error_bound_closed_form(orc, dtype, eb):
    """|x - x'| <= eb plus the rounding of x' to T (reading R-10)."""
    rng = np.random.default_rng(7)
    x = (rng.standard_normal(50000) * 20).astype(dtype)
    s, rc = orc.compress(x, eb, orc.ABS, orc.OUTLIER)
    assert rc == orc.OK
    y, rc = orc.decompress(s, x.size, dtype)
    assert rc == orc.OK
    err = np.abs(x.astype(np.float64) - y.astype(np.float64))
    mag = np.maximum(np.abs(x), np.abs(y)).astype(np.float64)
    if dtype == np.float32:
        bound = eb * (1 + 2.0 ** -20) + 2.0 ** -21 * mag
    else:
        bound = eb * (1 + 2.0 ** -40) + 2.0 ** -50 * mag
    assert np.all(err <= bound)
    # the quantization step really is 2eb: errors reach close to eb (a dropped
    # factor 2 would halve them, a doubled one would break the bound above)
    assert err.max() > 0.9 * eb


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
@pytest.mark.parametrize("eb", [0.5, 1e-3, 3.7e-5])
def test_error_bound_where_float_q_rounds(orc, dtype, eb):
    """R-10 bound for |x / 2eb| from 2^24 up to the R-3 limit (2^30 - 64 for
    f32), where (T)q is no longer exact in f32: x' = fl(fl(q)·s) (FORMAT.md §6.6)
    must still land within eb of x plus the rounding of x' to T."""
    rng = np.random.default_rng(11)
    lo, hi = 2.0 ** 24, 2.0 ** 30 - 64
    mag = np.exp(rng.uniform(np.log(lo), np.log(hi), 60000))
    t = mag * rng.choice([-1.0, 1.0], mag.size)
    x = (t * 2 * eb).astype(dtype)
    x = x[np.abs(x.astype(np.float64) * (1.0 / (2 * eb))) < hi - 64]  # keep t strictly in range
    s, rc = orc.compress(x, eb, orc.ABS, orc.PLAIN)
    assert rc == orc.OK
    y, rc = orc.decompress(s, x.size, dtype)
    assert rc == orc.OK
    err = np.abs(x.astype(np.float64) - y.astype(np.float64))
    m = np.maximum(np.abs(x), np.abs(y)).astype(np.float64)
    if dtype == np.float32:
        bound = eb * (1 + 2.0 ** -20) + 2.0 ** -21 * m
    else:
        bound = eb * (1 + 2.0 ** -40) + 2.0 ** -50 * m
    assert np.all(err <= bound)
    # the values really are that large: |q| spans [2^24, 2^30) (numpy's own rint)
    qa = np.abs(np.rint(x.astype(np.float64) / (2 * eb)))
    assert qa.min() >= 2.0 ** 24 - 1 and qa.max() >= 2.0 ** 29


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_large_integers_round_trip_exactly_at_half(orc, dtype):
    """eb = 0.5 (s = inv = 1): every f32 of magnitude >= 2^24 is an integer, so q = x and
    x' = (T)q·1 must give x back exactly, up to the R-3 limit 2^30 - 64 (f32) /
    2^30 - 1 (f64). A dequantizer that drops or wraps high bits of q, or converts
    through a narrower type, fails here (FORMAT.md §6.6)."""
    rng = np.random.default_rng(12)
    top = 2 ** 30 - 64 if dtype == np.float32 else 2 ** 30 - 1
    v = rng.integers(2 ** 24, top + 1, 40000).astype(np.float64)
    v = np.concatenate([v, [2.0 ** 24, 2.0 ** 24 + 2, 2.0 ** 29 + 2.0 ** 6, top]])
    x = (v * rng.choice([-1.0, 1.0], v.size)).astype(dtype)
    assert np.all(np.abs(x.astype(np.float64)) <= top)
    s, rc = orc.compress(x, 0.5, orc.ABS, orc.OUTLIER)
    assert rc == orc.OK
    y, rc = orc.decompress(s, x.size, dtype)
    assert rc == orc.OK
    iv = np.uint32 if dtype == np.float32 else np.uint64
    np.testing.assert_array_equal(y.view(iv), x.view(iv))


def test_range_status(orc):
    """|t| beyond 2^30-1 cannot be stored in the fl <= 31 code: RANGE."""
    x = np.array([0.0, 1.0, 3e9], dtype=np.float32)
    s, rc = orc.compress(x, 0.5, orc.ABS, orc.PLAIN)
    assert rc == orc.ERR_RANGE
    h = sp.header(s)
    assert h["status"] == 3 and h["payload_bytes"] == 0
    nb, T, O, D = sp.geometry(3)
    assert h["total_bytes"] == sp.roundup16(D) == s.size
    _, rc = orc.decompress(s, 3)
    assert rc == orc.ERR_RANGE
    # NaN / Inf also RANGE
    for bad in (np.nan, np.inf):
        _, rc = orc.compress(np.array([1.0, bad], np.float32), 0.5, orc.ABS, orc.PLAIN)
        assert rc == orc.ERR_RANGE
    # largest accepted f32 t is 2^30-64; the next float (2^30) is rejected
    _, rc = orc.compress(np.array([1073741760.0], np.float32), 0.5, orc.ABS, orc.PLAIN)
    assert rc == orc.OK
    _, rc = orc.compress(np.array([1073741824.0], np.float32), 0.5, orc.ABS, orc.PLAIN)
    assert rc == orc.ERR_RANGE


# ---------------------------------------------------------------- REL

@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_rel_is_lambda_times_value_range(orc, dtype):
    rng = np.random.default_rng(3)
    x = (rng.standard_normal(10001) * 5 + 2).astype(dtype)
    lam = 1e-3
    r = float(np.float64(x.max()) - np.float64(x.min()))
    assert orc.resolve_eb(x, lam, orc.REL) == lam * r
    # NaNs are ignored by the range
    x2 = x.copy()
    x2[17] = np.nan
    assert orc.resolve_eb(x2, lam, orc.REL) == lam * r
    # zero range falls back to lambda (reading R-15)
    assert orc.resolve_eb(np.full(100, 3.0, dtype), lam, orc.REL) == lam
    s, rc = orc.compress(x, lam, orc.REL, orc.OUTLIER)
    h = sp.header(s)
    assert h["eb_abs"] == lam * r and h["eb"] == lam and h["eb_mode"] == 1


# ---------------------------------------------------------------- ❷ encoding

@pytest.mark.parametrize("rec", RECORDS, ids=[r["name"] for r in RECORDS])
def test_worked_blocks(orc, rec):
    L = int(rec["L"])
    q = np.array(eval(rec["q"], {"i": 0, "range": range}), dtype=np.int32)  # noqa: S307 (fixture expr)
    assert q.size == L
    mode = orc.OUTLIER if rec["mode"] == "outlier" else orc.PLAIN
    ob, payload = orc.encode_block(q, mode, L)
    assert ob == int(rec["offset"], 16)
    if "payload" in rec:
        assert payload.hex().upper() == rec["payload"].replace(" ", "").upper()
    if "size" in rec:
        assert len(payload) == int(rec["size"])
    if "cr" in rec:  # the paper's CR counts data bytes only
        assert round(L * 4 / len(payload), 2) == pytest.approx(float(rec["cr"]), abs=0.01)
    q2, size = orc.decode_block(ob, payload, L)
    assert size == len(payload)
    np.testing.assert_array_equal(q2, q)
    # the independent numpy reader agrees
    d = sp.decode_block(ob, np.frombuffer(payload, np.uint8), L)
    np.testing.assert_array_equal(np.cumsum(d), q)


def test_paper_outlier_shortens_fixed_length():
    """"the presence of an outlier necessitates storing four bits for each
    integer, compared to just one bit in its absence" — the L=8 example's fl."""
    rec = {r["name"]: r for r in RECORDS}
    assert int(rec["paper_L8_plain"]["offset"], 16) & 31 == 4
    assert int(rec["paper_L8_outlier"]["offset"], 16) & 31 == 1


def _bitlen(v):
    v = np.asarray(v, dtype=np.int64)
    out = np.zeros(v.shape, dtype=np.int64)
    nz = v > 0
    out[nz] = np.floor(np.log2(v[nz])).astype(np.int64) + 1
    return out


def test_brute_force_all_L8_residual_blocks(orc):
    """Every residual block in [-3,3]^8 at L=8 (5,764,801 blocks): lossless
    round trip, sizes equal to P:139's rule computed with numpy, Outlier chosen
    exactly when strictly smaller, and never larger than Plain."""
    vals = np.arange(-3, 4, dtype=np.int32)
    grids = np.meshgrid(*([vals] * 8), indexing="ij")
    d = np.stack([g.ravel() for g in grids], axis=1)  # (7^8, 8)
    q = np.cumsum(d, axis=1).astype(np.int32).ravel()
    n = q.size
    nb = n // 8
    for mode in (orc.PLAIN, orc.OUTLIER):
        s = orc.compress_ints(q, mode, L=8)
        q2, rc = orc.decompress_ints(s, n)
        assert rc == orc.OK
        np.testing.assert_array_equal(q2, q)
        _, _, O, _ = sp.geometry(n, 8)
        offs = s[O:O + nb].astype(np.int64)
        a = np.abs(d)
        fl_p = _bitlen(np.bitwise_or.reduce(a, axis=1))
        size_p = np.where(fl_p > 0, 1 + fl_p, 0)
        if mode == orc.PLAIN:
            np.testing.assert_array_equal(offs, fl_p)
            sizes = size_p
        else:
            fl_o = _bitlen(np.bitwise_or.reduce(a[:, 1:], axis=1))
            ob = np.maximum(1, (_bitlen(a[:, 0]) + 7) // 8)
            size_o = 1 + ob + fl_o
            use_o = size_o < size_p
            exp = np.where(use_o, 0x80 | ((ob - 1) << 5) | fl_o, fl_p)
            np.testing.assert_array_equal(offs, exp)
            sizes = np.where(use_o, size_o, size_p)
            assert np.all(sizes <= size_p)
        assert sp.header(s)["payload_bytes"] == int(sizes.sum())


@pytest.mark.parametrize("mode", [0, 1])
def test_random_blocks_every_fixed_length(orc, mode):
    """L=32 blocks whose max |d| has each bit length 0..31 (0..31 fits
    5 bits) round-trip and are parsed identically by the numpy reader."""
    rng = np.random.default_rng(11)
    blocks = []
    for fl in range(32):
        for _ in range(4):
            hi = (1 << fl) - 1 if fl else 0
            dd = rng.integers(-hi, hi + 1, 32, dtype=np.int64) if fl else np.zeros(32, np.int64)
            if fl:
                dd[rng.integers(1, 32)] = hi * (1 if rng.random() < 0.5 else -1)
            q = np.cumsum(dd)
            if np.abs(q).max() > (1 << 30) - 1:  # keep |q| <= 2^30-1
                q = q - int(q.mean())
                dd = np.diff(np.concatenate([[0], q]))
                if np.abs(q).max() > (1 << 30) - 1:
                    continue
            blocks.append(q)
    q = np.concatenate(blocks).astype(np.int32)
    s = orc.compress_ints(q, mode)
    q2, rc = orc.decompress_ints(s, q.size)
    assert rc == orc.OK
    np.testing.assert_array_equal(q2, q)
    np.testing.assert_array_equal(sp.parse(s)["q"], q)


# ---------------------------------------------------------------- ❸ ❹ stream

def test_serial_prefix_and_layout(orc):
    """the offsets are a plain serial prefix of block sizes; FORMAT.md §2
    layout checked with the numpy reader (sizes from the offset bytes alone)."""
    rng = np.random.default_rng(5)
    n = 256 * 32 * 3 + 32 * 17 + 11  # 3 full tiles, a ragged tile, a ragged block
    x = np.cumsum(rng.standard_normal(n)).astype(np.float32)
    s, rc = orc.compress(x, 0.05, orc.ABS, orc.OUTLIER)
    assert rc == orc.OK
    p = sp.parse(s)
    nb, T, O, D = p["geometry"]
    assert T == 4 and nb == 256 * 3 + 18
    incl = np.cumsum(p["sizes"])
    ends = [min(256 * (t + 1), nb) - 1 for t in range(T)]
    np.testing.assert_array_equal(p["index"], (np.uint64(2) << np.uint64(62)) | incl[ends].astype(np.uint64))
    h = p["header"]
    assert h["payload_bytes"] == incl[-1]
    assert h["total_bytes"] == sp.roundup16(D + incl[-1]) == s.size
    assert not s[64 + 8 * T:O].any() and not s[O + nb:D].any() and not s[p["payload_end"]:].any()
    # reader's q equals numpy's own quantization of x (independent ❶ path)
    inv = np.float32(1.0 / (2.0 * 0.05))
    np.testing.assert_array_equal(p["q"], np.rint(x * inv).astype(np.int64))
    # tail padding q_i = q_{i-1}: zero residuals past n
    tail = p["q_padded"][n:]
    assert np.all(tail == p["q"][-1])


def test_header_fields(orc):
    x = np.linspace(-1, 1, 1000, dtype=np.float64)
    s, rc = orc.compress(x, 1e-3, orc.ABS, orc.PLAIN)
    h = sp.header(s)
    assert h["magic"] == 0x325A5343 and bytes(s[:4]) == b"CSZ2"
    assert (h["version"], h["dtype"], h["enc_mode"], h["log2L"], h["eb_mode"], h["status"], h["bpt"]) == (1, 1, 0, 5, 0, 0, 256)
    assert h["n"] == 1000 and h["eb"] == 1e-3 and h["eb_abs"] == 1e-3 and h["reserved"] == 0


def test_empty_input_is_header_only(orc):
    s, rc = orc.compress(np.zeros(0, np.float32), 1e-3, orc.ABS, orc.PLAIN)
    assert rc == orc.OK and s.size == 64
    assert sp.header(s)["total_bytes"] == 64
    y, rc = orc.decompress(s, 0)
    assert rc == orc.OK and y.size == 0


def test_all_zero_field_hits_cr_bound(orc):
    """Zero block = 1 byte so CR -> 128 for f32 at L=32 (JetIn 126.28,
    P:255); exactly n*4 / (64 + 8T pad + nb pad) here."""
    n = 1 << 20
    s, _ = orc.compress(np.zeros(n, np.float32), 1e-4, orc.ABS, orc.OUTLIER)
    nb, T, O, D = sp.geometry(n)
    assert s.size == D
    cr = n * 4 / s.size
    assert 123 < cr < 128
    s64, _ = orc.compress(np.zeros(n, np.float64), 1e-4, orc.ABS, orc.OUTLIER)
    assert 246 < n * 8 / s64.size < 256


# ---------------------------------------------------------------- invariants

def _field(n, seed=0):
    i = np.arange(n)
    rng = np.random.default_rng(seed)
    return (np.sin(i / 300.0) * 40 + 250 + rng.standard_normal(n) * 0.01).astype(np.float32)


def test_outlier_never_worse_and_same_reconstruction(orc):
    """P:302 (CUSZP2-O always >= CUSZP2-P in CR) and P:310 (same lossy step ->
    same reconstructed data)."""
    x = _field(100003)
    sP, _ = orc.compress(x, 1e-4, orc.REL, orc.PLAIN)
    sO, _ = orc.compress(x, 1e-4, orc.REL, orc.OUTLIER)
    pP, pO = sp.parse(sP), sp.parse(sO)
    assert np.all(pO["sizes"] <= pP["sizes"])
    assert sO.size < sP.size  # smooth field: O strictly better
    yP, _ = orc.decompress(sP, x.size)
    yO, _ = orc.decompress(sO, x.size)
    np.testing.assert_array_equal(yP.view(np.uint32), yO.view(np.uint32))


def test_psnr_closed_form(orc):
    """Uniform quantization error => PSNR = -20 log10(lambda) + 10 log10(3)
    (84.77 dB at REL 1e-4) on a dense smooth field (PSNR per reading R-16)."""
    i = np.arange(1 << 18, dtype=np.float64)
    x = (np.sin(i / 5000.0) * 100 + np.cos(i / 777.0) * 30).astype(np.float32)
    for lam in (1e-2, 1e-3, 1e-4):
        s, _ = orc.compress(x, lam, orc.REL, orc.OUTLIER)
        y, _ = orc.decompress(s, x.size)
        r = float(x.max()) - float(x.min())
        mse = np.mean((x.astype(np.float64) - y.astype(np.float64)) ** 2)
        psnr = 20 * math.log10(r) - 10 * math.log10(mse)
        assert psnr == pytest.approx(-20 * math.log10(lam) + 10 * math.log10(3), abs=1.0)


def test_abs_recompression_idempotent(orc):
    """ABS: x' is already on the 2eb grid, so re-compressing it reproduces the
    stream byte for byte while max|q| < 2^20 (FORMAT.md §6)."""
    x = _field(70001) - 250
    s, _ = orc.compress(x, 1e-3, orc.ABS, orc.OUTLIER)
    y, _ = orc.decompress(s, x.size)
    s2, _ = orc.compress(y, 1e-3, orc.ABS, orc.OUTLIER)
    np.testing.assert_array_equal(s, s2)


def test_decompress_rejects_corruption(orc):
    x = _field(5000)
    s, _ = orc.compress(x, 1e-3, orc.ABS, orc.PLAIN)
    bad = s.copy(); bad[0] ^= 1
    assert orc.decompress(bad, x.size)[1] == orc.ERR_FORMAT
    assert orc.decompress(s[:-16], x.size)[1] == orc.ERR_FORMAT
    assert orc.decompress(s, x.size + 1)[1] == orc.ERR_FORMAT
    nb, T, O, D = sp.geometry(x.size)
    bad = s.copy(); bad[O] = 0x60 | (bad[O] & 31)  # reserved bits in a Plain byte
    assert orc.decompress(bad, x.size)[1] == orc.ERR_FORMAT
    assert orc.decompress(s, x.size, np.float64)[1] == orc.ERR_FORMAT
