"""Independent numpy reader of a FORMAT.md stream (tests only).

Written directly from FORMAT.md with numpy bit unpacking instead of the
oracle's shift loops, so that a layout mistake in the oracle (transposed
plane/value index, wrong bit order, wrong field order) shows up as a mismatch
against this reader. It shares no code with the oracle or the CUDA path.
"""
from __future__ import annotations

import struct

import numpy as np

MAGIC = 0x325A5343


def roundup16(v: int) -> int:
    return (v + 15) // 16 * 16


def header(buf) -> dict:
    b = bytes(np.asarray(buf, dtype=np.uint8)[:64])
    magic, ver, dtype, enc, log2L, ebm, status, bpt, _r = struct.unpack_from("<IBBBBBBHI", b, 0)
    n, eb, eb_abs, pb, total, r2 = struct.unpack_from("<QddQQQ", b, 16)
    return dict(magic=magic, version=ver, dtype=dtype, enc_mode=enc, log2L=log2L, eb_mode=ebm,
                status=status, bpt=bpt, n=n, eb=eb, eb_abs=eb_abs, payload_bytes=pb,
                total_bytes=total, reserved=r2)


def geometry(n: int, L: int = 32, bpt: int = 256):
    nb = -(-n // L)
    T = -(-nb // bpt)
    O = roundup16(64 + 8 * T)
    D = roundup16(O + nb)
    return nb, T, O, D


def block_size(byte: int, L: int = 32) -> int:
    fb = L // 8
    fl = byte & 31
    if byte & 0x80:
        return fb + ((byte >> 5) & 3) + 1 + fb * fl
    assert byte & 0x60 == 0, "reserved bits set"
    return fb * (1 + fl) if fl else 0


def _field_bits(raw: np.ndarray, L: int) -> np.ndarray:
    """L/8 bytes -> L bits, value i = byte i//8 bit i%8 (little bit order)."""
    return np.unpackbits(raw, bitorder="little")[:L].astype(np.int64)


def decode_block(byte: int, payload: np.ndarray, L: int = 32) -> np.ndarray:
    """-> residuals d (int64) of one block."""
    fb = L // 8
    size = block_size(byte, L)
    assert payload.size == size
    if size == 0:
        return np.zeros(L, dtype=np.int64)
    sign = _field_bits(payload[:fb], L)
    pos = fb
    a = np.zeros(L, dtype=np.int64)
    if byte & 0x80:
        ob = ((byte >> 5) & 3) + 1
        a[0] = int.from_bytes(bytes(payload[pos:pos + ob]), "little")
        pos += ob
    for k in range(byte & 31):
        bits = _field_bits(payload[pos:pos + fb], L)
        if byte & 0x80:
            assert bits[0] == 0, "outlier slot of a plane must be 0"
        a += bits << k
        pos += fb
    return np.where(sign == 1, -a, a)


def parse(buf, L: int | None = None) -> dict:
    """Whole stream -> header, offsets, per-block sizes, q (int64, length n)."""
    buf = np.asarray(buf, dtype=np.uint8)
    h = header(buf)
    assert h["magic"] == MAGIC
    L = L or (1 << h["log2L"])
    n = h["n"]
    nb, T, O, D = geometry(n, L, h["bpt"])
    index = np.frombuffer(bytes(buf[64:64 + 8 * T]), dtype="<u8") if T else np.zeros(0, np.uint64)
    offs = buf[O:O + nb]
    sizes = np.array([block_size(int(b), L) for b in offs], dtype=np.int64)
    starts = np.concatenate([[0], np.cumsum(sizes)])
    q = np.zeros(nb * L, dtype=np.int64)
    for b in range(nb):
        d = decode_block(int(offs[b]), buf[D + starts[b]:D + starts[b + 1]], L)
        q[b * L:(b + 1) * L] = np.cumsum(d)
    return dict(header=h, index=index, offsets=offs, sizes=sizes, q=q[:n], q_padded=q,
                geometry=(nb, T, O, D), payload_end=D + int(starts[-1]))
