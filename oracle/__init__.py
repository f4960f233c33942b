"""ctypes wrapper around the plain C oracle (oracle/cszp2_oracle.c).

TEST INFRASTRUCTURE ONLY. Only tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / ``--impl reference`` legs may import this module. The product
package (paper_conf_sc_huangdlc24_b200) never imports it and never falls back
to it.

The oracle follows FORMAT.md (the stream format + arithmetic contract written
from PAPER.md) step by step; see cszp2_oracle.h for citations and pins.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "cszp2_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

F32, F64 = 0, 1
ABS, REL = 0, 1
PLAIN, OUTLIER = 0, 1
OK, ERR_ARG, ERR_RANGE, ERR_FORMAT = 0, 1, 3, 4

CFLAGS = ["-std=c11", "-O2", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared"]


def build(force: bool = False) -> str:
    """Compile liboracle.so in-tree (plain gcc, no FMA contraction)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < max(
        os.path.getmtime(_SRC), os.path.getmtime(os.path.join(_HERE, "cszp2_oracle.h"))
    ):
        subprocess.check_call(["gcc", *CFLAGS, "-o", _LIB, _SRC, "-lm"])
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        u64, i32, dbl, vp = ctypes.c_uint64, ctypes.c_int, ctypes.c_double, ctypes.c_void_p
        pu64 = ctypes.POINTER(ctypes.c_uint64)
        L.oracle_compress_bound.argtypes = [u64, i32]
        L.oracle_compress_bound.restype = u64
        L.oracle_resolve_eb.argtypes = [vp, u64, i32, dbl, i32, ctypes.POINTER(ctypes.c_double)]
        L.oracle_quantize.argtypes = [vp, u64, i32, dbl, vp]
        L.oracle_dequantize.argtypes = [vp, u64, i32, dbl, vp]
        L.oracle_dequantize.restype = None
        L.oracle_encode_block.argtypes = [vp, i32, i32, vp, vp]
        L.oracle_decode_block.argtypes = [ctypes.c_uint8, vp, i32, vp]
        L.oracle_block_size.argtypes = [ctypes.c_uint8, i32]
        L.oracle_compress.argtypes = [vp, u64, i32, dbl, i32, i32, i32, vp, pu64]
        L.oracle_compress_ints.argtypes = [vp, u64, i32, i32, vp, pu64]
        L.oracle_decompress.argtypes = [vp, u64, vp, u64, i32]
        L.oracle_decompress_ints.argtypes = [vp, u64, vp, u64]
        L.oracle_compress_bound_nd.argtypes = [u64, u64, u64, i32]
        L.oracle_compress_bound_nd.restype = u64
        L.oracle_compress_nd.argtypes = [vp, u64, u64, u64, i32, i32, dbl, i32, i32, vp, pu64]
        L.oracle_decompress_nd.argtypes = [vp, u64, vp, u64, u64, u64, i32, i32]
        _lib = L
    return _lib


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def _dtype_code(x: np.ndarray) -> int:
    if x.dtype == np.float32:
        return F32
    if x.dtype == np.float64:
        return F64
    raise TypeError(f"unsupported dtype {x.dtype}")


def compress_bound(n: int, L: int = 32) -> int:
    return int(lib().oracle_compress_bound(n, L))


def resolve_eb(x: np.ndarray, eb: float, eb_mode: int) -> float:
    x = np.ascontiguousarray(x)
    out = ctypes.c_double(0.0)
    rc = lib().oracle_resolve_eb(_ptr(x), x.size, _dtype_code(x), eb, eb_mode, ctypes.byref(out))
    if rc != OK:
        raise ValueError(f"oracle_resolve_eb rc={rc}")
    return out.value


def quantize(x: np.ndarray, eb_abs: float):
    x = np.ascontiguousarray(x)
    q = np.zeros(x.size, dtype=np.int32)
    rc = lib().oracle_quantize(_ptr(x), x.size, _dtype_code(x), eb_abs, _ptr(q))
    return q, rc


def dequantize(q: np.ndarray, eb_abs: float, dtype=np.float32) -> np.ndarray:
    q = np.ascontiguousarray(q, dtype=np.int32)
    out = np.empty(q.size, dtype=dtype)
    lib().oracle_dequantize(_ptr(q), q.size, _dtype_code(out), eb_abs, _ptr(out))
    return out


def encode_block(q: np.ndarray, enc_mode: int, L: int = 32):
    """One block of L quantization integers -> (offset byte, payload bytes)."""
    q = np.ascontiguousarray(q, dtype=np.int32)
    assert q.size == L
    ob = np.zeros(1, dtype=np.uint8)
    buf = np.zeros(4 * L + 8, dtype=np.uint8)
    size = lib().oracle_encode_block(_ptr(q), L, enc_mode, _ptr(ob), _ptr(buf))
    return int(ob[0]), bytes(buf[:size])


def decode_block(offset_byte: int, payload: bytes, L: int = 32):
    buf = np.zeros(4 * L + 8, dtype=np.uint8)
    buf[: len(payload)] = np.frombuffer(payload, dtype=np.uint8)
    q = np.zeros(L, dtype=np.int32)
    size = lib().oracle_decode_block(offset_byte, _ptr(buf), L, _ptr(q))
    return q, size


def block_size(offset_byte: int, L: int = 32) -> int:
    return int(lib().oracle_block_size(offset_byte, L))


def compress(x: np.ndarray, eb: float, eb_mode: int = ABS, enc_mode: int = PLAIN, L: int = 32):
    """Whole stream -> (bytes as np.uint8 array, rc)."""
    x = np.ascontiguousarray(x)
    out = np.zeros(compress_bound(x.size, L), dtype=np.uint8)
    nbytes = ctypes.c_uint64(0)
    rc = lib().oracle_compress(
        _ptr(x), x.size, _dtype_code(x), eb, eb_mode, enc_mode, L, _ptr(out), ctypes.byref(nbytes)
    )
    if rc == ERR_ARG:
        raise ValueError("oracle_compress: bad argument")
    return out[: nbytes.value].copy(), rc


def compress_ints(q: np.ndarray, enc_mode: int = PLAIN, L: int = 32) -> np.ndarray:
    q = np.ascontiguousarray(q, dtype=np.int32)
    out = np.zeros(compress_bound(q.size, L), dtype=np.uint8)
    nbytes = ctypes.c_uint64(0)
    rc = lib().oracle_compress_ints(_ptr(q), q.size, enc_mode, L, _ptr(out), ctypes.byref(nbytes))
    if rc != OK:
        raise ValueError(f"oracle_compress_ints rc={rc}")
    return out[: nbytes.value].copy()


def decompress(cmp: np.ndarray, n: int, dtype=np.float32):
    """Stream -> (values, rc)."""
    cmp = np.ascontiguousarray(cmp, dtype=np.uint8)
    out = np.zeros(n, dtype=dtype)
    rc = lib().oracle_decompress(_ptr(cmp), cmp.size, _ptr(out), n, F32 if dtype == np.float32 else F64)
    return out, rc


def decompress_ints(cmp: np.ndarray, n: int):
    cmp = np.ascontiguousarray(cmp, dtype=np.uint8)
    q = np.zeros(n, dtype=np.int32)
    rc = lib().oracle_decompress_ints(_ptr(cmp), cmp.size, _ptr(q), n)
    return q, rc


def compress_nd(x: np.ndarray, eb: float, eb_mode: int = ABS, enc_mode: int = OUTLIER):
    """NEXT #3: 2D (8x8 blocks) or 3D (4x4x4) Lorenzo stream of a 2D/3D array
    (last axis fastest). Returns (bytes, rc)."""
    x = np.ascontiguousarray(x)
    ndim = x.ndim
    if ndim == 2:
        ny, nx = x.shape
        nz = 1
    elif ndim == 3:
        nz, ny, nx = x.shape
    else:
        raise ValueError("2D or 3D array expected")
    out = np.zeros(lib().oracle_compress_bound_nd(nx, ny, nz, ndim), dtype=np.uint8)
    nbytes = ctypes.c_uint64(0)
    rc = lib().oracle_compress_nd(_ptr(x), nx, ny, nz, ndim, _dtype_code(x), eb, eb_mode, enc_mode,
                                  _ptr(out), ctypes.byref(nbytes))
    if rc == ERR_ARG:
        raise ValueError("oracle_compress_nd: bad argument")
    return out[: nbytes.value].copy(), rc


def decompress_nd(cmp: np.ndarray, shape, dtype=np.float32):
    cmp = np.ascontiguousarray(cmp, dtype=np.uint8)
    out = np.zeros(int(np.prod(shape)), dtype=dtype)
    if len(shape) == 2:
        (ny, nx), nz = shape, 1
    else:
        nz, ny, nx = shape
    rc = lib().oracle_decompress_nd(_ptr(cmp), cmp.size, _ptr(out), nx, ny, nz, len(shape),
                                    F32 if dtype == np.float32 else F64)
    return out.reshape(shape), rc
