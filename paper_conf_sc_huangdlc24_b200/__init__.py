"""B200-native cuSZp2 (Huang et al., SC'24): error-bounded lossy compression of
f32/f64 fields in one fused sm_100a kernel per direction.

This module is a thin ctypes binding over libcszp2.so (include/cszp2.h):
argument marshalling only. Every step of the hot path runs in the CUDA
kernels; there is no CPU fallback — importing fails loudly if the shared
library is missing, and calls fail if the tensors are not on a CUDA device.
"""
from __future__ import annotations

import ctypes
import os

import torch

from ._build import LIB as _LIB_PATH

# dev aid (scripts/ab_libs.py): load another build of the same C ABI for A/B timing
_LIB_PATH = os.environ.get("CSZP2_LIB", _LIB_PATH)

F32, F64 = 0, 1
EB_ABS, EB_REL = 0, 1
ENC_PLAIN, ENC_OUTLIER = 0, 1
OK, ERR_ARG, ERR_CUDA, ERR_RANGE, ERR_FORMAT = 0, 1, 2, 3, 4

_EB = {"abs": EB_ABS, "rel": EB_REL, EB_ABS: EB_ABS, EB_REL: EB_REL}
_ENC = {"plain": ENC_PLAIN, "outlier": ENC_OUTLIER, "p": ENC_PLAIN, "o": ENC_OUTLIER,
        ENC_PLAIN: ENC_PLAIN, ENC_OUTLIER: ENC_OUTLIER}
_DT = {torch.float32: F32, torch.float64: F64}
_TORCH_DT = {F32: torch.float32, F64: torch.float64}


class CszpError(RuntimeError):
    def __init__(self, fn: str, rc: int):
        super().__init__(f"{fn} failed with status {rc}")
        self.rc = rc


class Header(ctypes.Structure):
    _fields_ = [
        ("magic", ctypes.c_uint32),
        ("version", ctypes.c_uint8), ("dtype", ctypes.c_uint8), ("enc_mode", ctypes.c_uint8),
        ("log2L", ctypes.c_uint8), ("eb_mode", ctypes.c_uint8), ("status", ctypes.c_uint8),
        ("blocks_per_tile", ctypes.c_uint16),
        ("n", ctypes.c_uint64), ("eb", ctypes.c_double), ("eb_abs", ctypes.c_double),
        ("payload_bytes", ctypes.c_uint64), ("total_bytes", ctypes.c_uint64),
    ]

    def as_dict(self) -> dict:
        return {k: getattr(self, k) for k, _ in self._fields_}


def _load():
    if not os.path.exists(_LIB_PATH):
        raise ImportError(
            f"{_LIB_PATH} is missing: build it with `python -c 'import __graft_entry__ as g; g.build()'`"
        )
    L = ctypes.CDLL(_LIB_PATH)
    vp, u64, i32, dbl = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int, ctypes.c_double
    L.cszp2_compress_bound.argtypes = [u64, i32]
    L.cszp2_compress_bound.restype = u64
    sig = [vp, u64, i32, dbl, i32, i32, vp, vp, vp]
    L.cszp2_compress.argtypes = sig
    L.cszp2_compress_encode.argtypes = sig
    L.cszp2_compress_prepare.argtypes = [vp, u64, i32, dbl, i32, vp, vp]
    L.cszp2_value_range.argtypes = [vp, u64, i32, vp, vp]
    L.cszp2_compress_prepare_range.argtypes = [vp, u64, i32, dbl, vp, vp, vp]
    L.cszp2_compress_encode_ex.argtypes = [vp, u64, i32, dbl, i32, i32, vp, vp, ctypes.c_uint, vp]
    L.cszp2_decompress.argtypes = [vp, vp, u64, i32, vp, vp]
    L.cszp2_read_header.argtypes = [vp, ctypes.POINTER(Header), vp]
    L.cszp2_decompress_range.argtypes = [vp, u64, i32, u64, u64, vp, vp, vp]
    L.cszp2_compress_host.argtypes = [vp, u64, i32, dbl, i32, i32, vp, vp, vp, u64,
                                      ctypes.POINTER(ctypes.c_uint64), vp]
    L.cszp2_decompress_host.argtypes = [vp, u64, vp, vp, vp, u64, i32, vp, vp]
    L.cszp2_container_index.argtypes = [vp, i32, vp, vp]
    L.cszp2_decompress_scratch_bytes.argtypes = [u64]
    L.cszp2_decompress_scratch_bytes.restype = u64
    L.cszp2_decompress_tilewise.argtypes = [vp, vp, u64, i32, i32, vp, vp, vp]
    L.cszp2_compress_bound_nd.argtypes = [u64, u64, u64, i32, i32]
    L.cszp2_compress_bound_nd.restype = u64
    L.cszp2_compress_nd.argtypes = [vp, u64, u64, u64, i32, i32, dbl, i32, i32, vp, vp, vp]
    L.cszp2_compress_nd_ex.argtypes = [vp, u64, u64, u64, i32, i32, dbl, i32, i32, vp, vp, ctypes.c_uint, vp]
    L.cszp2_decompress_nd.argtypes = [vp, vp, u64, u64, u64, i32, i32, vp, vp]
    L.cszp2_version.restype = ctypes.c_char_p
    return L


_lib = _load()
LIBRARY_PATH = _LIB_PATH
EXPORTED = (
    "cszp2_compress_bound", "cszp2_compress", "cszp2_compress_prepare", "cszp2_compress_encode",
    "cszp2_compress_encode_ex", "cszp2_value_range", "cszp2_compress_prepare_range",
    "cszp2_decompress", "cszp2_decompress_range", "cszp2_read_header", "cszp2_compress_host", "cszp2_decompress_host",
    "cszp2_container_index", "cszp2_version",
    "cszp2_compress_bound_nd", "cszp2_compress_nd", "cszp2_compress_nd_ex", "cszp2_decompress_nd",
    "cszp2_decompress_scratch_bytes", "cszp2_decompress_tilewise",
)


def version() -> str:
    return _lib.cszp2_version().decode()


def _stream(stream) -> int:
    if stream is None:
        return torch.cuda.current_stream().cuda_stream
    if isinstance(stream, torch.cuda.Stream):
        return stream.cuda_stream
    return int(stream)


def _ptr(t: torch.Tensor | None):
    return None if t is None else ctypes.c_void_p(t.data_ptr())


def _check(fn: str, rc: int):
    if rc != OK:
        raise CszpError(fn, rc)


def _need_cuda(*ts):
    """Every given tensor is a CUDA tensor on one device; returns that device."""
    dev = None
    for t in ts:
        if t is None:
            continue
        if not t.is_cuda:
            raise ValueError("cszp2 operates on CUDA tensors only (no CPU fallback)")
        if dev is None:
            dev = t.device
        elif t.device != dev:
            raise ValueError(f"cszp2: tensors on different devices ({dev} and {t.device})")
    return dev


def _dt(t: torch.Tensor) -> int:
    if t.dtype not in _DT:
        raise ValueError(f"cszp2 compresses float32 / float64 tensors, not {t.dtype}")
    return _DT[t.dtype]


def _need_stream_buffer(out: torch.Tensor, n: int, dtype, what="out"):
    """A contiguous byte buffer of at least compress_bound(n) bytes (the kernels write
    payloads up to the bound and their ticket right after it)."""
    if out.dtype != torch.uint8 or not out.is_contiguous():
        raise ValueError(f"{what} must be a contiguous uint8 tensor")
    need = compress_bound(n, dtype)
    if out.numel() < need:
        raise ValueError(f"{what} holds {out.numel()} bytes; compress_bound({n}) = {need}")


def _need_word(t: torch.Tensor | None, dtypes, what):
    if t is not None and (t.dtype not in dtypes or t.numel() < 1 or not t.is_contiguous()):
        raise ValueError(f"{what} must be a contiguous tensor of >= 1 element of {dtypes}")


def _need_values(out: torch.Tensor, count: int, what="out"):
    if out.dtype not in _DT or not out.is_contiguous() or out.numel() != count:
        raise ValueError(f"{what} must be a contiguous float32/float64 tensor of {count} elements")


def compress_bound(n: int, dtype=torch.float32) -> int:
    return int(_lib.cszp2_compress_bound(n, _DT[dtype] if isinstance(dtype, torch.dtype) else dtype))


def compress(x: torch.Tensor, eb: float, eb_mode="abs", enc_mode="plain", out=None, out_bytes=None,
             stream=None):
    """Compress a contiguous CUDA f32/f64 tensor. Returns (stream buffer of
    compress_bound bytes, device uint64-as-int64 tensor holding the stream's
    byte count). Asynchronous on `stream` (default: torch's current stream)."""
    dev = _need_cuda(x, out, out_bytes)
    x = x.contiguous().view(-1)
    dt = _dt(x)
    if out is None:
        out = torch.empty(compress_bound(x.numel(), dt), dtype=torch.uint8, device=x.device)
    if out_bytes is None:
        out_bytes = torch.zeros(1, dtype=torch.int64, device=x.device)
    _need_stream_buffer(out, x.numel(), dt)
    _need_word(out_bytes, (torch.int64, torch.uint64), "out_bytes")
    with torch.cuda.device(dev):
        rc = _lib.cszp2_compress(_ptr(x), x.numel(), dt, float(eb), _EB[eb_mode], _ENC[enc_mode],
                                 _ptr(out), _ptr(out_bytes), _stream(stream))
    _check("cszp2_compress", rc)
    return out, out_bytes


def _need_input(x):
    if not x.is_contiguous():
        raise ValueError("x must be contiguous (the kernels read it as a flat array)")
    return _dt(x)


def compress_prepare(x, eb, eb_mode, out, stream=None):
    """Phase 1 of compress: zero the header; REL: device min/max -> eb_abs in the header."""
    dev = _need_cuda(x, out)
    dt = _need_input(x)
    _need_stream_buffer(out, x.numel(), dt)
    with torch.cuda.device(dev):
        rc = _lib.cszp2_compress_prepare(_ptr(x), x.numel(), dt, float(eb), _EB[eb_mode],
                                         _ptr(out), _stream(stream))
    _check("cszp2_compress_prepare", rc)


def compress_encode(x, eb, eb_mode, enc_mode, out, out_bytes=None, stream=None, prepared=False):
    """Phase 2 of compress: zero the tile index (skipped with prepared=True, when a
    compress_prepare on `out` precedes it), then the fused kernel (repeatable)."""
    compress_encode_ex(x, eb, eb_mode, enc_mode, out, out_bytes, FLAG_PREPARED if prepared else 0, stream,
                       _fn="cszp2_compress_encode")


def value_range(x: torch.Tensor, work=None, stream=None) -> torch.Tensor:
    """Device (min, max) of the non-NaN values of x as float64 (+inf, -inf if none):
    returns an 8-element float64 work tensor whose first two words hold them."""
    dev = _need_cuda(x, work)
    x = x.contiguous().view(-1)
    if work is None:
        work = torch.empty(8, dtype=torch.float64, device=x.device)
    if work.dtype != torch.float64 or work.numel() < 8 or not work.is_contiguous():
        raise ValueError("work must be a contiguous float64 tensor of >= 8 elements")
    with torch.cuda.device(dev):
        rc = _lib.cszp2_value_range(_ptr(x), x.numel(), _dt(x), _ptr(work), _stream(stream))
    _check("cszp2_value_range", rc)
    return work


def compress_prepare_range(x, eb, rng: torch.Tensor, out, stream=None):
    """compress_prepare for REL with a caller-supplied device range rng[0:2] =
    (min, max), e.g. reduced across ranks (global REL); then compress_encode(x, eb,
    "rel", ...)."""
    dev = _need_cuda(x, rng, out)
    if rng.dtype != torch.float64 or rng.numel() < 2 or not rng.is_contiguous():
        raise ValueError("rng must be a contiguous float64 CUDA tensor of >= 2 elements")
    dt = _need_input(x)
    _need_stream_buffer(out, x.numel(), dt)
    with torch.cuda.device(dev):
        rc = _lib.cszp2_compress_prepare_range(_ptr(x), x.numel(), dt, float(eb), _ptr(rng),
                                               _ptr(out), _stream(stream))
    _check("cszp2_compress_prepare_range", rc)


FLAG_CHAINED_SCAN = 1
FLAG_LOAD_VEC = 2
FLAG_LOAD_SCALAR = 4
FLAG_PREPARED = 8  # a prepare on this buffer precedes the encode: skip re-zeroing (include/cszp2.h)
FLAG_LB_WIDE = 16  # lookback first window 256 / 32 predecessors (default: by tile count, 32 below 2^16 tiles)
FLAG_LB_NARROW = 32


def compress_encode_ex(x, eb, eb_mode, enc_mode, out, out_bytes=None, flags=0, stream=None,
                       _fn="cszp2_compress_encode_ex"):
    """compress_encode with ablation flags (FLAG_CHAINED_SCAN: plain chained scan;
    FLAG_LOAD_VEC / FLAG_LOAD_SCALAR: per-thread global loads instead of TMA)."""
    dev = _need_cuda(x, out, out_bytes)
    dt = _need_input(x)
    _need_stream_buffer(out, x.numel(), dt)
    _need_word(out_bytes, (torch.int64, torch.uint64), "out_bytes")
    with torch.cuda.device(dev):
        rc = _lib.cszp2_compress_encode_ex(_ptr(x), x.numel(), dt, float(eb), _EB[eb_mode],
                                           _ENC[enc_mode], _ptr(out), _ptr(out_bytes), flags, _stream(stream))
    _check(_fn, rc)


def decompress(cmp: torch.Tensor, n: int, dtype=torch.float32, out=None, status=None, stream=None):
    """Decompress a device stream into n values. `status` (optional device
    int32 tensor, zeroed by the caller) receives CSZP2_ERR_FORMAT/RANGE bits."""
    dev = _need_cuda(cmp, out, status)
    if out is None:
        out = torch.empty(n, dtype=dtype, device=cmp.device)
    _need_values(out, n)
    _need_word(status, (torch.int32,), "status")
    if cmp.dtype != torch.uint8 or not cmp.is_contiguous():
        raise ValueError("cmp must be a contiguous uint8 tensor")
    with torch.cuda.device(dev):
        rc = _lib.cszp2_decompress(_ptr(cmp), _ptr(out), n, _DT[out.dtype], _ptr(status), _stream(stream))
    _check("cszp2_decompress", rc)
    return out


LOCATE_INDEX, LOCATE_LOOKBACK = 0, 1


def decompress_tilewise(cmp: torch.Tensor, n: int, dtype=torch.float32, locate=LOCATE_LOOKBACK, out=None,
                        scratch=None, status=None, stream=None):
    """Ablation: one-CTA-per-tile decompression locating tiles by a decoupled lookback
    (the paper's decompression-side ❸) or by the persisted tile index."""
    dev = _need_cuda(cmp, out, scratch, status)
    if out is None:
        out = torch.empty(n, dtype=dtype, device=cmp.device)
    if scratch is None:
        scratch = torch.empty(int(_lib.cszp2_decompress_scratch_bytes(n)), dtype=torch.uint8, device=cmp.device)
    _need_values(out, n)
    _need_word(status, (torch.int32,), "status")
    if scratch.numel() * scratch.element_size() < int(_lib.cszp2_decompress_scratch_bytes(n)) or \
            not scratch.is_contiguous():
        raise ValueError("scratch must be contiguous with cszp2_decompress_scratch_bytes(n) bytes")
    with torch.cuda.device(dev):
        rc = _lib.cszp2_decompress_tilewise(_ptr(cmp), _ptr(out), n, _DT[out.dtype], int(locate), _ptr(scratch),
                                            _ptr(status), _stream(stream))
    _check("cszp2_decompress_tilewise", rc)
    return out


def decompress_range(cmp: torch.Tensor, n: int, first: int, count: int, dtype=torch.float32, out=None,
                     status=None, stream=None):
    """Random access: values [first, first+count) of an n-value stream."""
    dev = _need_cuda(cmp, out, status)
    if out is None:
        out = torch.empty(count, dtype=dtype, device=cmp.device)
    _need_values(out, count)
    _need_word(status, (torch.int32,), "status")
    with torch.cuda.device(dev):
        rc = _lib.cszp2_decompress_range(_ptr(cmp), n, _DT[out.dtype], first, count, _ptr(out), _ptr(status),
                                         _stream(stream))
    _check("cszp2_decompress_range", rc)
    return out


def read_header(cmp: torch.Tensor, stream=None) -> dict:
    dev = _need_cuda(cmp)
    if cmp.numel() * cmp.element_size() < 64:
        raise ValueError("a stream starts with a 64-byte header")
    h = Header()
    with torch.cuda.device(dev):
        _check("cszp2_read_header", _lib.cszp2_read_header(_ptr(cmp), ctypes.byref(h), _stream(stream)))
    return h.as_dict()


def compress_host(h_in: torch.Tensor, eb: float, eb_mode, enc_mode, d_in_work, d_out_work,
                  h_out: torch.Tensor, stream=None) -> int:
    """End-to-end from HOST memory: H2D, compress, D2H of the stream. Returns
    the stream's byte count (synchronises)."""
    if h_in.is_cuda or h_out.is_cuda:
        raise ValueError("h_in / h_out are host tensors")
    dev = _need_cuda(d_in_work, d_out_work)
    dt = _dt(h_in)
    if not (h_in.is_contiguous() and h_out.is_contiguous() and h_out.dtype == torch.uint8):
        raise ValueError("h_in must be contiguous, h_out a contiguous uint8 tensor")
    if d_in_work.numel() * d_in_work.element_size() < h_in.numel() * h_in.element_size() or \
            not d_in_work.is_contiguous():
        raise ValueError("d_in_work must hold the input")
    _need_stream_buffer(d_out_work, h_in.numel(), dt, "d_out_work")
    nbytes = ctypes.c_uint64(0)
    with torch.cuda.device(dev):
        rc = _lib.cszp2_compress_host(_ptr(h_in), h_in.numel(), dt, float(eb), _EB[eb_mode],
                                      _ENC[enc_mode], _ptr(d_in_work), _ptr(d_out_work), _ptr(h_out),
                                      h_out.numel(), ctypes.byref(nbytes), _stream(stream))
    _check("cszp2_compress_host", rc)
    return nbytes.value


def decompress_host(h_cmp: torch.Tensor, cmp_bytes: int, d_cmp_work, d_out_work, h_out: torch.Tensor,
                    status=None, stream=None):
    if h_cmp.is_cuda or h_out.is_cuda:
        raise ValueError("h_cmp / h_out are host tensors")
    dev = _need_cuda(d_cmp_work, d_out_work, status)
    _need_word(status, (torch.int32,), "status")
    if h_cmp.numel() * h_cmp.element_size() < cmp_bytes or d_cmp_work.numel() * d_cmp_work.element_size() < cmp_bytes:
        raise ValueError("h_cmp / d_cmp_work hold fewer than cmp_bytes bytes")
    if d_out_work.numel() * d_out_work.element_size() < h_out.numel() * h_out.element_size() or \
            not h_out.is_contiguous():
        raise ValueError("d_out_work must hold the output; h_out must be contiguous")
    with torch.cuda.device(dev):
        rc = _lib.cszp2_decompress_host(_ptr(h_cmp), cmp_bytes, _ptr(d_cmp_work), _ptr(d_out_work),
                                        _ptr(h_out), h_out.numel(), _dt(h_out), _ptr(status),
                                        _stream(stream))
    _check("cszp2_decompress_host", rc)
    return h_out


def container_index(sizes: torch.Tensor, out=None, stream=None):
    """Exclusive scan of per-rank stream sizes (device int64[P]) -> int64[P+1]."""
    dev = _need_cuda(sizes, out)
    if out is None:
        out = torch.empty(sizes.numel() + 1, dtype=torch.int64, device=sizes.device)
    if sizes.dtype not in (torch.int64, torch.uint64) or not sizes.is_contiguous():
        raise ValueError("sizes must be a contiguous int64 tensor")
    if out.dtype not in (torch.int64, torch.uint64) or out.numel() < sizes.numel() + 1 or not out.is_contiguous():
        raise ValueError("out must be a contiguous int64 tensor of len(sizes) + 1 elements")
    with torch.cuda.device(dev):
        _check("cszp2_container_index",
               _lib.cszp2_container_index(_ptr(sizes), sizes.numel(), _ptr(out), _stream(stream)))
    return out


def _extents(shape):
    """(nx, ny, nz, ndim) of a 2D (ny, nx) or 3D (nz, ny, nx) shape, x fastest."""
    shape = tuple(int(v) for v in shape)
    if len(shape) == 2:
        return shape[1], shape[0], 1, 2
    if len(shape) == 3:
        return shape[2], shape[1], shape[0], 3
    raise ValueError("2D or 3D field expected")


def compress_bound_nd(shape, dtype=torch.float32) -> int:
    nx, ny, nz, nd = _extents(shape)
    return int(_lib.cszp2_compress_bound_nd(nx, ny, nz, nd, _DT[dtype] if isinstance(dtype, torch.dtype) else dtype))


def compress_nd(x: torch.Tensor, eb: float, eb_mode="abs", enc_mode="outlier", out=None, out_bytes=None,
                stream=None, flags=0):
    """2D (8x8 blocks) / 3D (4x4x4 blocks) Lorenzo compression of a 2D/3D CUDA
    tensor (last axis fastest; FORMAT.md §7). Returns (buffer, device byte count).
    flags: FLAG_LB_WIDE / FLAG_LB_NARROW force the lookback window (same stream)."""
    dev = _need_cuda(x, out, out_bytes)
    x = x.contiguous()
    nx, ny, nz, nd = _extents(x.shape)
    dt = _dt(x)
    if out is None:
        out = torch.empty(compress_bound_nd(x.shape, dt), dtype=torch.uint8, device=x.device)
    if out_bytes is None:
        out_bytes = torch.zeros(1, dtype=torch.int64, device=x.device)
    if out.dtype != torch.uint8 or not out.is_contiguous() or out.numel() < compress_bound_nd(x.shape, dt):
        raise ValueError("out must be a contiguous uint8 tensor of compress_bound_nd bytes")
    _need_word(out_bytes, (torch.int64, torch.uint64), "out_bytes")
    with torch.cuda.device(dev):
        rc = _lib.cszp2_compress_nd_ex(_ptr(x), nx, ny, nz, nd, dt, float(eb), _EB[eb_mode], _ENC[enc_mode],
                                       _ptr(out), _ptr(out_bytes), int(flags), _stream(stream))
    _check("cszp2_compress_nd", rc)
    return out, out_bytes


def decompress_nd(cmp: torch.Tensor, shape, dtype=torch.float32, out=None, status=None, stream=None):
    """Inverse of compress_nd into a tensor of `shape`."""
    dev = _need_cuda(cmp, out, status)
    nx, ny, nz, nd = _extents(shape)
    if out is None:
        out = torch.empty(tuple(shape), dtype=dtype, device=cmp.device)
    _need_values(out, nx * ny * nz)
    _need_word(status, (torch.int32,), "status")
    with torch.cuda.device(dev):
        rc = _lib.cszp2_decompress_nd(_ptr(cmp), _ptr(out), nx, ny, nz, nd, _DT[out.dtype], _ptr(status),
                                      _stream(stream))
    _check("cszp2_decompress_nd", rc)
    return out
