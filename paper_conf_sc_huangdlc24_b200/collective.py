"""Compression-accelerated all-gather (the paper's motivating
use, P:67-77 — "compressing data before [GPU-to-GPU] transfer … reduces the volume
of data", gZCCL-style collectives P:491-495).

Every rank holds an equal-sized shard x_r (n values). Instead of moving n·w bytes
per rank, each rank

  1. compresses its shard with the single-kernel compressor (cszp2_compress),
  2. all-gathers the 8-byte compressed sizes (NCCL, device to device),
  3. all-gathers the compressed streams in slots of the largest size (one NCCL
     all_gather_into_tensor; one 8-byte device->host read to size the slots),
  4. decompresses every rank's stream into its slice of the output.

The result equals all_gather(decompress(compress(x_r))) bit for bit; the bytes on
the wire are world · max_r(stream_r) instead of world · n·w. Error bound: each
shard's own (per-rank REL uses the shard's range, R-21).

The codec is the CUDA one; `codec=` exists so the host-side logic can be tested
with world-size-2 gloo on CPU (tests/test_multi_gloo.py passes a test-only codec).
"""
from __future__ import annotations

from dataclasses import dataclass

import torch
import torch.distributed as dist

from .multi import gather_sizes


@dataclass
class CudaCodec:
    """The product codec: libcszp2 kernels on CUDA tensors."""

    eb: float
    eb_mode: str = "rel"
    enc_mode: str = "outlier"

    def compress(self, x: torch.Tensor, workspace: dict | None = None, stream=None):
        """One fused compression kernel; reuses workspace["cmp"] / ["nbytes"] when given."""
        from . import compress, compress_bound

        ws = {} if workspace is None else workspace
        bound = compress_bound(x.numel(), x.dtype)
        buf = ws.get("cmp")
        if buf is None or buf.numel() < bound or buf.device != x.device:
            buf = ws["cmp"] = torch.empty(bound, dtype=torch.uint8, device=x.device)
            ws["nbytes"] = torch.zeros(1, dtype=torch.int64, device=x.device)
        return compress(x, self.eb, self.eb_mode, self.enc_mode, out=buf[:bound], out_bytes=ws["nbytes"],
                        stream=stream)

    def decompress(self, cmp: torch.Tensor, n: int, out: torch.Tensor, status: torch.Tensor, stream=None):
        """Decode into `out`; `status` (zeroed device int32) receives FORMAT/RANGE bits."""
        from . import decompress

        decompress(cmp, n, out.dtype, out=out, status=status, stream=stream)


def _all_gather_bytes(recv: torch.Tensor, send: torch.Tensor, group=None):
    if send.is_cuda:
        dist.all_gather_into_tensor(recv, send, group=group)
    else:  # gloo (host-logic tests)
        parts = list(recv.split(send.numel()))
        dist.all_gather(parts, send, group=group)
        recv.copy_(torch.cat(parts))


def compressed_all_gather(x: torch.Tensor, eb: float, eb_mode: str = "rel", enc_mode: str = "outlier",
                          group=None, codec=None, out: torch.Tensor | None = None, stats: dict | None = None,
                          workspace: dict | None = None):
    """All-gather equal-sized shards through the compressor. Returns a tensor of
    world·n values (rank order), like all_gather_into_tensor of the lossy shards.
    `stats` (optional dict) receives the per-rank stream sizes and wire bytes.
    `workspace` (optional dict, kept by the caller across calls) holds the compressed
    buffer, the receive buffer and the status words, so repeated calls allocate nothing."""
    codec = codec or CudaCodec(eb, eb_mode, enc_mode)
    x = x.contiguous().view(-1)
    world = dist.get_world_size(group)
    n, w = x.numel(), x.element_size()
    if (n * w) % 16:
        raise ValueError("shard size must be a multiple of 16 bytes (output slices stay 16-byte aligned)")
    if out is None:
        out = torch.empty(world * n, dtype=x.dtype, device=x.device)
    ws = {} if workspace is None else workspace
    buf, nbytes = codec.compress(x, ws)             # 1. one fused compression kernel
    sizes = gather_sizes(nbytes.view(1), group)     # 2. 8 B per rank over NCCL
    slot = (int(sizes.max().item()) + 15) // 16 * 16  # the one host read
    if slot > buf.numel():
        raise RuntimeError("compressed stream larger than its buffer")
    recv = ws.get("recv")
    if recv is None or recv.numel() < world * slot or recv.device != x.device:
        recv = ws["recv"] = torch.empty(world * slot, dtype=torch.uint8, device=x.device)
    recv = recv[: world * slot]
    _all_gather_bytes(recv, buf[:slot], group)      # 3. the compressed payloads
    status = ws.get("status")
    if status is None or status.numel() != world or status.device != x.device:
        status = ws["status"] = torch.zeros(world, dtype=torch.int32, device=x.device)
    else:
        status.zero_()
    for r in range(world):                          # 4. P decompression kernels
        codec.decompress(recv[r * slot:(r + 1) * slot], n, out[r * n:(r + 1) * n], status[r:r + 1])
    bad = [(r, int(v)) for r, v in enumerate(status.tolist()) if v]  # host sync after the decodes
    if bad:
        # a rank's shard was out of range (NaN/Inf, |x/2eb| > 2^30-1: header status RANGE)
        # or its stream did not decode: its slice of `out` is not valid data
        from . import CszpError

        raise CszpError(f"compressed_all_gather: rank {bad[0][0]}'s stream", bad[0][1])
    if stats is not None:
        stats.update(sizes=sizes.tolist(), slot=slot, wire_bytes=world * slot, raw_bytes=world * n * w)
    return out
