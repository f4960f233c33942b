"""Multi-GPU slab sharding of one field (BASELINE config 5).

One process per GPU. Rank r owns the block-aligned contiguous slab
[r*S, min(n, (r+1)*S)), S = ceil(n/P/32)*32, compresses it independently
(blocks never reference neighbours) and the only collective is one
all-gather of the 8-byte compressed sizes; the container index is their
exclusive scan (cszp2_container_index kernel). Decompression needs no
collective.
"""
from __future__ import annotations

import torch
import torch.distributed as dist

L = 32


def slab(n: int, world: int, rank: int) -> tuple[int, int]:
    """(start, count) of rank's slab; start is a multiple of the block size."""
    if world < 1 or not 0 <= rank < world:
        raise ValueError("bad world/rank")
    S = -(-n // world)
    S = -(-S // L) * L
    s0 = min(n, rank * S)
    return s0, min(n, s0 + S) - s0


def gather_sizes(nbytes: torch.Tensor, group=None) -> torch.Tensor:
    """All-gather every rank's 1-element int64 size tensor -> int64[world]
    (NCCL on CUDA tensors; gloo on CPU tensors for the host-side tests)."""
    world = dist.get_world_size(group)
    out = torch.empty(world, dtype=nbytes.dtype, device=nbytes.device)
    if nbytes.is_cuda:
        dist.all_gather_into_tensor(out, nbytes.view(1), group=group)
    else:
        parts = list(out.split(1))
        dist.all_gather(parts, nbytes.view(1), group=group)
        out = torch.cat(parts)
    return out


def compress_slab(x_slab: torch.Tensor, eb: float, eb_mode: str, enc_mode: str, out=None,
                  nbytes=None, group=None, stream=None):
    """Compress this rank's slab and build the container index on the device:
    returns (stream buffer, this rank's size tensor, offsets int64[world+1])."""
    from . import compress, container_index

    out, nbytes = compress(x_slab, eb, eb_mode, enc_mode, out=out, out_bytes=nbytes, stream=stream)
    if dist.is_available() and dist.is_initialized():
        sizes = gather_sizes(nbytes, group)
    else:
        sizes = nbytes.view(1)
    offsets = container_index(sizes, stream=stream)
    return out, nbytes, offsets
