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


def reduce_range(rng: torch.Tensor, group=None) -> torch.Tensor:
    """Global (min, max) from every rank's (min, max) in rng[0:2] (float64): one
    16-byte all-reduce of (min, -max) with MIN (optional global REL)."""
    t = torch.stack([rng[0], -rng[1]])
    if dist.is_available() and dist.is_initialized():
        dist.all_reduce(t, op=dist.ReduceOp.MIN, group=group)
    return torch.stack([t[0], -t[1]]).contiguous()


def compress_slab(x_slab: torch.Tensor, eb: float, eb_mode: str, enc_mode: str, out=None,
                  nbytes=None, group=None, stream=None, rel_scope: str = "rank"):
    """Compress this rank's slab and build the container index on the device:
    returns (stream buffer, this rank's size tensor, offsets int64[world+1]).

    rel_scope (REL only): "rank" — each rank's own slab range r_s <= r, which still
    meets the dataset-level bound with no extra collective (the default);
    "global" — the whole field's range through one 16-byte all-reduce, so that the
    ranks' offset bytes and payloads concatenate to the single-GPU stream's."""
    from . import (compress, compress_bound, compress_encode, compress_prepare_range,
                   container_index, value_range)

    if rel_scope not in ("rank", "global"):
        raise ValueError("rel_scope must be 'rank' or 'global'")
    x = x_slab.contiguous().view(-1)
    cur = torch.cuda.current_stream(x.device) if stream is None else stream
    # every launch AND both collectives are ordered on `cur`: torch.distributed orders a
    # collective after the current stream's work and the current stream after the
    # collective, so the size all-gather reads d_out_bytes after the compressor wrote it
    # and the container-index kernel reads the sizes after NCCL delivered them
    with torch.cuda.device(x.device), torch.cuda.stream(cur):
        if eb_mode == "rel" and rel_scope == "global":
            if out is None:
                out = torch.empty(compress_bound(x.numel(), x.dtype), dtype=torch.uint8, device=x.device)
            if nbytes is None:
                nbytes = torch.zeros(1, dtype=torch.int64, device=x.device)
            rng = reduce_range(value_range(x, stream=cur), group)
            compress_prepare_range(x, eb, rng, out, stream=cur)
            compress_encode(x, eb, "rel", enc_mode, out, nbytes, stream=cur, prepared=True)
        else:
            out, nbytes = compress(x, eb, eb_mode, enc_mode, out=out, out_bytes=nbytes, stream=cur)
        if dist.is_available() and dist.is_initialized():
            sizes = gather_sizes(nbytes, group)
        else:
            sizes = nbytes.view(1)
        offsets = container_index(sizes, stream=cur)
    return out, nbytes, offsets
