"""World-size-2 gloo tests of the N>1 host logic (CPU, no GPU): slab partition,
the all-gather of compressed sizes, container offsets, and that the per-rank
streams' offset bytes / payloads concatenate to the single-stream ones
(block independence). The per-slab compressor here is the oracle
(test infrastructure); the CUDA path runs the same logic in bench.py."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from tests import streamparse as sp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, n, eb, enc, result_q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        from paper_conf_sc_huangdlc24_b200.multi import gather_sizes, slab
        from synthetic import make_field

        s0, cnt = slab(n, world, rank)
        x = make_field("cfg2", "cpu", s0, cnt).numpy()
        s, rc = oracle.compress(x, eb, oracle.ABS, enc)
        sizes = gather_sizes(torch.tensor([s.size], dtype=torch.int64))
        offsets = np.concatenate([[0], np.cumsum(sizes.numpy())])
        streams = [None] * world
        dist.all_gather_object(streams, s.tobytes())
        result_q.put((rank, s0, cnt, rc, sizes.tolist(), offsets.tolist(), streams if rank == 0 else None))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("enc", [0, 1])
def test_two_rank_slabs_concatenate_to_single_stream(orc, enc):
    world, n, eb = 2, 3 * 8192 + 32 * 7 + 5, 1e-3
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, n, eb, enc, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted([q.get(timeout=120) for _ in range(world)])
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    # slabs: contiguous, block-aligned, cover [0, n)
    assert res[0][1] == 0 and res[0][1] + res[0][2] == res[1][1] and res[1][1] + res[1][2] == n
    assert res[1][1] % 32 == 0
    assert all(r[3] == orc.OK for r in res)
    streams = [np.frombuffer(b, np.uint8) for b in res[0][6]]
    sizes = res[0][4]
    assert sizes == [s.size for s in streams] and res[1][4] == sizes  # every rank sees the same sizes
    assert res[0][5] == [0, sizes[0], sizes[0] + sizes[1]]
    # block independence: per-rank offset bytes and payloads concatenate to the P=1 stream's
    from synthetic import make_field

    full, _ = orc.compress(make_field("cfg2", "cpu", 0, n).numpy(), eb, orc.ABS, enc)
    pf = sp.parse(full)
    parts = [sp.parse(s) for s in streams]
    np.testing.assert_array_equal(np.concatenate([p["offsets"] for p in parts]), pf["offsets"])
    _, _, _, D = pf["geometry"]
    pay = lambda s, p: s[p["geometry"][3]:p["geometry"][3] + p["header"]["payload_bytes"]]
    np.testing.assert_array_equal(np.concatenate([pay(s, p) for s, p in zip(streams, parts)]),
                                  pay(full, pf))
    np.testing.assert_array_equal(np.concatenate([p["q"] for p in parts]), pf["q"])


def test_slab_edge_cases():
    from paper_conf_sc_huangdlc24_b200.multi import slab

    for n in (0, 1, 31, 33, 1000, 2**33):
        for world in (1, 2, 4, 8):
            spans = [slab(n, world, r) for r in range(world)]
            assert spans[0][0] == 0
            assert sum(c for _, c in spans) == n
            for (a, c), (b, _) in zip(spans, spans[1:]):
                assert a + c == b
                assert b % 32 == 0 or b == n
    assert slab(2**33, 8, 3) == (3 * 2**30, 2**30)


class _OracleCodec:
    """Test-only codec for the host logic of the compressed all-gather on CPU: the
    oracle behind the same (compress, decompress) interface as CudaCodec."""

    def __init__(self, eb, eb_mode, enc):
        self.eb, self.eb_mode, self.enc = eb, eb_mode, enc

    def compress(self, x, workspace=None):
        import oracle

        s, rc = oracle.compress(x.numpy(), self.eb, self.eb_mode, self.enc)
        assert rc in (oracle.OK, oracle.ERR_RANGE)  # a RANGE stream is still a stream
        buf = torch.zeros(oracle.compress_bound(x.numel()) + 16, dtype=torch.uint8)
        buf[: s.size] = torch.from_numpy(s)
        return buf, torch.tensor([s.size], dtype=torch.int64)

    def decompress(self, cmp, n, out, status, stream=None):
        import oracle

        y, rc = oracle.decompress(cmp.numpy(), n, np.float32 if out.dtype == torch.float32 else np.float64)
        status.fill_(rc)
        if rc == oracle.OK:
            out.copy_(torch.from_numpy(y))


def _cag_worker(rank, world, port, n, eb, enc, result_q, nan_rank=-1):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_sc_huangdlc24_b200 import CszpError
        from paper_conf_sc_huangdlc24_b200.collective import compressed_all_gather
        from synthetic import make_field

        x = make_field("cfg2", "cpu", rank * n, n)  # shard r of one field
        if rank == nan_rank:
            x[n // 3] = float("nan")
        stats = {}
        try:
            y = compressed_all_gather(x, eb, "rel", "outlier", codec=_OracleCodec(eb, 1, enc), stats=stats)
        except CszpError as e:
            result_q.put((rank, "error", str(e)))
            return
        result_q.put((rank, y.numpy().tobytes(), stats))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("enc", [0, 1])
def test_compressed_all_gather_two_ranks(orc, enc):
    """NEXT #4 host logic: sizes all-gathered, payloads gathered in max-size slots,
    every rank ends with the same world·n values = each shard's lossy round trip."""
    world, n, eb = 2, 3 * 8192 + 32 * 7 + 4, 1e-4
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_cag_worker, args=(r, world, port, n, eb, enc, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted([q.get(timeout=120) for _ in range(world)], key=lambda r: r[0])
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    from synthetic import make_field

    expect, sizes = [], []
    for r in range(world):
        x = make_field("cfg2", "cpu", r * n, n).numpy()
        s, rc = orc.compress(x, eb, orc.REL, enc)
        sizes.append(s.size)
        y, rc = orc.decompress(s, n, np.float32)
        expect.append(y)
    expect = np.concatenate(expect)
    for rank, yb, stats in res:
        np.testing.assert_array_equal(np.frombuffer(yb, np.float32).view(np.uint32), expect.view(np.uint32))
        assert stats["sizes"] == sizes
        assert stats["slot"] == (max(sizes) + 15) // 16 * 16
        assert stats["wire_bytes"] == world * stats["slot"] < stats["raw_bytes"]


def test_compressed_all_gather_reports_a_bad_shard(orc):
    """A shard whose stream has RANGE status (a NaN, FORMAT.md §6.3) must not come back
    as data: every rank raises CszpError naming that rank."""
    world, n, eb = 2, 2 * 8192 + 32, 1e-4
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_cag_worker, args=(r, world, port, n, eb, 1, q, 1)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted([q.get(timeout=120) for _ in range(world)], key=lambda r: r[0])
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, kind, msg in res:
        assert kind == "error" and "rank 1" in msg and "status 3" in msg


def _grel_worker(rank, world, port, n, lam, enc, result_q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        from paper_conf_sc_huangdlc24_b200.multi import reduce_range, slab
        from synthetic import make_field

        s0, cnt = slab(n, world, rank)
        x = make_field("cfg2", "cpu", s0, cnt).numpy()
        local = torch.tensor([np.nanmin(x).astype(np.float64), np.nanmax(x).astype(np.float64)])
        rng = reduce_range(local)  # the product's 16-byte all-reduce (gloo here, NCCL on GPUs)
        eb_abs = lam * (float(rng[1]) - float(rng[0]))  # FORMAT.md §6.1 on the global range
        s, rc = oracle.compress(x, eb_abs, oracle.ABS, enc)
        result_q.put((rank, rc, rng.tolist(), local.tolist(), eb_abs, s.tobytes()))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("enc", [0, 1])
def test_global_rel_two_ranks_matches_single_stream(orc, enc):
    """SURVEY §8(e) optional global REL: the reduced range is the field's, so every
    rank quantizes with the single-GPU eb_abs and the ranks' offset bytes and
    payloads concatenate to the REL stream of the whole field."""
    world, n, lam = 2, 5 * 8192 + 32 * 3 + 9, 1e-3
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_grel_worker, args=(r, world, port, n, lam, enc, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted([q.get(timeout=120) for _ in range(world)])
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    from synthetic import make_field

    full_x = make_field("cfg2", "cpu", 0, n).numpy()
    full, rc = orc.compress(full_x, lam, orc.REL, enc)
    assert rc == orc.OK and all(r[1] == orc.OK for r in res)
    gmin, gmax = float(np.nanmin(full_x)), float(np.nanmax(full_x))
    for r in res:
        assert r[2] == [gmin, gmax]                       # every rank holds the global range
        assert r[3][0] >= gmin and r[3][1] <= gmax
    pf = sp.parse(full)
    assert pf["header"]["eb_abs"] == res[0][4] == res[1][4]
    parts = [sp.parse(np.frombuffer(r[5], np.uint8)) for r in res]
    np.testing.assert_array_equal(np.concatenate([p["offsets"] for p in parts]), pf["offsets"])
    np.testing.assert_array_equal(np.concatenate([p["q"] for p in parts]), pf["q"])
