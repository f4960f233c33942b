"""NEXT #4 on the GPU: compressed all-gather through the CUDA codec and NCCL
(world size 1 here: the round-end box has one GPU; the N>1 host logic is
covered by tests/test_multi_gloo.py). The gathered values must equal the
oracle's lossy round trip of the shard bit for bit."""
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist

pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import oracle  # noqa: E402
from paper_conf_sc_huangdlc24_b200.collective import compressed_all_gather  # noqa: E402
from synthetic import make_field  # noqa: E402


@pytest.fixture(scope="module")
def nccl_group():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    torch.cuda.set_device(0)
    dist.init_process_group("nccl", init_method=f"tcp://127.0.0.1:{port}", rank=0, world_size=1,
                            device_id=torch.device("cuda:0"))
    yield
    dist.destroy_process_group()


@pytest.mark.parametrize("enc", ["plain", "outlier"])
def test_compressed_all_gather_world1(nccl_group, enc):
    n = 5 * 8192 + 32 * 3 + 12
    x = make_field("cfg2", "cuda:0", 0, n)
    stats = {}
    y = compressed_all_gather(x, 1e-4, "rel", enc, stats=stats)
    torch.cuda.synchronize()
    s, rc = oracle.compress(x.cpu().numpy(), 1e-4, oracle.REL, oracle.OUTLIER if enc == "outlier" else oracle.PLAIN)
    assert rc == oracle.OK and stats["sizes"] == [s.size]
    yr, rc = oracle.decompress(s, n, np.float32)
    np.testing.assert_array_equal(y.cpu().numpy().view(np.uint32), yr.view(np.uint32))
    assert stats["wire_bytes"] < stats["raw_bytes"]


# ---- SURVEY §8(e) optional global REL (cszp2_value_range + cszp2_compress_prepare_range)
import paper_conf_sc_huangdlc24_b200 as cz  # noqa: E402
from paper_conf_sc_huangdlc24_b200.multi import compress_slab, slab  # noqa: E402
from tests import streamparse as sp  # noqa: E402


def test_compressed_all_gather_reuses_its_workspace(nccl_group):
    """With a caller-kept workspace, repeated calls reuse the compressed, receive and
    status buffers (same storage) and still return the oracle's round trip."""
    n = 3 * 8192 + 32 * 3 + 12
    ws = {}
    ptrs = None
    for seed in range(3):
        x = make_field("cfg2", "cuda:0", seed * n, n)
        y = compressed_all_gather(x, 1e-4, "rel", "outlier", workspace=ws)
        torch.cuda.synchronize()
        s, rc = oracle.compress(x.cpu().numpy(), 1e-4, oracle.REL, oracle.OUTLIER)
        yr, rc2 = oracle.decompress(s, n)
        np.testing.assert_array_equal(y.cpu().numpy().view(np.uint32), yr.view(np.uint32))
        p = (ws["cmp"].data_ptr(), ws["recv"].data_ptr(), ws["status"].data_ptr())
        if ptrs is not None:
            assert p[0] == ptrs[0] and p[2] == ptrs[2]  # same compressed buffer and status words
        ptrs = p


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_value_range_exact(dtype):
    rng = np.random.default_rng(7)
    for n in (0, 1, 37, 8192 * 40 + 5, 3 * 2**20 + 11):  # both reduction kernels, ragged tails
        xh = (rng.standard_normal(n) * 1e3).astype(dtype)
        if n > 40:
            xh[rng.integers(0, n, 5)] = np.nan
        w = cz.value_range(torch.from_numpy(xh).cuda()).cpu().numpy()
        if n == 0:
            assert w[0] == np.inf and w[1] == -np.inf
        else:
            assert w[0] == float(np.nanmin(xh)) and w[1] == float(np.nanmax(xh))
    w = cz.value_range(torch.full((1000,), np.nan, dtype=torch.float32, device="cuda")).cpu().numpy()
    assert w[0] == np.inf and w[1] == -np.inf


@pytest.mark.parametrize("enc", ["plain", "outlier"])
@pytest.mark.parametrize("dtype", [torch.float32, torch.float64])
def test_prepare_range_with_own_range_is_rel(enc, dtype):
    """prepare_range fed the field's own range == the ordinary REL stream, byte for byte."""
    n = 9 * 8192 + 32 * 5 + 3
    x = make_field("cfg2", "cuda:0", 0, n).to(dtype)
    ref, nb_ref = cz.compress(x, 1e-3, "rel", enc)
    out = torch.full_like(ref, 0xAA)
    nb = torch.zeros(1, dtype=torch.int64, device="cuda")
    cz.compress_prepare_range(x, 1e-3, cz.value_range(x), out)
    cz.compress_encode(x, 1e-3, "rel", enc, out, nb)
    torch.cuda.synchronize()
    assert int(nb.item()) == int(nb_ref.item())
    assert torch.equal(out[: int(nb.item())], ref[: int(nb.item())])


@pytest.mark.parametrize("enc", ["plain", "outlier"])
def test_global_rel_slabs_concatenate_to_oracle_stream(enc):
    """Four slabs with the reduced (global) range: their offset bytes and payloads
    concatenate to the oracle's REL stream of the whole field."""
    n, lam, world = 7 * 8192 + 32 * 9 + 21, 1e-4, 4
    x = make_field("cfg3a", "cuda:0", 0, n)
    spans = [slab(n, world, r) for r in range(world)]
    ranges = [cz.value_range(x[s0:s0 + c]) for s0, c in spans]
    g = torch.stack([torch.stack([w[0] for w in ranges]).min(), torch.stack([w[1] for w in ranges]).max()])
    parts = []
    for s0, c in spans:
        xs = x[s0:s0 + c]
        out = torch.full((cz.compress_bound(c),), 0xAA, dtype=torch.uint8, device="cuda")
        nb = torch.zeros(1, dtype=torch.int64, device="cuda")
        cz.compress_prepare_range(xs, lam, g.contiguous(), out)
        cz.compress_encode(xs, lam, "rel", enc, out, nb)
        torch.cuda.synchronize()
        parts.append(sp.parse(out[: int(nb.item())].cpu().numpy()))
    full, rc = oracle.compress(x.cpu().numpy(), lam, oracle.REL, oracle.OUTLIER if enc == "outlier" else oracle.PLAIN)
    assert rc == oracle.OK
    pf = sp.parse(full)
    assert all(p["header"]["eb_abs"] == pf["header"]["eb_abs"] for p in parts)
    np.testing.assert_array_equal(np.concatenate([p["offsets"] for p in parts]), pf["offsets"])
    np.testing.assert_array_equal(np.concatenate([p["q"] for p in parts]), pf["q"])


def test_compress_slab_global_rel_world1(nccl_group):
    """multi.compress_slab(rel_scope='global') through NCCL (world 1) == the oracle stream."""
    n = 3 * 8192 + 32 * 2 + 7
    x = make_field("cfg2", "cuda:0", 0, n)
    out, nb, offs = compress_slab(x, 1e-3, "rel", "outlier", rel_scope="global")
    torch.cuda.synchronize()
    s, rc = oracle.compress(x.cpu().numpy(), 1e-3, oracle.REL, oracle.OUTLIER)
    assert rc == oracle.OK and int(nb.item()) == s.size
    np.testing.assert_array_equal(out[: s.size].cpu().numpy(), s)
    assert offs.cpu().tolist() == [0, s.size]


@pytest.mark.parametrize("scope", ["rank", "global"])
def test_compress_slab_on_a_side_stream(nccl_group, scope):
    """compress_slab(stream=s) orders the compressor, the size all-gather (NCCL) and the
    container-index kernel on `s`: with a side stream whose queue is kept
    busy ahead of the call, the offsets still read the stream's final size."""
    n = 40 * 8192 + 32 * 5 + 3
    x = make_field("cfg2", "cuda:0", 0, n)
    side = torch.cuda.Stream()
    busy = torch.empty(1 << 26, device="cuda:0")
    with torch.cuda.stream(side):
        for _ in range(8):
            busy.mul_(1.0001)  # queue work ahead of the compressor on the side stream
    out, nb, offs = compress_slab(x, 1e-3, "rel", "outlier", stream=side, rel_scope=scope)
    torch.cuda.synchronize()
    s, rc = oracle.compress(x.cpu().numpy(), 1e-3, oracle.REL, oracle.OUTLIER)
    assert rc == oracle.OK and int(nb.item()) == s.size
    np.testing.assert_array_equal(out[: s.size].cpu().numpy(), s)
    assert offs.cpu().tolist() == [0, s.size]
