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
