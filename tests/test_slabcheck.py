"""The streaming whole-stream checker (tests/slabcheck.py) itself, on CPU: it must
accept a stream the oracle wrote for the whole field and reject one changed byte
in every region it claims to cover (not gpu; the checker is test infrastructure
for the config-5 and > 4 GiB GPU parity tests)."""
import numpy as np
import pytest
import torch

import oracle
from tests import slabcheck
from tests import streamparse as sp


@pytest.fixture(scope="module")
def case():
    rng = np.random.default_rng(5)
    n = 8192 * 9 + 32 * 7 + 5
    xh = (np.cumsum(rng.standard_normal(n)) * 0.4).astype(np.float32)
    ref, rc = oracle.compress(xh, 1e-3, oracle.REL, oracle.OUTLIER)
    assert rc == oracle.OK
    y, rc = oracle.decompress(ref, n)
    eb_abs = sp.header(ref)["eb_abs"]
    return torch.from_numpy(xh), torch.from_numpy(ref), torch.from_numpy(y), eb_abs


def test_accepts_the_oracle_whole_stream(case):
    x, s, y, eb_abs = case
    assert slabcheck.rel_eb_abs(x, 1e-3, chunk=10000) == eb_abs
    r = slabcheck.slab_parity(x, s, y, oracle.OUTLIER, eb_abs, slab_tiles=4, workers=3)
    assert r["slabs"] == 3 and r["tiles"] == 10


@pytest.mark.parametrize("where", ["index", "offsets", "payload_head", "payload_tail", "pad", "values"])
def test_rejects_one_changed_byte(case, where):
    x, s, y, eb_abs = case
    nb, T, O, D = sp.geometry(x.numel())
    s, y = s.clone(), y.clone()
    pb = sp.header(s.numpy())["payload_bytes"]
    if where == "index":
        s[64 + 8 * 5] ^= 1
    elif where == "offsets":
        s[O + 300] ^= 0x01
    elif where == "payload_head":
        s[D + 3] ^= 0x10
    elif where == "payload_tail":
        s[D + pb - 1] ^= 0x80
    elif where == "pad":
        s[O + nb] = 1
    else:
        y.view(torch.int32)[12345] += 1  # one ulp
    with pytest.raises(AssertionError):
        slabcheck.slab_parity(x, s, y, oracle.OUTLIER, eb_abs, slab_tiles=4, workers=2)
