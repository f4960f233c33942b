"""C-ABI library checks that need no GPU: libcszp2.so loads, exports every
function include/cszp2.h declares, and pure host helpers agree with FORMAT.md."""
import os
import re
import subprocess

import pytest

from tests import streamparse as sp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    txt = open(os.path.join(ROOT, "include", "cszp2.h")).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(cszp2_[a-z_0-9]+)\s*\(", txt)))


def test_library_exports_every_declared_symbol():
    import paper_conf_sc_huangdlc24_b200 as cz

    out = subprocess.check_output(["nm", "-D", "--defined-only", cz.LIBRARY_PATH], text=True)
    exported = {l.split()[-1] for l in out.splitlines() if " T " in l}
    declared = _declared()
    assert declared, "no declarations parsed"
    missing = [s for s in declared if s not in exported]
    assert not missing, missing
    assert set(cz.EXPORTED) == set(declared)


def test_library_is_sm100a():
    import paper_conf_sc_huangdlc24_b200 as cz

    out = subprocess.check_output(["/usr/local/cuda/bin/cuobjdump", "--list-elf", cz.LIBRARY_PATH], text=True)
    assert "sm_100a" in out
    assert cz.version().endswith("sm_100a")


@pytest.mark.parametrize("n", [0, 1, 31, 32, 33, 8192, 8193, 1 << 20, 280953867, 1 << 33])
def test_compress_bound_matches_format(n):
    import paper_conf_sc_huangdlc24_b200 as cz

    nb, T, O, D = sp.geometry(n)
    assert cz.compress_bound(n, cz.F32) == sp.roundup16(D + 128 * nb) + 16  # + ticket scratch
    assert cz.compress_bound(n, cz.F64) == sp.roundup16(D + 128 * nb) + 16
    assert cz.compress_bound(n, 7) == 0


def test_cpu_tensors_are_rejected():
    """No CPU fallback: the binding refuses host tensors instead of computing."""
    import torch

    import paper_conf_sc_huangdlc24_b200 as cz

    x = torch.zeros(10)
    buf = torch.zeros(cz.compress_bound(10), dtype=torch.uint8)
    nb = torch.zeros(1, dtype=torch.int64)
    calls = [
        lambda: cz.compress(x, 1e-3),
        lambda: cz.compress_prepare(x, 1e-3, "rel", buf),
        lambda: cz.compress_encode(x, 1e-3, "rel", "outlier", buf, nb),
        lambda: cz.compress_encode_ex(x, 1e-3, "abs", "plain", buf, nb, flags=1),
        lambda: cz.compress_prepare_range(x, 1e-3, torch.zeros(2, dtype=torch.float64), buf),
        lambda: cz.value_range(x),
        lambda: cz.decompress(buf, 10),
        lambda: cz.decompress_range(buf, 10, 0, 5),
        lambda: cz.decompress_tilewise(buf, 10),
        lambda: cz.read_header(buf),
        lambda: cz.container_index(nb),
        lambda: cz.compress_nd(torch.zeros(4, 4), 1e-3),
        lambda: cz.decompress_nd(buf, (4, 4)),
        lambda: cz.compress_host(x, 1e-3, "abs", "plain", x, buf, buf),
    ]
    for i, c in enumerate(calls):
        with pytest.raises(ValueError):
            c()


def test_nd_extent_limit_matches_1d():
    """One size limit for every entry point: nx*ny*nz <= 2^35 values, as the
    1D n <= 2^35; beyond it the nD bound is 0 (invalid) for compression and the same
    geometry is rejected by decompression (checked on the GPU by the ABI test)."""
    import paper_conf_sc_huangdlc24_b200 as cz

    assert cz.compress_bound_nd((2 ** 11, 2 ** 12, 2 ** 12)) > 0          # 2^35 values
    assert cz.compress_bound_nd((2 ** 11, 2 ** 12, 2 ** 12 + 4)) == 0      # just past 2^35
    assert cz.compress_bound_nd((2 ** 17, 2 ** 18)) > 0                    # 2D, 2^35
    assert cz.compress_bound_nd((2 ** 17 + 1, 2 ** 18)) == 0
    assert cz.compress_bound(2 ** 35) > 0
