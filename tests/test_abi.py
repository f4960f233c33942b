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

    with pytest.raises(ValueError):
        cz.compress(torch.zeros(10), 1e-3)
