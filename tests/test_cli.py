"""The `cszp2` command-line tool (SURVEY §8(b) CLI; csrc/cszp2_cli.cpp): usage and
argument errors here (no CUDA call is made on those paths); a whole run on the GPU,
whose stored stream and reconstruction must equal the oracle's."""
import os
import re
import subprocess

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CLI = os.path.join(ROOT, "paper_conf_sc_huangdlc24_b200", "cszp2")


def setup_module(_):
    """build() makes the tool; build it here if only the library is in place."""
    if not os.access(CLI, os.X_OK):
        import importlib.util

        spec = importlib.util.spec_from_file_location(
            "_cszp2_build", os.path.join(ROOT, "paper_conf_sc_huangdlc24_b200", "_build.py"))
        b = importlib.util.module_from_spec(spec)
        spec.loader.exec_module(b)
        if not os.path.exists(b.LIB):
            b.build()
        b.build_cli()


def run(*args):
    return subprocess.run([CLI, *map(str, args)], capture_output=True, text=True, timeout=300)


def test_cli_usage_and_argument_errors():
    assert os.access(CLI, os.X_OK), "build() must produce the cszp2 tool"
    r = run("--help")
    assert r.returncode == 0 and "usage: cszp2" in r.stdout
    assert run().returncode == 1
    for bad in (["-m", "Q", "-a", "x.f32", "1e-3"], ["-m", "P", "x.f32", "1e-3"],          # mode / no -a|-r
                ["-m", "P", "-a", "x.f32", "0"], ["-m", "P", "-a", "x.f32", "abc"],        # bound
                ["-m", "P", "-a", "-t", "f16", "x.f32", "1e-3"], ["-x", "a.cszp", "10"]):  # dtype / -x form
        r = run(*bad)
        assert r.returncode == 1 and "usage" in r.stderr, bad


@pytest.mark.gpu
@pytest.mark.parametrize("mode,ebflag,eb,dtype", [("O", "-r", 1e-4, np.float32), ("P", "-a", 1e-3, np.float32),
                                                  ("O", "-r", 1e-3, np.float64)])
def test_cli_round_trip_matches_oracle(tmp_path, mode, ebflag, eb, dtype):
    import oracle
    from synthetic import make_field

    n = 5 * 8192 + 32 * 7 + 13
    x = make_field("cfg2", "cpu", 0, n).numpy().astype(dtype)
    ext = "f32" if dtype == np.float32 else "f64"
    src, z, d = tmp_path / f"in.{ext}", tmp_path / "out.cszp", tmp_path / f"rec.{ext}"
    x.tofile(src)
    r = run("-m", mode, ebflag, src, eb, "-z", z, "-d", d, "-w", 1, "-k", 2)
    assert r.returncode == 0, r.stdout + r.stderr
    assert "Pass error check!" in r.stdout
    assert re.search(r"compression\s+end-to-end speed: [0-9.]+ GB/s", r.stdout)
    ref, rc = oracle.compress(x, eb, oracle.REL if ebflag == "-r" else oracle.ABS,
                              oracle.OUTLIER if mode == "O" else oracle.PLAIN)
    assert rc == oracle.OK
    np.testing.assert_array_equal(np.fromfile(z, np.uint8), ref)           # stored stream
    cr = float(re.search(r"compression ratio: ([0-9.]+)", r.stdout).group(1))
    assert abs(cr - x.nbytes / ref.size) < 1e-4 * cr
    yr, _ = oracle.decompress(ref, n, dtype)
    iv = np.uint32 if dtype == np.float32 else np.uint64
    np.testing.assert_array_equal(np.fromfile(d, dtype).view(iv), yr.view(iv))  # reconstruction
    back = tmp_path / f"back.{ext}"
    r = run("-x", z, n, "-t", ext, back)                                    # stored-stream decode
    assert r.returncode == 0, r.stderr
    np.testing.assert_array_equal(np.fromfile(back, dtype).view(iv), yr.view(iv))
