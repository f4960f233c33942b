"""bench.py's multi-rank launch without a GPU (the driver's own command
form `python bench.py --gpus N` must start N ranks itself): the self-launch re-execs
under torch.distributed.run on 127.0.0.1 and every rank joins the process group."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(args, env=None):
    e = dict(os.environ)
    for k in ("WORLD_SIZE", "RANK", "LOCAL_RANK", "MASTER_ADDR", "MASTER_PORT"):
        e.pop(k, None)
    e.update(env or {})
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], capture_output=True, text=True,
                       timeout=300, env=e, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout  # rank 0 alone prints
    return json.loads(lines[0])


def test_bench_self_launches_n_ranks():
    out = _run(["--gpus", "3", "--launcher-selftest"])
    assert out["n_gpus"] == 3 and out["gpus_arg"] == 3 and out["self_launched"]
    assert sorted(r["rank"] for r in out["ranks"]) == [0, 1, 2]
    assert sorted(r["local_rank"] for r in out["ranks"]) == [0, 1, 2]
    assert len({r["pid"] for r in out["ranks"]}) == 3  # one process per rank
    assert out["max_over_ranks"] == 3.0


def test_bench_single_rank_runs_in_process():
    out = _run(["--gpus", "1", "--launcher-selftest"], env={"WORLD_SIZE": "1", "RANK": "0", "LOCAL_RANK": "0",
                                                            "MASTER_ADDR": "127.0.0.1", "MASTER_PORT": "29731"})
    assert out["n_gpus"] == 1 and not out["self_launched"]
