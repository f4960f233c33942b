"""NEXT #4 measurement: raw NCCL all-gather vs the compressed all-gather
(paper_conf_sc_huangdlc24_b200.collective) of one cfg5 (NYX-like 2048^3) slab per
rank. Launch with torchrun for N>1 (one process per GPU); N=1 runs standalone.
Device time with CUDA events, max over ranks; one JSON line from rank 0."""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

from paper_conf_sc_huangdlc24_b200.collective import compressed_all_gather  # noqa: E402
from synthetic import make_field  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--shard-values", type=int, default=1 << 28)
    ap.add_argument("--eb", type=float, default=1e-4)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    a = ap.parse_args()
    rank, world = int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1))
    local = int(os.environ.get("LOCAL_RANK", 0))
    torch.cuda.set_device(local)
    if "MASTER_ADDR" not in os.environ:
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT="29533")
    dist.init_process_group("nccl", rank=rank, world_size=world, device_id=torch.device(f"cuda:{local}"))
    n = a.shard_values
    x = make_field("cfg5", f"cuda:{local}", rank * n, n)
    raw_out = torch.empty(world * n, dtype=x.dtype, device=x.device)
    cmp_out = torch.empty_like(raw_out)

    def timed(fn):
        for _ in range(a.warmup):
            fn()
        dist.barrier()
        torch.cuda.synchronize()
        s, e = torch.cuda.Event(True), torch.cuda.Event(True)
        s.record()
        for _ in range(a.steps):
            fn()
        e.record()
        torch.cuda.synchronize()
        t = torch.tensor([s.elapsed_time(e) / a.steps], device=x.device)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return t.item() * 1e-3

    stats = {}
    t_raw = timed(lambda: dist.all_gather_into_tensor(raw_out, x))
    t_cmp = timed(lambda: compressed_all_gather(x, a.eb, "rel", "outlier", out=cmp_out, stats=stats))
    err = (cmp_out.double() - raw_out.double()).abs().max().item()
    if rank == 0:
        gathered = world * n * x.element_size()
        print(json.dumps({
            "metric": "all-gather GB/s of uncompressed data (output bytes / device time)",
            "n_gpus": world, "shard_bytes": n * x.element_size(), "workload": "cfg5 slab per rank, REL 1e-4, Outlier",
            "raw_nccl": {"ms": round(t_raw * 1e3, 3), "GBps": round(gathered / t_raw / 1e9, 1)},
            "compressed": {"ms": round(t_cmp * 1e3, 3), "GBps": round(gathered / t_cmp / 1e9, 1),
                           "wire_bytes": stats["wire_bytes"], "raw_bytes": stats["raw_bytes"],
                           "cr_on_wire": round(stats["raw_bytes"] / stats["wire_bytes"], 2)},
            "max_abs_err_vs_raw": err,
        }), flush=True)
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
