"""Synthetic HPC-shaped fields (see synthetic/__init__.py and DESIGN.md §5).

Recipes (BASELINE.json configs; structure from what PAPER.md says about its
datasets: CESM/HACC-xx/Miranda/S3D are globally smooth,
HACC-vx/QMCPack are not, JetIn is sparse). Noise amplitudes
were calibrated once (scripts/calibrate_fields.py) so that the Outlier-mode CR
at REL 1e-4 lands near the paper's Table III averages (CESM 14.97, HACC 4.84,
NYX 24.12) — a plausibility target, not a parity pin.
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

import numpy as np
import torch

# SplitMix64 constants as signed int64 (two's complement wrap is what we want)
_C1 = 0x9E3779B97F4A7C15 - (1 << 64)
_C2 = 0xBF58476D1CE4E5B9 - (1 << 64)
_C3 = 0x94D049BB133111EB - (1 << 64)


def _lsr(x: torch.Tensor, k: int) -> torch.Tensor:
    """Logical right shift of an int64 tensor."""
    return (x >> k) & ((1 << (64 - k)) - 1)


def _splitmix64(x: torch.Tensor) -> torch.Tensor:
    x = x + _C1
    x = (x ^ _lsr(x, 30)) * _C2
    x = (x ^ _lsr(x, 27)) * _C3
    return x ^ _lsr(x, 31)


def _uniform01(key: torch.Tensor) -> torch.Tensor:
    """(0,1) float64 from the top 24 bits of a hash."""
    h = _splitmix64(key)
    return (_lsr(h, 40).to(torch.float64) + 0.5) * (1.0 / (1 << 24))


def _seed_offset(seed: int) -> int:
    return (int(seed) * 0x9E3779B1) & ((1 << 61) - 1)


def gauss(idx: torch.Tensor, seed: int) -> torch.Tensor:
    """Counter-based N(0,1): Box-Muller over two hashed uniforms of (seed, idx)."""
    base = idx * 2 + _seed_offset(seed)
    u1 = _uniform01(base)
    u2 = _uniform01(base + 1)
    return torch.sqrt(-2.0 * torch.log(u1)) * torch.cos((2.0 * math.pi) * u2)


def uniform_pm1(idx: torch.Tensor, seed: int) -> torch.Tensor:
    return _uniform01(idx * 2 + _seed_offset(seed ^ 0x5A5A) + 1) * 2.0 - 1.0


@dataclass(frozen=True)
class FieldSpec:
    name: str
    shape: tuple
    dtype: torch.dtype
    kind: str
    seed: int
    eb_mode: str  # "abs" | "rel"
    ebs: tuple
    modes: tuple  # subset of ("plain", "outlier")
    params: dict = field(default_factory=dict)

    @property
    def n(self) -> int:
        return int(np.prod(self.shape))

    @property
    def itemsize(self) -> int:
        return 4 if self.dtype == torch.float32 else 8


CONFIGS = {
    # BASELINE.json configs[0]: 1D smooth, ABS 1e-3, Plain
    "cfg1": FieldSpec("smooth1d-1M", (1 << 20,), torch.float32, "smooth1d", 0xC5200001,
                      "abs", (1e-3,), ("plain", "outlier"), {"sigma": 2e-3}),
    # configs[1]: CESM-ATM-shaped 2D 1800x3600
    "cfg2": FieldSpec("cesm-1800x3600", (1800, 3600), torch.float32, "cesm", 0xC5200002,
                      "rel", (1e-2, 1e-3, 1e-4), ("plain", "outlier"), {"sigma": 1e-5, "wave": 0.5, "modes": 0.15}),
    # configs[2]: Hurricane-shaped and NYX-shaped 3D
    "cfg3a": FieldSpec("hurricane-100x500x500", (100, 500, 500), torch.float32, "hurricane",
                       0xC5200003, "rel", (1e-4,), ("outlier",), {"sigma": 2e-3}),
    "cfg3b": FieldSpec("nyx-512^3", (512, 512, 512), torch.float32, "nyx", 0xC5200004,
                       "rel", (1e-4,), ("outlier",), {"sigma": 2e-3, "a": 2.8}),
    # configs[3]: HACC-shaped 1D particle array + f64 NYX
    "cfg4a": FieldSpec("hacc-280953867", (280953867,), torch.float32, "hacc", 0xC5200005,
                       "rel", (1e-4,), ("plain", "outlier"), {"jitter": 0.55}),
    "cfg4b": FieldSpec("nyx-512^3-f64", (512, 512, 512), torch.float64, "nyx", 0xC5200006,
                       "rel", (1e-4,), ("outlier",), {"sigma": 2e-3, "a": 2.8}),
    # configs[4]: 2048^3 slab-sharded across 1/2/4/8 GPUs
    "cfg5": FieldSpec("nyx-2048^3", (2048, 2048, 2048), torch.float32, "nyx", 0xC5200007,
                      "rel", (1e-4,), ("plain", "outlier"), {"sigma": 2e-3, "a": 2.8}),
}


def field_spec(name: str) -> FieldSpec:
    return CONFIGS[name]


def _modes(seed: int, count: int, kmax: int):
    rs = np.random.RandomState(seed & 0x7FFFFFFF)
    k = rs.randint(1, kmax + 1, size=(count, 3)) * rs.choice([-1, 1], size=(count, 3))
    amp = rs.uniform(0.3, 1.0, size=count) / (1.0 + np.abs(k).sum(axis=1) / kmax)
    th = rs.uniform(0, 2 * math.pi, size=count)
    return k, amp, th


def _eval(spec: FieldSpec, idx: torch.Tensor) -> torch.Tensor:
    """float64 field values at global linear indices idx (int64)."""
    p = spec.params
    if spec.kind == "smooth1d":
        i = idx.to(torch.float64)
        return (torch.sin(i * (2 * math.pi / 4096)) + 0.5 * torch.sin(i * (2 * math.pi / 333) + 1.0)
                + p["sigma"] * gauss(idx, spec.seed))
    if spec.kind == "cesm":
        ny, nx = spec.shape
        r = (idx // nx).to(torch.float64)
        c = (idx % nx).to(torch.float64)
        phi = -math.pi / 2 + math.pi * (r + 0.5) / ny
        lam = (2 * math.pi / nx) * c
        v = 250.0 + 40.0 * torch.cos(phi) + p["wave"] * torch.sin(3 * lam) * torch.cos(2 * phi)
        k, amp, th = _modes(spec.seed, 8, 6)
        for m in range(8):
            v = v + p["modes"] * amp[m] * torch.sin(float(abs(k[m, 0])) * lam + float(k[m, 1]) * phi + th[m])
        return v + p["sigma"] * 100.0 * gauss(idx, spec.seed)
    if spec.kind == "hurricane":
        nz, ny, nx = spec.shape
        z = (idx // (ny * nx)).to(torch.float64)
        y = ((idx // nx) % ny).to(torch.float64)
        x = (idx % nx).to(torch.float64)
        cx = nx / 2 + 0.08 * nx * torch.sin(z / 30.0)
        cy = ny / 2 + 0.08 * ny * torch.cos(z / 40.0)
        rr = torch.sqrt((x - cx) ** 2 + (y - cy) ** 2)
        R = 0.08 * nx
        v = 60.0 * (rr / R) * torch.exp(1.0 - rr / R) * (1.0 - 0.8 * z / nz)
        v = v + 3.0 * torch.sin(x * (2 * math.pi / 97) + y * (2 * math.pi / 131) + z * 0.05)
        return v + p["sigma"] * 60.0 * gauss(idx, spec.seed)
    if spec.kind == "nyx":
        N = spec.shape[0]
        i = (idx // (N * N)).to(torch.float64)
        j = ((idx // N) % N).to(torch.float64)
        l = (idx % N).to(torch.float64)
        k, amp, th = _modes(0xC5200004, 16, 4)  # same structure for every NYX-shaped size
        g = torch.zeros_like(i)
        w = 2 * math.pi / N
        for m in range(16):
            g = g + amp[m] * torch.sin(w * (float(k[m, 0]) * i + float(k[m, 1]) * j + float(k[m, 2]) * l) + th[m])
        g = g / math.sqrt(float((amp ** 2).sum()) / 2.0)
        g = g + p["sigma"] * gauss(idx, spec.seed)
        return torch.exp(p["a"] * g)
    if spec.kind == "hacc":
        i = idx
        saw = (i % 65536).to(torch.float64) * (256.0 / 65536.0)
        return saw + p["jitter"] * uniform_pm1(idx, spec.seed)
    raise ValueError(spec.kind)


def make_field(name_or_spec, device="cpu", start: int = 0, count: int | None = None,
               out: torch.Tensor | None = None, chunk: int = 1 << 24) -> torch.Tensor:
    """Values at global linear indices [start, start+count) of a config's field,
    as a 1D tensor of the config's dtype on `device` (generated in chunks)."""
    spec = CONFIGS[name_or_spec] if isinstance(name_or_spec, str) else name_or_spec
    if count is None:
        count = spec.n - start
    if out is None:
        out = torch.empty(count, dtype=spec.dtype, device=device)
    for s in range(0, count, chunk):
        e = min(count, s + chunk)
        idx = torch.arange(start + s, start + e, dtype=torch.int64, device=out.device)
        out[s:e] = _eval(spec, idx).to(spec.dtype)
    return out
