"""Seeded synthetic fields shaped like the paper's HPC datasets.

This module holds NONE of the compressor's arithmetic. It is shared by the
tests, bench.py and smoke(); both the CUDA path and the oracle consume the
exact same bits (fields are generated once, on the device or the CPU, and
copied where needed).

Every value is a deterministic function of (config, global linear index), so a
slab of a field generated on rank r is bit-identical regardless of how many
ranks there are (on a given device type). Noise is a counter-based hash
(SplitMix64 of seed ^ index) pushed through Box-Muller.
"""
from .fields import CONFIGS, FieldSpec, make_field, field_spec  # noqa: F401
