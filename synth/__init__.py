"""Seeded synthetic workloads shared by the oracle side (tests/) and the CUDA side (bench.py).

This package holds NO MDNorm/BinMD arithmetic: it only draws instruments, flux tables,
crystal orientations, symmetry-op sets and events (SURVEY.md §8(d) "Synthetic inputs").
"""
from .workloads import (  # noqa: F401
    Workload, make_workload, CONFIGS, hex_6mmm_ops, cubic_ops, lattice_B,
    rot_x, rot_y, rot_z, events_for_run,
)
