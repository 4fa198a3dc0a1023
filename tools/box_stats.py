#!/usr/bin/env python
"""NEXT #4 (hierarchical-box BinMD) sizing: for Morton-ordered boxes of B consecutive
events, the fraction that (a) can be skipped -- the box's Q bounding box misses the grid for every
op -- and (b) could be bulk-added -- the box lies inside one bin for an op.  Host-only (numpy, fp64
interval arithmetic on the box corners), on the BASELINE synthetic workloads.

  python tools/box_stats.py [--events 2000000]
"""
import argparse
import itertools
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def box_fractions(wl, ev, N, B):
    n = len(ev) // B * B
    q = ev[:n, 1:].astype(np.float64).reshape(-1, B, 3)
    lo, hi = q.min(axis=1), q.max(axis=1)                  # [nbox, 3]
    corners = np.stack([np.where(np.array(c)[None, :] == 0, lo, hi) for c in itertools.product((0, 1), repeat=3)],
                       axis=1)                           # [nbox, 8, 3]
    skip = np.ones(len(lo), bool)
    bulk_any = np.zeros(len(lo), bool)
    for Nm in N:
        x = corners @ Nm.T                                # [nbox, 8, 3] grid coordinates (linear map)
        xl, xh = x.min(axis=1), x.max(axis=1)
        t_lo = (xl - wl.lo) / ((wl.hi - wl.lo) / wl.nbins)
        t_hi = (xh - wl.lo) / ((wl.hi - wl.lo) / wl.nbins)
        miss = ((t_hi < 0) | (t_lo >= wl.nbins)).any(axis=1)
        skip &= miss
        one_bin = (np.floor(t_lo) == np.floor(t_hi)).all(axis=1) & ~miss
        bulk_any |= one_bin
    return skip.mean(), bulk_any.mean()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--events", type=int, default=2_000_000)
    a = ap.parse_args()
    import oracle
    import synth
    for name, kw in (("corelli", {}), ("topaz", dict(nops=48))):
        wl = synth.make_workload(name, **kw)
        ev = synth.events_for_run(wl, 0, n=a.events)
        N = oracle.binmd_matrices(wl.UB, wl.ops, wl.W)
        for B in (32, 256, 1024):
            s, b = box_fractions(wl, ev, N, B)
            print(f"{name:8s} box {B:5d} events: skippable (misses the grid for every op) {100 * s:6.2f}%  "
                  f"bulk-addable for some op (inside one bin) {100 * b:6.3f}%")


if __name__ == "__main__":
    main()
