"""Multi-threaded driver of the fp64 oracle for the full-size GPU parity tests (test
infrastructure only).  Each host thread calls the unchanged C oracle (ctypes releases the GIL) on
an interleaved pixel shard with its own compensated histogram pair; the partial histograms are
summed in fixed thread order.  The oracle's arithmetic per trajectory is untouched; only the
order in which per-trajectory contributions are added differs from one call (within the 1e-12
per-bin bar: every contribution is >= 0, so there is no cancellation)."""
from __future__ import annotations

import os
from concurrent.futures import ThreadPoolExecutor

import numpy as np

import oracle


def host_threads(cap: int | None = None) -> int:
    try:
        n = len(os.sched_getaffinity(0))
    except AttributeError:  # pragma: no cover
        n = os.cpu_count() or 1
    return max(1, min(n, cap) if cap else n)


def mdnorm(grid, pix_dir, solid, fk, fF, M, charge, k_min, k_max, pix_begin=0, pix_stride=1,
           threads=None, mem_cap_bytes=24 << 30):
    """oracle.mdnorm over pixels pix_begin, pix_begin + pix_stride, ... split over threads."""
    t = threads or host_threads()
    # one (sum, comp) fp64 pair per thread: stay under mem_cap_bytes of host memory
    t = max(1, min(t, mem_cap_bytes // max(1, 16 * grid.nbins)))

    def one(i):
        acc = oracle.Accumulator(grid.nbins)
        oracle.mdnorm(grid, pix_dir, solid, fk, fF, M, charge, k_min, k_max,
                      pix_begin=pix_begin + i * pix_stride, pix_stride=pix_stride * t, acc=acc)
        return acc.value()

    with ThreadPoolExecutor(t) as ex:
        parts = list(ex.map(one, range(t)))
    out = parts[0]
    for p in parts[1:]:
        out = out + p
    return out


def binmd(grid, N, events, threads=None):
    t = threads or host_threads()
    cuts = np.linspace(0, len(events), t + 1).astype(np.int64)

    def one(i):
        return oracle.binmd(grid, N, np.ascontiguousarray(events[cuts[i]:cuts[i + 1]]))

    with ThreadPoolExecutor(t) as ex:
        parts = list(ex.map(one, range(t)))
    out = parts[0]
    for p in parts[1:]:
        out = out + p
    return out
