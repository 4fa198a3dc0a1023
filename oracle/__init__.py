"""Python (ctypes) front end of the plain fp64 CPU oracle (oracle.c).

TEST INFRASTRUCTURE ONLY: imported by tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / --impl reference legs.  The product package never imports it, and it never
imports the product package.

Parity status per function (DESIGN.md §3 lists the pins):
  compose_mdnorm / compose_binmd  -- pinned (identity/rotation closed forms, Bragg condition)
  flux                            -- pinned (knots, uniform closed form, monotonicity)
  mdnorm / mdnorm_trajectory      -- pinned (axis-aligned closed forms, ties, brute force,
                                     telescoping, op invariances, P:114 bound)
  binmd / binmd_bins              -- pinned (bin centres, full-cover totals, brute force)
  cross_section                   -- pinned (flat-S(Q) statistical test, NaN mask)
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
import time

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
CFLAGS = ["-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared"]


def build(force: bool = False) -> str:
    """Compile oracle.c with gcc (building the checker is not using it)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < max(
            os.path.getmtime(_SRC), os.path.getmtime(os.path.join(_HERE, "oracle.h"))):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


class _Grid(C.Structure):
    _fields_ = [("lo", C.c_double * 3), ("hi", C.c_double * 3), ("n", C.c_int64 * 3)]


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = C.CDLL(build())
        P = C.c_void_p
        i64, i32, d = C.c_int64, C.c_int32, C.c_double
        _lib.orc_compose_mdnorm.argtypes = [P, P, P, P, P]
        _lib.orc_compose_binmd.argtypes = [P, P, P, P]
        _lib.orc_flux.argtypes = [i64, P, P, d]
        _lib.orc_flux.restype = d
        _lib.orc_mdnorm.argtypes = [P, i64, P, P, i64, P, P, i32, P, P, d, d, i64, i64, i64, P, P]
        _lib.orc_mdnorm.restype = i64
        _lib.orc_mdnorm_trajectory.argtypes = [P, P, d, i64, P, P, P, d, d, d, P, P, P, i64]
        _lib.orc_mdnorm_trajectory.restype = i32
        _lib.orc_binmd.argtypes = [P, i32, P, i64, P, i64, i32, i32, P, P]
        _lib.orc_binmd.restype = i64
        _lib.orc_binmd_bins.argtypes = [P, i32, P, i64, P, i64, i32, i32, P]
        _lib.orc_cross_section.argtypes = [i64, P, P, P]
        _lib.orc_mdnorm_krange.argtypes = [P, i64, P, P, P, P, i64, P, P, i32, P, P, d, d, i64, i64, i64,
                                           P, P]
        _lib.orc_mdnorm_krange.restype = i64
        _lib.orc_mdnorm_tables.argtypes = [P, i64, P, P, P, P, i32, P, P, P, P, i32, P, P, d, d, i64, i64,
                                           i64, P, P]
        _lib.orc_mdnorm_tables.restype = i64
        _lib.orc_binmd_err.argtypes = [P, i32, P, i64, P, i64, i32, i32, P, P]
        _lib.orc_binmd_err.restype = i64
        _lib.orc_cross_section_err.argtypes = [i64, P, P, P]
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data_as(C.c_void_p)


def _f64(a) -> np.ndarray:
    return np.ascontiguousarray(a, dtype=np.float64)


class Grid:
    """Uniform half-open grid [lo, hi) with n bins per axis, first axis fastest (reading #4)."""

    def __init__(self, lo, hi, n):
        self.lo = [float(x) for x in lo]
        self.hi = [float(x) for x in hi]
        self.n = [int(x) for x in n]
        self._c = _Grid((C.c_double * 3)(*self.lo), (C.c_double * 3)(*self.hi),
                        (C.c_int64 * 3)(*self.n))

    @property
    def nbins(self) -> int:
        return self.n[0] * self.n[1] * self.n[2]

    @property
    def ref(self):
        return C.byref(self._c)


def compose_mdnorm(R, UB, S, W) -> np.ndarray:
    out = np.empty(9)
    if lib().orc_compose_mdnorm(_p(_f64(R)), _p(_f64(UB)), _p(_f64(S)), _p(_f64(W)), _p(out)):
        raise ValueError("singular R*UB*S*W")
    return out.reshape(3, 3)


def compose_binmd(UB, S, W) -> np.ndarray:
    out = np.empty(9)
    if lib().orc_compose_binmd(_p(_f64(UB)), _p(_f64(S)), _p(_f64(W)), _p(out)):
        raise ValueError("singular UB*S*W")
    return out.reshape(3, 3)


def mdnorm_matrices(R_list, UB, ops, W) -> np.ndarray:
    """[nruns*nops, 3, 3] matrices, run-major (m = r * nops + s)."""
    return np.stack([compose_mdnorm(R, UB, S, W) for R in R_list for S in ops])


def binmd_matrices(UB, ops, W) -> np.ndarray:
    return np.stack([compose_binmd(UB, S, W) for S in ops])


def flux(fk, fF, x: float) -> float:
    fk, fF = _f64(fk), _f64(fF)
    return lib().orc_flux(len(fk), _p(fk), _p(fF), float(x))


class Accumulator:
    """Compensated fp64 histogram pair (sum, comp); value() = sum + comp."""

    def __init__(self, nbins: int):
        self.sum = np.zeros(nbins)
        self.comp = np.zeros(nbins)

    def value(self) -> np.ndarray:
        return self.sum + self.comp


def mdnorm(grid: Grid, pix_dir, solid, fk, fF, M, charge, k_min, k_max,
           pix_begin=0, pix_end=None, pix_stride=1, acc: Accumulator | None = None) -> np.ndarray:
    """norm histogram (nbins) for matrices M [nmat,3,3] with charge[nmat]."""
    d, s, fk, fF = _f64(pix_dir), _f64(solid), _f64(fk), _f64(fF)
    M = _f64(M).reshape(-1, 9)
    charge = _f64(np.broadcast_to(np.asarray(charge, dtype=np.float64), (len(M),)))
    acc = acc or Accumulator(grid.nbins)
    pix_end = len(s) if pix_end is None else pix_end
    lib().orc_mdnorm(grid.ref, len(s), _p(d), _p(s), len(fk), _p(fk), _p(fF), len(M), _p(M),
                     _p(charge), float(k_min), float(k_max), int(pix_begin), int(pix_end),
                     int(pix_stride), _p(acc.sum), _p(acc.comp))
    return acc.value()


def mdnorm_krange(grid: Grid, pix_dir, solid, pix_kmin, pix_kmax, fk, fF, M, charge, k_min, k_max,
                  pix_begin=0, pix_end=None, pix_stride=1, acc: Accumulator | None = None) -> np.ndarray:
    """mdnorm with per-pixel momentum limits (None = no limit on that side)."""
    d, s, fk, fF = _f64(pix_dir), _f64(solid), _f64(fk), _f64(fF)
    lo = None if pix_kmin is None else _f64(pix_kmin)
    hi = None if pix_kmax is None else _f64(pix_kmax)
    M = _f64(M).reshape(-1, 9)
    charge = _f64(np.broadcast_to(np.asarray(charge, dtype=np.float64), (len(M),)))
    acc = acc or Accumulator(grid.nbins)
    pix_end = len(s) if pix_end is None else pix_end
    lib().orc_mdnorm_krange(grid.ref, len(s), _p(d), _p(s), None if lo is None else _p(lo),
                            None if hi is None else _p(hi), len(fk), _p(fk), _p(fF), len(M), _p(M),
                            _p(charge), float(k_min), float(k_max), int(pix_begin), int(pix_end),
                            int(pix_stride), _p(acc.sum), _p(acc.comp))
    return acc.value()


def mdnorm_tables(grid: Grid, pix_dir, solid, tables, pixel_table, M, charge, k_min, k_max,
                  pix_kmin=None, pix_kmax=None, pix_begin=0, pix_end=None, pix_stride=1,
                  acc: Accumulator | None = None) -> np.ndarray:
    """mdnorm with per-bank flux tables: tables = [(k, F), ...], pixel_table[p] = table index."""
    d, s = _f64(pix_dir), _f64(solid)
    fk = _f64(np.concatenate([t[0] for t in tables]))
    fF = _f64(np.concatenate([t[1] for t in tables]))
    offs = np.ascontiguousarray(np.concatenate([[0], np.cumsum([len(t[0]) for t in tables])]), dtype=np.int64)
    pt = None if pixel_table is None else np.ascontiguousarray(pixel_table, dtype=np.int32)
    lo = None if pix_kmin is None else _f64(pix_kmin)
    hi = None if pix_kmax is None else _f64(pix_kmax)
    M = _f64(M).reshape(-1, 9)
    charge = _f64(np.broadcast_to(np.asarray(charge, dtype=np.float64), (len(M),)))
    acc = acc or Accumulator(grid.nbins)
    pix_end = len(s) if pix_end is None else pix_end
    lib().orc_mdnorm_tables(grid.ref, len(s), _p(d), _p(s), None if lo is None else _p(lo),
                            None if hi is None else _p(hi), len(tables), _p(offs), _p(fk), _p(fF),
                            None if pt is None else _p(pt), len(M), _p(M), _p(charge), float(k_min),
                            float(k_max), int(pix_begin), int(pix_end), int(pix_stride), _p(acc.sum),
                            _p(acc.comp))
    return acc.value()


def binmd_err(grid: Grid, N, events, stride=None, col_e=1, col_q=5,
              acc: Accumulator | None = None) -> np.ndarray:
    """error-squared histogram from column col_e."""
    ev, n, stride = _events(events, stride, col_e, col_q)
    N = _f64(N).reshape(-1, 9)
    acc = acc or Accumulator(grid.nbins)
    lib().orc_binmd_err(grid.ref, len(N), _p(N), n, _p(ev), stride, col_e, col_q, _p(acc.sum),
                        _p(acc.comp))
    return acc.value()


def cross_section_err(err2_h, norm_h) -> np.ndarray:
    e, n = _f64(err2_h), _f64(norm_h)
    out = np.empty_like(e)
    lib().orc_cross_section_err(len(e), _p(e), _p(n), _p(out))
    return out


def mdnorm_trajectory(grid: Grid, d, solid, fk, fF, M, charge, k_min, k_max, max_segs=4096):
    """(n_cross, bins[int64], vals[f64]) for one trajectory."""
    d, fk, fF, M = _f64(d), _f64(fk), _f64(fF), _f64(M).reshape(9)
    bins = np.zeros(max_segs, dtype=np.int64)
    vals = np.zeros(max_segs)
    nc = C.c_int32(0)
    ns = lib().orc_mdnorm_trajectory(grid.ref, _p(d), float(solid), len(fk), _p(fk), _p(fF),
                                     _p(M), float(charge), float(k_min), float(k_max),
                                     C.byref(nc), _p(bins), _p(vals), max_segs)
    ns_kept = min(ns, max_segs)
    return nc.value, ns, bins[:ns_kept], vals[:ns_kept]


def _events(events, stride, col_w, col_q):
    ev = np.ascontiguousarray(events, dtype=np.float32)
    if ev.ndim == 2:
        stride = ev.shape[1] if stride is None else stride
        n = ev.shape[0]
    else:
        n = len(ev) // stride
    return ev, n, stride


def binmd(grid: Grid, N, events, stride=None, col_w=0, col_q=1,
          acc: Accumulator | None = None) -> np.ndarray:
    ev, n, stride = _events(events, stride, col_w, col_q)
    N = _f64(N).reshape(-1, 9)
    acc = acc or Accumulator(grid.nbins)
    lib().orc_binmd(grid.ref, len(N), _p(N), n, _p(ev), stride, col_w, col_q, _p(acc.sum),
                    _p(acc.comp))
    return acc.value()


def binmd_bins(grid: Grid, N, events, stride=None, col_w=0, col_q=1) -> np.ndarray:
    ev, n, stride = _events(events, stride, col_w, col_q)
    N = _f64(N).reshape(-1, 9)
    out = np.empty(len(N) * n, dtype=np.int64)
    lib().orc_binmd_bins(grid.ref, len(N), _p(N), n, _p(ev), stride, col_w, col_q, _p(out))
    return out.reshape(len(N), n)


def cross_section(binmd_h, norm_h) -> np.ndarray:
    b, n = _f64(binmd_h), _f64(norm_h)
    xs = np.empty_like(b)
    lib().orc_cross_section(len(b), _p(b), _p(n), _p(xs))
    return xs


def workload_grid(wl) -> Grid:
    return Grid(wl.lo, wl.hi, wl.nbins)


def run_workload(wl, runs=None, events=None, pix_stride=1, event_stride=1, timings=None):
    """Algorithm 1 on one process: sum MDNorm and BinMD over runs, then divide.

    events: dict run -> [n,4] float32 array (drawn by synth.events_for_run if absent).
    Returns (norm, binmd, xs).  Used by tests and by bench.py's cpu_baseline leg only.
    """
    from synth import events_for_run  # input generator only

    g = workload_grid(wl)
    runs = range(wl.nruns) if runs is None else runs
    na, ba = Accumulator(g.nbins), Accumulator(g.nbins)
    N = binmd_matrices(wl.UB, wl.ops, wl.W)
    t_md = t_bm = 0.0
    for r in runs:
        M = mdnorm_matrices(wl.R[r:r + 1], wl.UB, wl.ops, wl.W)
        t0 = time.perf_counter()
        mdnorm(g, wl.pix_dir, wl.solid, wl.flux_k, wl.flux_F, M, wl.charge[r], wl.k_min,
               wl.k_max, pix_stride=pix_stride, acc=na)
        t1 = time.perf_counter()
        ev = events[r] if events is not None else events_for_run(wl, r)
        ev = ev[::event_stride]
        t2 = time.perf_counter()
        binmd(g, N, ev, acc=ba)
        t3 = time.perf_counter()
        t_md += t1 - t0
        t_bm += t3 - t2
    if timings is not None:
        timings["mdnorm_s"] = t_md
        timings["binmd_s"] = t_bm
    norm, bm = na.value(), ba.value()
    return norm, bm, cross_section(bm, norm)
