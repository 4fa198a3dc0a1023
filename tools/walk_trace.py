#!/usr/bin/env python
"""Developer timeline of the MDNorm walk kernel (per-warp start, first round, end; rounds per warp)
for one CORELLI run and for four copies of its pixels in one launch.  Needs a library built with
-DMDN_WALK_TRACE=1:

  python tools/variants.py trace:MDN_WALK_TRACE=1
  MDN_LIB_PATH=$PWD/variants/lib_trace.so python tools/walk_trace.py
"""
import sys, os, ctypes as C
sys.path.insert(0, os.getcwd())
import torch, numpy as np, bench
import paper_conf_sc_hahnfgmmshvvs24_b200 as m
from paper_conf_sc_hahnfgmmshvvs24_b200 import _native
wl = bench.make_bench_workload(1)
lib = _native.load()
for rep in (1, 4):
    g = m.mdnorm_create_grid(0, wl.lo, wl.hi, wl.nbins, wl.W, m.MDN_ACC_F64)
    m.mdnorm_set_instrument(g, np.tile(wl.pix_dir, (rep, 1)), np.tile(wl.solid, rep)); m.mdnorm_set_flux(g, wl.flux_k, wl.flux_F)
    for it in range(3):
        m.mdnorm_accumulate(g, wl.UB, wl.R[0], wl.ops, wl.k_min, wl.k_max, 1.0)
        torch.cuda.synchronize()
    buf = np.zeros(4 * 148 * 32, np.uint64)
    assert lib.mdn_debug_walk_trace(C.c_void_p(buf.ctypes.data), len(buf)) == 0
    t = buf.reshape(-1, 4).astype(np.int64)
    t0 = t[:, 0].min()
    start = (t[:, 0] - t0) / 1e3; first = (t[:, 1] - t0) / 1e3; end = (t[:, 2] - t0) / 1e3
    rounds = t[:, 3] & 0xffffffff
    print(f"rep {rep}: kernel span {end.max():.1f} us; warp start (after staging) p0 {start.min():.1f} p50 {np.median(start):.1f} p100 {start.max():.1f}; "
          f"first round p50 {np.median(first):.1f} max {first.max():.1f}; end p0 {end.min():.1f} p10 {np.percentile(end,10):.1f} p50 {np.median(end):.1f} p90 {np.percentile(end,90):.1f} max {end.max():.1f}; "
          f"rounds p50 {np.median(rounds):.0f} min {rounds.min()} max {rounds.max()}", flush=True)
    # occupancy over time: fraction of warps alive at each decile of the span
    span = end.max()
    alive = [np.mean((start <= x) & (end > x)) for x in np.linspace(0, span, 11)]
    print("   alive fraction at deciles:", " ".join(f"{a:.2f}" for a in alive))
    g.close()
