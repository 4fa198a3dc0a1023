#!/usr/bin/env python
"""Small invocations of the code paths smoke() does not reach, for compute-sanitizer runs
(memcheck / racecheck / synccheck) on one GPU:

  compute-sanitizer --tool racecheck python tools/sanitize_paths.py

MDBox extents and box-culled BinMD, a flux table that makes the interval guess miss and one that
has no guess (cell-table search), the multi-slab cull/walk path, the per-bank flux tables, the
error column and its divide, the host-event staging ring, and BinMD in L2 slabs.  Prints one line per path; checks
only that each call returns (numbers are the tests' business).
"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth  # noqa: E402
import paper_conf_sc_hahnfgmmshvvs24_b200 as m  # noqa: E402


def grid(wl, priv=m.MDN_PRIV_AUTO, nbins=None):
    g = m.mdnorm_create_grid(0, wl.lo, wl.hi, wl.nbins if nbins is None else nbins, wl.W, m.MDN_ACC_F64)
    m.mdnorm_set_privatization(g, priv)
    m.mdnorm_set_instrument(g, wl.pix_dir, wl.solid)
    return g


def main():
    wl = synth.make_workload("corelli", events_per_run=60_000)
    ev = synth.events_for_run(wl, 0)
    dev = torch.from_numpy(ev).cuda()
    rng = np.random.default_rng(3)

    # flux tables: guess with misses (jittered 1/k knots), no guess (random knots)
    k, F = wl.flux_k, wl.flux_F
    kj = k.copy()
    for i in rng.choice(np.arange(1, len(k) - 1), len(k) // 8, replace=False):
        kj[i] = k[i] + rng.uniform(-0.45, 0.45) * min(k[i] - k[i - 1], k[i + 1] - k[i])
    kr = np.unique(np.concatenate([[k[0], k[-1]], rng.uniform(k[0], k[-1], len(k) - 2)]))
    for name, (fk, fF) in {"guess-miss": (kj, F), "no-guess": (kr, np.interp(kr, k, F))}.items():
        g = grid(wl)
        m.mdnorm_set_flux(g, fk, fF)
        m.mdnorm_accumulate(g, wl.UB, wl.R[0], wl.ops, wl.k_min, wl.k_max, 1.0, pix_stride=53)
        torch.cuda.synchronize()
        print("flux", name, m.mdnorm_debug_flux_guess(g), flush=True)
        g.close()

    # multi-slab cull/walk (forced small slab limit)
    g = grid(wl)
    m.mdnorm_set_flux(g, k, F)
    m.mdnorm_debug_set_max_slab(g, 4096)
    m.mdnorm_accumulate(g, wl.UB, wl.R[0], wl.ops[:4], wl.k_min, wl.k_max, 1.0, pix_stride=29)
    print("multi-slab", m.mdnorm_debug_last_launch(g), flush=True)
    g.close()

    # MDBox extents + box-culled BinMD; host events through the staging ring; error column + divide
    g = grid(wl)
    m.mdnorm_set_flux(g, k, F)
    m.mdnorm_accumulate(g, wl.UB, wl.R[0], wl.ops, wl.k_min, wl.k_max, 1.0, pix_stride=97)
    bounds = m.binmd_box_bounds(g, dev, box_events=256)
    m.binmd_accumulate_boxes(g, wl.UB, wl.ops, dev, 256, bounds)
    m.binmd_accumulate(g, wl.UB, wl.ops, ev)  # pageable host events
    ev8 = np.zeros((len(ev), 8), np.float32)
    ev8[:, 0] = ev[:, 0]
    ev8[:, 1] = ev[:, 0]
    ev8[:, 5:8] = ev[:, 1:4]
    m.binmd_accumulate_err(g, wl.UB, wl.ops, torch.from_numpy(ev8).cuda(), col_w=0, col_e=1, col_q=5)
    xs, err = m.mdnorm_cross_section_err(g)
    print("boxes + host events + error column", int(np.isfinite(xs).sum()), flush=True)
    g.close()

    # per-bank flux tables (global-memory flux path)
    g = grid(wl)
    m.mdnorm_set_flux_tables(g, [(k, F), (k, 2 * F)], (np.arange(wl.npix) % 2).astype(np.int32))
    m.mdnorm_accumulate(g, wl.UB, wl.R[0], wl.ops[:6], wl.k_min, wl.k_max, 1.0, pix_stride=41)
    torch.cuda.synchronize()
    print("per-bank flux", m.mdnorm_accumulation_paths(g), flush=True)
    g.close()

    # TOPAZ 3-D slice with several runs (mdnorm_accumulate_runs), privatisation off
    wt = synth.make_workload("topaz", nops=4, nruns=3, events_per_run=20_000)
    g = grid(wt, m.MDN_PRIV_OFF)
    m.mdnorm_set_flux(g, wt.flux_k, wt.flux_F)
    m.mdnorm_accumulate_runs(g, wt.UB, wt.R, np.ones(len(wt.R)), wt.ops, wt.k_min, wt.k_max, pix_stride=1999)
    torch.cuda.synchronize()
    print("topaz runs", m.mdnorm_debug_last_launch(g), flush=True)
    g.close()

    # BinMD on a grid larger than L2 (154 MB: two L2 slabs of the last axis) with the error column
    g = m.mdnorm_create_grid(0, [-6.0, -6.0, -3.0], [6.0, 6.0, 3.0], [400, 400, 120], wt.W, m.MDN_ACC_F64)
    evt = torch.from_numpy(synth.events_for_run(wt, 0)).cuda()
    m.binmd_accumulate(g, wt.UB, wt.ops, evt)
    rows = torch.zeros((evt.shape[0], 8), dtype=torch.float32, device="cuda")
    rows[:, 0] = evt[:, 0]
    rows[:, 1] = evt[:, 0]
    rows[:, 5:8] = evt[:, 1:4]
    m.binmd_accumulate_err(g, wt.UB, wt.ops, rows)
    torch.cuda.synchronize()
    print("l2 slabs", float(m.packed_histograms(g)[g.nbins_total:2 * g.nbins_total].sum().item()), flush=True)
    g.close()
    print("sanitize_paths: done")


if __name__ == "__main__":
    main()
