"""Seeded sweep of random small configurations through the production path against the fp64
oracle: random pixel subsets of the CORELLI / TOPAZ instruments, random op subsets, a random
crystal orientation and goniometer angle, random grids (1-48 bins per axis, 2-D slices included,
windows that do or do not contain Q = 0, any projection W of the workload), random k ranges and
three kinds of flux table (the workload's, uniform, randomly jittered knots that defeat the
interval guess).  MDNorm per bin at 1e-12 with equal zero patterns; BinMD with unit weights
exactly equal (Listing 1, Listing 3; DESIGN.md §3 readings)."""
import dataclasses

import numpy as np
import pytest

import oracle
import synth
from synth.workloads import flux_table

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def mdn():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    import paper_conf_sc_hahnfgmmshvvs24_b200 as m
    from paper_conf_sc_hahnfgmmshvvs24_b200 import build
    build.build()
    return m


def random_config(seed):
    rng = np.random.default_rng(1000 + seed)
    base = synth.make_workload("corelli" if seed % 2 == 0 else "topaz", nops=48 if seed % 2 else None,
                               events_per_run=20_000)
    pix = np.sort(rng.choice(base.npix, int(rng.integers(256, 2049)), replace=False))
    ops = base.ops[np.sort(rng.choice(base.nops, int(rng.integers(1, 9)), replace=False))]
    rot = synth.rot_x(rng.uniform(-40, 40)) @ synth.rot_z(rng.uniform(-180, 180))
    n = [int(rng.integers(1, 49)) for _ in range(3)]
    if seed % 3 == 0:
        n[2] = 1  # a 2-D slice
    centre = rng.uniform(-3.0, 3.0, 3)
    half = rng.uniform(0.2, 8.0, 3)
    if seed % 4 == 1:
        centre = centre + np.sign(centre) * (half + 0.05)  # a window that excludes Q = 0 on every axis
    lo, hi = centre - half, centre + half
    k, F = base.flux_k, base.flux_F
    kind = seed % 3
    if kind == 1:
        k, F = flux_table("uniform", float(base.flux_k[0]), float(base.flux_k[-1]))
    elif kind == 2:  # jittered knots: the interval guess misses, the cell table decides
        k = k.copy()
        for i in rng.choice(np.arange(1, len(k) - 1), len(k) // 6, replace=False):
            k[i] = k[i] + rng.uniform(-0.45, 0.45) * min(k[i] - k[i - 1], k[i + 1] - k[i])
    span = float(k[-1] - k[0])
    kmin = float(k[0] + rng.uniform(-0.05, 0.3) * span)
    kmax = float(kmin + rng.uniform(0.2, 0.8) * span)
    return dataclasses.replace(base, pix_dir=base.pix_dir[pix], solid=base.solid[pix], ops=ops,
                               UB=rot @ base.UB, R=np.stack([synth.rot_y(rng.uniform(0, 360))]),
                               charge=np.array([rng.uniform(0.5, 2.0)]), lo=lo, hi=hi,
                               nbins=np.array(n, dtype=np.int64), flux_k=k, flux_F=F,
                               k_min=kmin, k_max=kmax)


@pytest.mark.parametrize("seed", range(48))
def test_random_config(mdn, seed):
    import torch
    wl = random_config(seed)
    g = mdn.mdnorm_create_grid(0, wl.lo, wl.hi, wl.nbins, wl.W, mdn.MDN_ACC_F64)
    mdn.mdnorm_set_privatization(g, mdn.MDN_PRIV_OFF if seed % 2 else mdn.MDN_PRIV_AUTO)
    mdn.mdnorm_set_instrument(g, wl.pix_dir, wl.solid)
    mdn.mdnorm_set_flux(g, wl.flux_k, wl.flux_F)
    mdn.mdnorm_accumulate(g, wl.UB, wl.R[0], wl.ops, wl.k_min, wl.k_max, float(wl.charge[0]))
    ev = synth.events_for_run(dataclasses.replace(wl, k_min=float(wl.flux_k[0]), k_max=float(wl.flux_k[-1])), 0,
                              unit_weights=True)
    mdn.binmd_accumulate(g, wl.UB, wl.ops, torch.from_numpy(ev).cuda())
    torch.cuda.synchronize()
    packed = mdn.packed_histograms(g).cpu().numpy()
    nb = g.nbins_total
    norm, bm = packed[:nb], packed[nb:2 * nb]
    g.close()
    og = oracle.Grid(wl.lo, wl.hi, wl.nbins)
    M = oracle.mdnorm_matrices(wl.R, wl.UB, wl.ops, wl.W)
    onorm = oracle.mdnorm(og, wl.pix_dir, wl.solid, wl.flux_k, wl.flux_F, M, float(wl.charge[0]), wl.k_min,
                          wl.k_max)
    obm = oracle.binmd(og, oracle.binmd_matrices(wl.UB, wl.ops, wl.W), ev)
    assert np.array_equal(norm == 0, onorm == 0), "norm zero pattern"
    assert np.all(np.abs(norm - onorm) <= 1e-12 * np.abs(onorm)), "norm values"
    assert np.array_equal(bm, obm), "binmd counts"


@pytest.mark.parametrize("seed", range(24))
def test_random_config_runs_banks_errors(mdn, seed):
    """The same random configurations with the Mantid-compatible inputs (NEXT #1) and the batched
    rotation scan: 2-4 runs through mdnorm_accumulate_runs (random angles and charges), per-pixel
    k limits on a random half of the pixels (some empty), 2-3 per-bank flux tables on a random
    pixel map, and 8-column events with an error-squared column through binmd_accumulate_err --
    against Algorithm 1 on the oracle (norm 1e-12 per bin, counts and integer error sums exact)."""
    import torch
    wl = random_config(100 + seed)
    rng = np.random.default_rng(5000 + seed)
    nruns = int(rng.integers(2, 5))
    R = np.stack([synth.rot_y(rng.uniform(0, 360)) for _ in range(nruns)])
    charge = rng.uniform(0.5, 2.0, nruns)
    npix = wl.npix
    span = wl.k_max - wl.k_min
    pk_lo = np.full(npix, wl.k_min)
    pk_hi = np.full(npix, wl.k_max)
    sel = rng.random(npix) < 0.5
    pk_lo[sel] = wl.k_min + rng.uniform(-0.2, 0.6, sel.sum()) * span
    pk_hi[sel] = pk_lo[sel] + rng.uniform(-0.1, 0.8, sel.sum()) * span  # some empty
    ntab = int(rng.integers(2, 4))
    tables = [(wl.flux_k, wl.flux_F * (1.0 + 0.5 * t)) for t in range(ntab)]
    ptab = rng.integers(0, ntab, npix).astype(np.int32)
    g = mdn.mdnorm_create_grid(0, wl.lo, wl.hi, wl.nbins, wl.W, mdn.MDN_ACC_F64)
    mdn.mdnorm_set_instrument(g, wl.pix_dir, wl.solid)
    mdn.mdnorm_set_flux_tables(g, tables, ptab)
    mdn.mdnorm_set_pixel_krange(g, pk_lo, pk_hi)
    mdn.mdnorm_accumulate_runs(g, wl.UB, R, charge, wl.ops, wl.k_min, wl.k_max)
    ev = synth.events_for_run(dataclasses.replace(wl, k_min=float(wl.flux_k[0]), k_max=float(wl.flux_k[-1])), 0,
                              unit_weights=True)
    rows = np.zeros((len(ev), 8), np.float32)
    rows[:, 0] = ev[:, 0]
    rows[:, 1] = rng.integers(1, 5, len(ev)).astype(np.float32)  # error^2: integer sums are exact
    rows[:, 5:8] = ev[:, 1:]
    mdn.binmd_accumulate_err(g, wl.UB, wl.ops, torch.from_numpy(rows).cuda())
    torch.cuda.synchronize()
    packed = mdn.packed_histograms(g).cpu().numpy()
    nb = g.nbins_total
    norm, bm, e2 = packed[:nb], packed[nb:2 * nb], packed[2 * nb:3 * nb]
    g.close()
    og = oracle.Grid(wl.lo, wl.hi, wl.nbins)
    M = oracle.mdnorm_matrices(R, wl.UB, wl.ops, wl.W)
    onorm = oracle.mdnorm_tables(og, wl.pix_dir, wl.solid, tables, ptab, M, np.repeat(charge, wl.nops),
                                 wl.k_min, wl.k_max, pix_kmin=pk_lo, pix_kmax=pk_hi)
    N = oracle.binmd_matrices(wl.UB, wl.ops, wl.W)
    obm = oracle.binmd(og, N, rows, stride=8, col_w=0, col_q=5)
    oe2 = oracle.binmd_err(og, N, rows, stride=8, col_e=1, col_q=5)
    assert np.array_equal(norm == 0, onorm == 0), "norm zero pattern"
    assert np.all(np.abs(norm - onorm) <= 1e-12 * np.abs(onorm)), "norm values"
    assert np.array_equal(bm, obm), "binmd counts"
    assert np.array_equal(e2, oe2), "error-squared sums"
