"""GPU parity of the S§8(f) NEXT #1 inputs: per-pixel momentum limits and the error-squared
histogram / cross-section error, through the C ABI against the fp64 oracle."""
import numpy as np
import pytest

import oracle
import synth

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


def _packed(mdn, g):
    import torch
    torch.cuda.synchronize()
    t = mdn.packed_histograms(g).cpu().numpy()
    n = g.nbins_total
    return t[:n].copy(), t[n:2 * n].copy(), t[2 * n:].copy()


def _assert_rel(a, b, rel=1e-12):
    assert np.array_equal(a == 0, b == 0)
    assert np.all(np.abs(a - b) <= rel * np.abs(b))


def test_pixel_krange_parity(mdn):
    wl = synth.make_workload("corelli")
    rng = np.random.default_rng(31)
    lo = rng.uniform(1.5, 5.0, wl.npix)
    hi = lo + rng.uniform(0.2, 6.0, wl.npix)
    hi[::7] = lo[::7] - 0.1  # some empty ranges
    g = mdn.mdnorm_create_grid(0, wl.lo, wl.hi, wl.nbins, wl.W)
    mdn.mdnorm_set_instrument(g, wl.pix_dir, wl.solid)
    mdn.mdnorm_set_flux(g, wl.flux_k, wl.flux_F)
    mdn.mdnorm_set_pixel_krange(g, lo, hi)
    stride = 5
    mdn.mdnorm_accumulate(g, wl.UB, wl.R[0], wl.ops, wl.k_min, wl.k_max, 1.0, pix_stride=stride)
    norm, _, _ = _packed(mdn, g)
    og = oracle.workload_grid(wl)
    M = oracle.mdnorm_matrices(wl.R, wl.UB, wl.ops, wl.W)
    onorm = oracle.mdnorm_krange(og, wl.pix_dir, wl.solid, lo, hi, wl.flux_k, wl.flux_F, M, 1.0,
                                 wl.k_min, wl.k_max, pix_stride=stride)
    assert onorm.sum() > 0
    _assert_rel(norm, onorm)
    # per-trajectory geometry with the limits through the debug entry
    ids = rng.integers(0, 4 * wl.npix, size=2000)
    nc, ns, bins, vals = mdn.mdnorm_debug_trajectories(g, M[:4], np.ones(4), wl.k_min, wl.k_max, ids, 512)
    for t, tid in enumerate(ids):
        m, p = divmod(int(tid), wl.npix)
        onc, ons, ob, ov = oracle.mdnorm_trajectory(og, wl.pix_dir[p], wl.solid[p], wl.flux_k, wl.flux_F, M[m],
                                                    1.0, max(wl.k_min, lo[p]), min(wl.k_max, hi[p]), 512)
        assert (nc[t], ns[t]) == (onc, ons)
        assert np.array_equal(bins[t, :ons], ob) and np.array_equal(vals[t, :ons], ov)
    # removing the limits restores the plain result
    mdn.mdnorm_set_pixel_krange(g, None, None)
    mdn.mdnorm_reset(g)
    mdn.mdnorm_accumulate(g, wl.UB, wl.R[0], wl.ops, wl.k_min, wl.k_max, 1.0, pix_stride=stride)
    norm2, _, _ = _packed(mdn, g)
    _assert_rel(norm2, oracle.mdnorm(og, wl.pix_dir, wl.solid, wl.flux_k, wl.flux_F, M, 1.0, wl.k_min,
                                     wl.k_max, pix_stride=stride))
    with pytest.raises(mdn.MdnError, match="MDN_EINVAL"):
        mdn.mdnorm_set_pixel_krange(g, lo[:10], hi[:10])


@pytest.mark.parametrize("cfg", ["corelli", "topaz"])
def test_per_bank_flux_tables(mdn, cfg):
    """Pixel -> flux-table map: each bank (TOPAZ: 25 banks of 65536 pixels; CORELLI: 3 random
    groups) reads its own cumulative-flux table with its own knots."""
    wl = synth.make_workload(cfg, nops=8) if cfg == "topaz" else synth.make_workload(cfg)
    rng = np.random.default_rng(33)
    nt = 25 if cfg == "topaz" else 3
    tables = []
    for t in range(nt):
        kk = np.sort(np.unique(np.concatenate([wl.flux_k[:: 2 + t % 3], rng.uniform(wl.flux_k[0], wl.flux_k[-1], 50)])))
        FF = np.interp(kk, wl.flux_k, wl.flux_F) * (0.5 + rng.uniform())
        FF[0] = 0.0
        FF = np.maximum.accumulate(FF)
        tables.append((kk, FF))
    pt = (np.arange(wl.npix) // 65536).astype(np.int32) if cfg == "topaz" else \
        rng.integers(0, nt, wl.npix).astype(np.int32)
    g = mdn.mdnorm_create_grid(0, wl.lo, wl.hi, wl.nbins, wl.W)
    mdn.mdnorm_set_instrument(g, wl.pix_dir, wl.solid)
    mdn.mdnorm_set_flux_tables(g, tables, pt)
    stride = 7 if cfg == "corelli" else 997
    mdn.mdnorm_accumulate(g, wl.UB, wl.R[0], wl.ops, wl.k_min, wl.k_max, 1.0, pix_stride=stride)
    norm, _, _ = _packed(mdn, g)
    og = oracle.workload_grid(wl)
    M = oracle.mdnorm_matrices(wl.R, wl.UB, wl.ops, wl.W)
    onorm = oracle.mdnorm_tables(og, wl.pix_dir, wl.solid, tables, pt, M, 1.0, wl.k_min, wl.k_max,
                                 pix_stride=stride)
    assert onorm.sum() > 0
    _assert_rel(norm, onorm)
    ids = rng.integers(0, len(M) * wl.npix, size=1500)
    nc, ns, bins, vals = mdn.mdnorm_debug_trajectories(g, M, np.ones(len(M)), wl.k_min, wl.k_max, ids, 700)
    for t, tid in enumerate(ids):
        m, p = divmod(int(tid), wl.npix)
        kk, FF = tables[pt[p]]
        onc, ons, ob, ov = oracle.mdnorm_trajectory(og, wl.pix_dir[p], wl.solid[p], kk, FF, M[m], 1.0,
                                                    wl.k_min, wl.k_max, 700)
        assert (nc[t], ns[t]) == (onc, ons)
        assert np.array_equal(bins[t, :ons], ob) and np.array_equal(vals[t, :ons], ov)
    with pytest.raises(mdn.MdnError, match="MDN_EINVAL"):
        mdn.mdnorm_set_flux_tables(g, tables, np.full(wl.npix, nt, np.int32))


def test_error_histogram_and_xs_err(mdn):
    import torch
    wl = synth.make_workload("corelli", events_per_run=1_000_000)
    ev = synth.events_for_run(wl, 0)
    rng = np.random.default_rng(32)
    ev8 = np.zeros((len(ev), 8), np.float32)
    ev8[:, 0] = ev[:, 0]
    ev8[:, 1] = (ev[:, 0] * rng.uniform(0.5, 1.5, len(ev))).astype(np.float32)
    ev8[:, 5:8] = ev[:, 1:4]
    g = mdn.mdnorm_create_grid(0, wl.lo, wl.hi, wl.nbins, wl.W)
    mdn.mdnorm_set_instrument(g, wl.pix_dir, wl.solid)
    mdn.mdnorm_set_flux(g, wl.flux_k, wl.flux_F)
    mdn.mdnorm_accumulate(g, wl.UB, wl.R[0], wl.ops, wl.k_min, wl.k_max, 1.0, pix_stride=3)
    mdn.binmd_accumulate_err(g, wl.UB, wl.ops, torch.from_numpy(ev8).cuda(), col_w=0, col_e=1, col_q=5)
    mdn.binmd_accumulate_err(g, wl.UB, wl.ops, ev8[:1001], col_w=0, col_e=1, col_q=5)  # host path
    norm, bm, e2 = _packed(mdn, g)
    og = oracle.workload_grid(wl)
    N = oracle.binmd_matrices(wl.UB, wl.ops, wl.W)
    M = oracle.mdnorm_matrices(wl.R, wl.UB, wl.ops, wl.W)
    onorm = oracle.mdnorm(og, wl.pix_dir, wl.solid, wl.flux_k, wl.flux_F, M, 1.0, wl.k_min, wl.k_max,
                          pix_stride=3)
    ob, oe = oracle.Accumulator(og.nbins), oracle.Accumulator(og.nbins)
    for part in (ev8, ev8[:1001]):
        oracle.binmd(og, N, part, col_w=0, col_q=5, acc=ob)
        oracle.binmd_err(og, N, part, col_e=1, col_q=5, acc=oe)
    _assert_rel(norm, onorm)
    _assert_rel(bm, ob.value())
    _assert_rel(e2, oe.value())
    xs, xe = mdn.mdnorm_cross_section_err(g)
    oxs = oracle.cross_section(ob.value(), onorm)
    oxe = oracle.cross_section_err(oe.value(), onorm)
    assert np.array_equal(np.isnan(xs), np.isnan(oxs)) and np.array_equal(np.isnan(xe), np.isnan(oxe))
    ok = ~np.isnan(oxs)
    assert np.all(np.abs(xs[ok] - oxs[ok]) <= 3e-12 * np.abs(oxs[ok]))
    assert np.all(np.abs(xe[ok] - oxe[ok]) <= 3e-12 * np.abs(oxe[ok]))
    # device outputs agree with host outputs; plain binmd_accumulate leaves err2 alone
    dxs = torch.empty(g.nbins_total, dtype=torch.float64, device="cuda")
    dxe = torch.empty_like(dxs)
    mdn.mdnorm_cross_section_err(g, dxs, dxe)
    assert np.array_equal(dxs.cpu().numpy(), xs, equal_nan=True)
    assert np.array_equal(dxe.cpu().numpy(), xe, equal_nan=True)
    mdn.binmd_accumulate(g, wl.UB, wl.ops, torch.from_numpy(ev).cuda())
    _, _, e2b = _packed(mdn, g)
    assert np.array_equal(e2b, e2)
    with pytest.raises(mdn.MdnError, match="MDN_EINVAL"):
        mdn.binmd_accumulate_err(g, wl.UB, wl.ops, ev8, col_w=0, col_e=5, col_q=5)
