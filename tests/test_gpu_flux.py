"""M5 flux look-up with the interval guess (reading #10 of the flux definition):
whatever guess mode mdnorm_set_flux picks for a table -- uniform in 1/k (wavelength), uniform in
k, or none -- and however often the guess misses, every segment value is bit-identical to the fp64
oracle's and every histogram bin agrees to 1e-12.  The tables are built so that each mode and its
miss path are taken (checked through mdnorm_debug_flux_guess)."""
import numpy as np
import pytest

import oracle
import synth

pytestmark = pytest.mark.gpu

REL64 = 1e-12


@pytest.fixture(scope="module")
def mdn():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    import paper_conf_sc_hahnfgmmshvvs24_b200 as m
    from paper_conf_sc_hahnfgmmshvvs24_b200 import build
    build.build()
    return m


@pytest.fixture(scope="module")
def wl():
    return synth.make_workload("corelli")


def flux_variants(wl):
    """name -> (kappa, Phi, expected guess mode)."""
    k, F = wl.flux_k, wl.flux_F  # 'maxwell': knots uniform in wavelength
    rng = np.random.default_rng(11)
    out = {"inv_k": (k, F, 2)}
    # 1 in 8 knots moved by up to 45% of its smaller neighbouring spacing: still mode 2, with misses
    kj = k.copy()
    for i in rng.choice(np.arange(1, len(k) - 1), len(k) // 8, replace=False):
        kj[i] = k[i] + rng.uniform(-0.45, 0.45) * min(k[i] - k[i - 1], k[i + 1] - k[i])
    out["inv_k_jitter"] = (kj, F, 2)
    ku = np.linspace(k[0], k[-1], len(k))
    out["lin_k"] = (ku, np.interp(ku, k, F), 1)
    kr = np.unique(np.concatenate([[k[0], k[-1]], rng.uniform(k[0], k[-1], len(k) - 2)]))
    out["random"] = (kr, np.interp(kr, k, F), 0)
    return out


@pytest.mark.parametrize("name", ["inv_k", "inv_k_jitter", "lin_k", "random"])
def test_flux_guess_segments_bit_exact(mdn, wl, name):
    fk, fF, mode = flux_variants(wl)[name]
    g = mdn.mdnorm_create_grid(0, wl.lo, wl.hi, wl.nbins, wl.W, mdn.MDN_ACC_F64)
    mdn.mdnorm_set_instrument(g, wl.pix_dir, wl.solid)
    mdn.mdnorm_set_flux(g, fk, fF)
    gs = mdn.mdnorm_debug_flux_guess(g)
    assert gs["mode"] == mode, gs
    if mode:
        assert 0.9 <= gs["hit"] <= 1.0
        if name == "inv_k_jitter":
            assert gs["hit"] < 0.99  # the miss path is exercised
    og = oracle.workload_grid(wl)
    M = oracle.mdnorm_matrices(wl.R[:1], wl.UB, wl.ops, wl.W)
    charge = np.full(len(M), 1.25)
    rng = np.random.default_rng(5)
    ids = rng.integers(0, len(M) * wl.npix, size=6000)
    nc, ns, bins, vals = mdn.mdnorm_debug_trajectories(g, M, charge, wl.k_min, wl.k_max, ids, 1024)
    hits = 0
    for t, tid in enumerate(ids):
        m, p = divmod(int(tid), wl.npix)
        onc, ons, obins, ovals = oracle.mdnorm_trajectory(og, wl.pix_dir[p], wl.solid[p], fk, fF, M[m],
                                                          charge[m], wl.k_min, wl.k_max, 1024)
        assert (nc[t], ns[t]) == (onc, ons), tid
        k = min(ons, 1024)
        assert np.array_equal(bins[t, :k], obins), tid
        assert np.array_equal(vals[t, :k], ovals), tid
        hits += onc > 0
    assert hits > 100


@pytest.mark.parametrize("name", ["inv_k", "inv_k_jitter", "lin_k", "random"])
def test_flux_guess_walk_histogram(mdn, wl, name):
    """The production walk (flux records in shared memory) on every 8th pixel, all 24 ops."""
    import torch
    fk, fF, _ = flux_variants(wl)[name]
    d, s = wl.pix_dir[::8].copy(), wl.solid[::8].copy()
    g = mdn.mdnorm_create_grid(0, wl.lo, wl.hi, wl.nbins, wl.W, mdn.MDN_ACC_F64)
    mdn.mdnorm_set_privatization(g, 0)
    mdn.mdnorm_set_instrument(g, d, s)
    mdn.mdnorm_set_flux(g, fk, fF)
    mdn.mdnorm_accumulate(g, wl.UB, wl.R[0], wl.ops, wl.k_min, wl.k_max, wl.charge[0])
    torch.cuda.synchronize()
    norm = mdn.packed_histograms(g).cpu().numpy()[: g.nbins_total]
    M = oracle.mdnorm_matrices(wl.R[:1], wl.UB, wl.ops, wl.W)
    ref = oracle.mdnorm(oracle.workload_grid(wl), d, s, fk, fF, M, wl.charge[0], wl.k_min, wl.k_max)
    assert np.array_equal(norm == 0, ref == 0)
    assert np.all(np.abs(norm - ref) <= REL64 * np.abs(ref))
    assert (ref > 0).sum() > 1000
