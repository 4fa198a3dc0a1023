"""Pins of the CPU oracle against what the paper and the mathematics fix (no GPU).

Each test names the pin of SURVEY.md §8(c) / DESIGN.md §3 it implements.  None of them compares
the oracle with a retyped copy of itself: expected values come from hand derivations
(tests/golden/, cited), closed forms, brute-force fine-step integration written independently
in numpy, invariants of the definition, or the Bragg condition.
"""
import json
import math
import os

import numpy as np
import pytest

import synth

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _golden(name):
    with open(os.path.join(GOLDEN, name)) as f:
        return json.load(f)


# ----------------------------------------------------------------------------- golden fixtures


@pytest.mark.parametrize("name", ["mdnorm_backscatter_axis2.json", "mdnorm_diagonal_ties.json"])
def test_golden_trajectory(orc, name):
    """Hand-derived worked examples of Listing 1; see each fixture's derivation."""
    g = _golden(name)
    grid = orc.Grid(g["grid"]["lo"], g["grid"]["hi"], g["grid"]["n"])
    nc, ns, bins, vals = orc.mdnorm_trajectory(grid, g["dir"], g["solid"], g["flux_k"], g["flux_F"],
                                               np.array(g["M"]), g["charge"], g["k_min"], g["k_max"])
    assert nc == g["expect_n_cross"]
    assert ns == len(g["expect_seg_bins"])
    assert bins.tolist() == g["expect_seg_bins"]
    assert vals.tolist() == g["expect_seg_vals"]  # every value is exactly representable
    # the histogram path gives the same numbers
    h = orc.mdnorm(grid, np.array([g["dir"]]), np.array([g["solid"]]), g["flux_k"], g["flux_F"],
                   np.array(g["M"])[None], [g["charge"]], g["k_min"], g["k_max"])
    expect = np.zeros(grid.nbins)
    expect[g["expect_seg_bins"]] = g["expect_seg_vals"]
    np.testing.assert_array_equal(h, expect)


def test_golden_binmd(orc):
    """Hand-derived BinMD example (Listing 3)."""
    g = _golden("binmd_hand.json")
    grid = orc.Grid(g["grid"]["lo"], g["grid"]["hi"], g["grid"]["n"])
    ev = np.array(g["events"], dtype=np.float32)
    N = np.array(g["N"])
    bins = orc.binmd_bins(grid, N, ev)
    assert bins[0].tolist() == g["expect_bins_op0"]
    assert bins[1].tolist() == g["expect_bins_op1"]
    h = orc.binmd(grid, N, ev)
    expect = np.zeros(grid.nbins)
    for k, v in g["expect_hist"].items():
        expect[int(k)] = v
    np.testing.assert_array_equal(h, expect)


# ----------------------------------------------------------------------------- M5 flux


def test_flux_knots_uniform_and_clamp(orc):
    wl = synth.make_workload("corelli")
    fk, fF = wl.flux_k, wl.flux_F
    # F(kappa_i) = Phi_i exactly at the knots (interpolation weight 0)
    for i in [0, 1, 7, 100, 2047, 4094, 4095]:
        assert orc.flux(fk, fF, fk[i]) == fF[i]
    # clamped outside the table (reading #9)
    assert orc.flux(fk, fF, fk[0] - 1.0) == fF[0]
    assert orc.flux(fk, fF, fk[-1] + 1.0) == fF[-1]
    # monotone non-decreasing between random points
    rng = np.random.default_rng(0)
    xs = np.sort(rng.uniform(fk[0] - 0.5, fk[-1] + 0.5, 2000))
    F = np.array([orc.flux(fk, fF, x) for x in xs])
    assert np.all(np.diff(F) >= 0)
    # each value lies between its neighbouring knots' values
    i = np.clip(np.searchsorted(fk, xs, side="right") - 1, 0, len(fk) - 2)
    inner = (xs > fk[0]) & (xs < fk[-1])
    assert np.all(F[inner] >= fF[i[inner]]) and np.all(F[inner] <= fF[i[inner] + 1])
    # uniform flux: F(x) = x - kappa_0 (closed form), to rounding
    ufk, ufF = np.array([2.0, 12.0]), np.array([0.0, 10.0])
    for x in rng.uniform(2.0, 12.0, 50):
        assert abs(orc.flux(ufk, ufF, x) - (x - 2.0)) <= 4e-15 * 12


# ----------------------------------------------------------------------------- M0 matrices


def test_compose_bragg_condition(orc):
    """Bragg pin: an event at Q_sample = 2 pi UB S W x must land at grid coordinate x (B0-B3),
    and M_{r,s} applied to Q_lab = R Q_sample agrees with N_s (reading #1-#2)."""
    wl = synth.make_workload("corelli")
    rng = np.random.default_rng(1)
    for s in [0, 5, 13, 23]:
        S = wl.ops[s]
        N = orc.compose_binmd(wl.UB, S, wl.W)
        x = rng.uniform(-5, 5, 3)
        Q = 2 * math.pi * wl.UB @ S @ wl.W @ x
        np.testing.assert_allclose(N @ Q, x, rtol=0, atol=1e-12)
        R = synth.rot_y(rng.uniform(0, 360))
        M = orc.compose_mdnorm(R, wl.UB, S, wl.W)
        np.testing.assert_allclose(M @ (R @ Q), x, rtol=0, atol=1e-12)
        np.testing.assert_allclose(M, N @ R.T, rtol=0, atol=1e-14)
        # R = I: I * UB is exact, so M and N agree bit for bit
        assert np.array_equal(orc.compose_mdnorm(np.eye(3), wl.UB, S, wl.W), N)
    with pytest.raises(ValueError):
        orc.compose_binmd(np.zeros((3, 3)), np.eye(3), np.eye(3))


def test_binmd_bragg_events_land_on_hkl(orc):
    """Events placed exactly at integer HKL (CORELLI UB, W) land in the bin of x = W^-1 h."""
    wl = synth.make_workload("corelli")
    off = 0.0125  # half a bin: integer and half-integer x sit at bin centres
    grid = orc.Grid([-7.5 + off, -7.5 + off, -0.1], [7.5 + off, 7.5 + off, 0.1], [600, 600, 1])
    N = orc.binmd_matrices(wl.UB, wl.ops[:1], wl.W)
    hs = np.array([[1, 1, 0], [2, 0, 0], [-3, 1, 0], [4, -2, 0], [0, 5, 0]], dtype=float)
    Q = (2 * math.pi * wl.UB @ hs.T).T
    ev = np.concatenate([np.ones((len(hs), 1)), Q], axis=1).astype(np.float32)
    bins = orc.binmd_bins(grid, N, ev)[0]
    x = np.linalg.solve(wl.W, hs.T).T
    w = 15.0 / 600
    i = np.floor((x[:, :2] + 7.5 - off) / w).astype(int)
    expect = i[:, 0] + 600 * i[:, 1]
    frac = ((x[:, :2] + 7.5 - off) / w) % 1.0
    assert np.all(np.abs(frac - 0.5) < 1e-3)  # float32 rounding of Q moves x by ~1e-6 only
    assert np.array_equal(bins, expect)


# ----------------------------------------------------------------------------- M1-M7 closed forms


def _closed_form_axis2(lo2, hi2, n2, v2, kmin, kmax, omega_c, phi0):
    """Exact segment values for x(k) = k*v with only axis 2 binned and uniform flux phi0."""
    w = (hi2 - lo2) / n2
    out = np.zeros(n2)
    for j in range(n2):
        a, b = lo2 + j * w, lo2 + (j + 1) * w
        ka, kb = sorted((a / v2, b / v2))
        lo_k, hi_k = max(ka, kmin), min(kb, kmax)
        if hi_k > lo_k:
            out[j] = omega_c * phi0 * (hi_k - lo_k)
    return out


def test_axis_aligned_closed_form(orc):
    """M = alpha*I, any pixel direction: x(k) = k*alpha*(z - d) (reading #1, M1).  With axes 0,1
    covered by one wide bin, bin j of axis 2 gets Omega c phi0 |overlap([e_j,e_j+1]/v2, [k_min,k_max])|."""
    rng = np.random.default_rng(2)
    phi0 = 3.0
    fk, fF = np.array([0.5, 30.0]), np.array([0.0, phi0 * 29.5])
    for _ in range(40):
        d = rng.normal(size=3)
        d /= np.linalg.norm(d)
        if 1 - d[2] < 0.05:
            continue
        alpha = rng.uniform(0.2, 2.0)
        v2 = alpha * (1 - d[2])
        n2 = int(rng.integers(3, 40))
        lo2, hi2 = rng.uniform(-1, 2), rng.uniform(4, 30)
        grid = orc.Grid([-1e3, -1e3, lo2], [1e3, 1e3, hi2], [1, 1, n2])
        kmin, kmax = rng.uniform(1, 4), rng.uniform(6, 25)
        solid, charge = rng.uniform(0.1, 2), rng.uniform(0.5, 2)
        h = orc.mdnorm(grid, d[None], [solid], fk, fF, (alpha * np.eye(3))[None], [charge], kmin, kmax)
        expect = _closed_form_axis2(lo2, hi2, n2, v2, kmin, kmax, solid * charge, phi0)
        np.testing.assert_allclose(h, expect, rtol=1e-12, atol=1e-12 * expect.max())


def test_backscatter_q_is_2z(orc):
    """d = -z gives q = (0,0,2) (|q| = 2 sin(theta) at 2theta = 180 deg): with M = I the walk
    along axis 2 crosses plane e at k = e/2 exactly."""
    grid = orc.Grid([-1, -1, 0.0], [1, 1, 64.0], [1, 1, 64])
    fk, fF = np.array([0.0, 100.0]), np.array([0.0, 100.0])
    nc, ns, bins, vals = orc.mdnorm_trajectory(grid, [0, 0, -1.0], 1.0, fk, fF, np.eye(3), 1.0,
                                               1.0, 20.0)
    # points 2k in [2, 40] -> planes 3..39 inside, bins 2..39; interior segments have dk = 0.5
    assert nc == 2 + 37
    assert bins.tolist() == list(range(2, 40))
    np.testing.assert_allclose(vals, 0.5, rtol=1e-14)  # F(k) = 100 * (k / 100): rounding only


def test_intersection_bound_p114(orc):
    """intersections per trajectory < hBins + kBins + lBins + 2."""
    rng = np.random.default_rng(3)
    fk, fF = np.array([0.0, 50.0]), np.array([0.0, 50.0])
    for _ in range(200):
        n = rng.integers(1, 30, size=3)
        grid = orc.Grid([-5, -5, -5], [5, 5, 5], n)
        d = rng.normal(size=3)
        d /= np.linalg.norm(d)
        M = rng.normal(size=(3, 3))
        nc, ns, _, _ = orc.mdnorm_trajectory(grid, d, 1.0, fk, fF, M, 1.0, 0.1, 40.0)
        assert nc < n.sum() + 2
        assert ns <= max(nc - 1, 0)


# ----------------------------------------------------------------------------- brute force


def _brute_force(lo, hi, n, d, omega_c, M, fk, fF, kmin, kmax, nsub):
    """Independent fine-step integration: sum dF over 'nsub' sub-steps into bin(k_mid * v)."""
    lo, hi, n = np.asarray(lo, float), np.asarray(hi, float), np.asarray(n)
    v = M @ np.array([-d[0], -d[1], 1 - d[2]])
    ks = np.linspace(kmin, kmax, nsub + 1)
    F = np.interp(ks, fk, fF)
    dF = np.diff(F)
    km = 0.5 * (ks[1:] + ks[:-1])
    t = (km[:, None] * v[None, :] - lo) / ((hi - lo) / n)
    inside = np.all((t >= 0) & (t < n), axis=1)
    i = np.floor(t[inside]).astype(np.int64)
    b = i[:, 0] + n[0] * (i[:, 1] + n[1] * i[:, 2])
    return np.bincount(b, weights=dF[inside] * omega_c, minlength=int(np.prod(n))), dF.max()


@pytest.mark.parametrize("case", range(8))
def test_brute_force_integration(orc, case):
    """Whole-MDNorm pin: fine-step integration (10^6 sub-steps) converges to the oracle; the L1
    error is bounded by 2 * n_cross * max sub-step dF * Omega c (each crossing misattributes at
    most one sub-step)."""
    rng = np.random.default_rng(100 + case)
    wl = synth.make_workload("corelli")
    fk, fF = wl.flux_k, wl.flux_F
    n = [int(x) for x in rng.integers(2, 12, size=3)]
    lo, hi = [-3.0, -3.0, -2.0], [3.0, 3.0, 2.0]
    grid = orc.Grid(lo, hi, n)
    d = rng.normal(size=3)
    d /= np.linalg.norm(d)
    M = orc.compose_mdnorm(synth.rot_y(rng.uniform(0, 360)), wl.UB, wl.ops[case % 24], wl.W)
    omega_c = rng.uniform(0.5, 2.0)
    kmin, kmax = 2.17, 9.67
    h = orc.mdnorm(grid, d[None], [omega_c], fk, fF, M[None], [1.0], kmin, kmax)
    nc, _, _, _ = orc.mdnorm_trajectory(grid, d, omega_c, fk, fF, M, 1.0, kmin, kmax)
    bf, dfmax = _brute_force(lo, hi, n, d, omega_c, M, fk, fF, kmin, kmax, 1_000_000)
    bound = 2 * max(nc, 1) * dfmax * omega_c + 1e-12 * max(h.sum(), 1e-300)
    assert np.abs(bf - h).sum() <= bound
    assert abs(bf.sum() - h.sum()) <= bound


def test_brute_force_tiny_config(orc):
    """Tiny config (BASELINE configs[0]) whole histogram vs brute force over all 64 pixels."""
    wl = synth.make_workload("tiny")
    grid = orc.workload_grid(wl)
    M = orc.mdnorm_matrices(wl.R, wl.UB, wl.ops, wl.W)[0]
    h = orc.mdnorm(grid, wl.pix_dir, wl.solid, wl.flux_k, wl.flux_F, M[None], [1.0], wl.k_min, wl.k_max)
    bf = np.zeros(grid.nbins)
    bound = 0.0
    for p in range(wl.npix):
        b, dfm = _brute_force(wl.lo, wl.hi, wl.nbins, wl.pix_dir[p], wl.solid[p], M, wl.flux_k,
                              wl.flux_F, wl.k_min, wl.k_max, 200_000)
        nc, _, _, _ = orc.mdnorm_trajectory(grid, wl.pix_dir[p], wl.solid[p], wl.flux_k, wl.flux_F,
                                            M, 1.0, wl.k_min, wl.k_max)
        bf += b
        bound += 2 * max(nc, 1) * dfm * wl.solid[p]
    assert np.abs(bf - h).sum() <= bound * 1.0001
    assert h.sum() > 0


# ----------------------------------------------------------------------------- invariants


def test_telescoping_per_trajectory(orc):
    """M7 invariant: a trajectory's contributions sum to Omega c (F(k_max) - F(k_min)) when the
    grid covers it (BASELINE north_star)."""
    wl = synth.make_workload("corelli")
    grid = orc.Grid([-40, -40, -40], [40, 40, 40], [37, 23, 11])
    rng = np.random.default_rng(4)
    Fmin, Fmax = orc.flux(wl.flux_k, wl.flux_F, wl.k_min), orc.flux(wl.flux_k, wl.flux_F, wl.k_max)
    for p in rng.integers(0, wl.npix, 30):
        M = orc.compose_mdnorm(wl.R[0], wl.UB, wl.ops[p % 24], wl.W)
        nc, ns, bins, vals = orc.mdnorm_trajectory(grid, wl.pix_dir[p], 1.5, wl.flux_k, wl.flux_F,
                                                   M, 2.0, wl.k_min, wl.k_max)
        assert nc >= 2
        expect = 3.0 * (Fmax - Fmin)
        assert abs(vals.sum() - expect) <= 1e-12 * expect


def _corelli_subset(orc, stride=997, nbin=60):
    wl = synth.make_workload("corelli")
    grid = orc.Grid(wl.lo, wl.hi, [nbin, nbin, 1])
    return wl, grid, wl.pix_dir[::stride].copy(), wl.solid[::stride].copy()


def test_op_invariances(orc):
    """Permuting ops, left-multiplying all ops by a group element, or using S^-1 for S leaves
    norm unchanged; duplicating an op doubles its contribution; scaling c or Omega by 2 scales
    exactly by 2 (BASELINE north_star invariants)."""
    wl, grid, d, s = _corelli_subset(orc)
    args = (wl.flux_k, wl.flux_F)

    def run(ops, charge=1.0, solid=s):
        M = orc.mdnorm_matrices(wl.R, wl.UB, ops, wl.W)
        return orc.mdnorm(grid, d, solid, *args, M, np.full(len(M), charge), wl.k_min, wl.k_max)

    base = run(wl.ops)
    assert base.sum() > 0
    rng = np.random.default_rng(5)
    perm = run(wl.ops[rng.permutation(24)])
    np.testing.assert_allclose(perm, base, rtol=1e-13, atol=1e-13 * base.max())
    g = wl.ops[7]
    left = run(np.stack([g @ S for S in wl.ops]))
    np.testing.assert_allclose(left, base, rtol=1e-13, atol=1e-13 * base.max())
    inv = run(np.stack([np.round(np.linalg.inv(S)) for S in wl.ops]))
    np.testing.assert_allclose(inv, base, rtol=1e-13, atol=1e-13 * base.max())
    one = run(wl.ops[:1])
    two = run(np.stack([wl.ops[0], wl.ops[0]]))
    np.testing.assert_allclose(two, 2 * one, rtol=1e-15, atol=0)
    assert np.array_equal(run(wl.ops[:3], charge=2.0), 2 * run(wl.ops[:3]))
    assert np.array_equal(run(wl.ops[:3], solid=2 * s), 2 * run(wl.ops[:3]))


def test_sharding_invariance(orc):
    """Algorithm 1: the sum of G per-rank partial histograms (pixel stride or
    run blocks) equals the single-process result to rounding."""
    wl, grid, d, s = _corelli_subset(orc, stride=499)
    M = orc.mdnorm_matrices(wl.R, wl.UB, wl.ops[:6], wl.W)
    c = np.ones(len(M))
    full = orc.mdnorm(grid, d, s, wl.flux_k, wl.flux_F, M, c, wl.k_min, wl.k_max)
    for G in (2, 3, 8):
        parts = sum(orc.mdnorm(grid, d, s, wl.flux_k, wl.flux_F, M, c, wl.k_min, wl.k_max,
                               pix_begin=g, pix_stride=G) for g in range(G))
        np.testing.assert_allclose(parts, full, rtol=1e-14, atol=1e-14 * full.max())
    # run-block split of a 4-run scan
    R4 = np.stack([synth.rot_y(3.0 * r) for r in range(4)])
    M4 = orc.mdnorm_matrices(R4, wl.UB, wl.ops[:2], wl.W)
    c4 = np.ones(len(M4))
    full4 = orc.mdnorm(grid, d, s, wl.flux_k, wl.flux_F, M4, c4, wl.k_min, wl.k_max)
    a = orc.mdnorm(grid, d, s, wl.flux_k, wl.flux_F, M4[:4], c4[:4], wl.k_min, wl.k_max)
    b = orc.mdnorm(grid, d, s, wl.flux_k, wl.flux_F, M4[4:], c4[4:], wl.k_min, wl.k_max)
    np.testing.assert_allclose(a + b, full4, rtol=1e-14, atol=1e-14 * full4.max())


def test_binmd_bin_centres_and_full_cover(orc):
    """BinMD: events at bin centres give exact integer counts; a grid covering every transformed
    event receives n_s * sum(w) in total (weight conservation)."""
    grid = orc.Grid([-1.25, -2.0, 0.5], [1.25, 2.0, 3.5], [10, 8, 6])
    cx = -1.25 + (np.arange(10) + 0.5) * 0.25
    cy = -2.0 + (np.arange(8) + 0.5) * 0.5
    cz = 0.5 + (np.arange(6) + 0.5) * 0.5
    X, Y, Z = np.meshgrid(cx, cy, cz, indexing="ij")
    q = np.stack([X.ravel(), Y.ravel(), Z.ravel()], axis=1)
    ev = np.concatenate([np.ones((len(q), 1)), q], axis=1).astype(np.float32)
    h = orc.binmd(grid, np.stack([np.eye(3), np.eye(3)]), ev)
    np.testing.assert_array_equal(h, np.full(grid.nbins, 2.0))
    wl = synth.make_workload("corelli", events_per_run=20000)
    evs = synth.events_for_run(wl, 0)
    N = orc.binmd_matrices(wl.UB, wl.ops, wl.W)
    big = orc.Grid([-100, -100, -100], [100, 100, 100], [7, 5, 3])
    tot = orc.binmd(big, N, evs).sum()
    expect = 24 * evs[:, 0].astype(np.float64).sum()
    assert abs(tot - expect) <= 1e-12 * expect


def test_binmd_permutation_of_ops(orc):
    wl = synth.make_workload("corelli", events_per_run=20000)
    evs = synth.events_for_run(wl, 0)
    grid = orc.Grid(wl.lo, wl.hi, [60, 60, 1])
    N = orc.binmd_matrices(wl.UB, wl.ops, wl.W)
    a = orc.binmd(grid, N, evs)
    b = orc.binmd(grid, N[np.random.default_rng(6).permutation(24)], evs)
    np.testing.assert_allclose(a, b, rtol=1e-13, atol=1e-13 * a.max())
    assert a.sum() > 0


# ----------------------------------------------------------------------------- MDNorm <-> BinMD


@pytest.mark.parametrize("ops", ["one", "6/mmm"])
def test_flat_sq_statistical(orc, ops):
    """Flat-S(Q) pin: events drawn from the normalization measure itself make
    xs constant = N_ev / (c * sum Omega * (F(k_max) - F(k_min))) within Poisson error.  This is
    the pin on the Q sign, the 2 pi and the matrix composition agreeing between the two halves."""
    wl = synth.make_workload("tiny", events_per_run=200_000)
    if ops == "6/mmm":
        wl.ops = synth.hex_6mmm_ops()
    grid = orc.workload_grid(wl)
    ev = synth.events_for_run(wl, 0)
    norm, bm, xs = orc.run_workload(wl, events={0: ev})
    F = lambda k: orc.flux(wl.flux_k, wl.flux_F, k)  # noqa: E731
    C = len(ev) / (wl.charge[0] * wl.solid.sum() * (F(wl.k_max) - F(wl.k_min)))
    assert np.all(bm[norm == 0] == 0), "events landed where no trajectory passes"
    sel = bm >= 400
    assert sel.sum() >= 20
    z = (xs[sel] / C - 1.0) * np.sqrt(bm[sel] / len(wl.ops))
    assert np.all(np.abs(z) < 5.5), np.abs(z).max()
    inside_frac = bm.sum() / (len(ev) * len(wl.ops))
    assert abs(bm.sum() / norm.sum() / C - 1) < 5 / math.sqrt(inside_frac * len(ev))
    assert np.all(np.isnan(xs[norm == 0]))


def test_cross_section_nan_mask(orc):
    """X2 reading #12: xs = binmd/norm where norm > 0, NaN where norm == 0."""
    norm = np.array([0.0, 1.0, 2.0, 0.0, 4.0])
    bm = np.array([0.0, 3.0, 1.0, 5.0, 0.0])
    xs = orc.cross_section(bm, norm)
    assert np.isnan(xs[0]) and np.isnan(xs[3])
    assert xs[1] == 3.0 and xs[2] == 0.5 and xs[4] == 0.0


# ----------------------------------------------------------------------------- NEXT #1 inputs


def test_pixel_krange_closed_form_and_additivity(orc):
    """Per-pixel momentum limits (Mantid MDNorm_low/high): each pixel's trajectory is clipped to
    [max(k_min, lo_p), min(k_max, hi_p)] -- closed form on axis-aligned trajectories, identity when
    the limits equal the global range, additivity when the range is split at k_c."""
    rng = np.random.default_rng(21)
    phi0 = 2.0
    fk, fF = np.array([0.5, 30.0]), np.array([0.0, phi0 * 29.5])
    n2, lo2, hi2 = 17, 0.5, 25.0
    grid = orc.Grid([-1e3, -1e3, lo2], [1e3, 1e3, hi2], [1, 1, n2])
    d = rng.normal(size=(12, 3))
    d /= np.linalg.norm(d, axis=1)[:, None]
    d = d[1 - d[:, 2] > 0.1]
    s = rng.uniform(0.5, 2.0, len(d))
    alpha = 0.8
    kmin, kmax = 1.5, 18.0
    plo = rng.uniform(1.0, 8.0, len(d))
    phi = plo + rng.uniform(0.5, 9.0, len(d))
    h = orc.mdnorm_krange(grid, d, s, plo, phi, fk, fF, (alpha * np.eye(3))[None], [1.0], kmin, kmax)
    expect = sum(_closed_form_axis2(lo2, hi2, n2, alpha * (1 - dp[2]), max(kmin, a), min(kmax, b), sp, phi0)
                 for dp, sp, a, b in zip(d, s, plo, phi))
    np.testing.assert_allclose(h, expect, rtol=1e-12, atol=1e-12 * expect.max())
    wl = synth.make_workload("corelli")
    g2 = orc.Grid(wl.lo, wl.hi, [60, 60, 1])
    dd, ss = wl.pix_dir[::997], wl.solid[::997]
    M = orc.mdnorm_matrices(wl.R, wl.UB, wl.ops[:4], wl.W)
    ones = np.ones(len(ss))
    base = orc.mdnorm(g2, dd, ss, wl.flux_k, wl.flux_F, M, 1.0, wl.k_min, wl.k_max)
    same = orc.mdnorm_krange(g2, dd, ss, wl.k_min * ones, wl.k_max * ones, wl.flux_k, wl.flux_F, M, 1.0,
                             wl.k_min, wl.k_max)
    assert np.array_equal(base, same)
    kc = 5.3
    lower = orc.mdnorm_krange(g2, dd, ss, None, kc * ones, wl.flux_k, wl.flux_F, M, 1.0, wl.k_min, wl.k_max)
    upper = orc.mdnorm_krange(g2, dd, ss, kc * ones, None, wl.flux_k, wl.flux_F, M, 1.0, wl.k_min, wl.k_max)
    np.testing.assert_allclose(lower + upper, base, rtol=1e-11, atol=1e-11 * base.max())
    none = orc.mdnorm_krange(g2, dd, ss, 20.0 * ones, None, wl.flux_k, wl.flux_F, M, 1.0, wl.k_min, wl.k_max)
    assert not none.any()


def test_error_histogram_pins(orc):
    """Error-squared histogram (8-column events: signal col 0, error^2 col 1, Q cols 5-7):
    err2 equals the weight histogram when err^2 = w (Poisson counts); the hand example of
    tests/golden/binmd_hand.json with err^2 = w^2 gives the squared weights; duplicating every
    event doubles binmd and err2, so xs is unchanged and xs_err scales by 1/sqrt(2)."""
    wl = synth.make_workload("corelli", events_per_run=30000)
    ev = synth.events_for_run(wl, 0)
    ev8 = np.zeros((len(ev), 8), np.float32)
    ev8[:, 0] = ev[:, 0]
    ev8[:, 1] = ev[:, 0]
    ev8[:, 5:8] = ev[:, 1:4]
    g = orc.Grid(wl.lo, wl.hi, [60, 60, 1])
    N = orc.binmd_matrices(wl.UB, wl.ops, wl.W)
    b = orc.binmd(g, N, ev8, col_w=0, col_q=5)
    e2 = orc.binmd_err(g, N, ev8, col_e=1, col_q=5)
    assert np.array_equal(b, e2) and b.sum() > 0
    gj = _golden("binmd_hand.json")
    grid = orc.Grid(gj["grid"]["lo"], gj["grid"]["hi"], gj["grid"]["n"])
    hev = np.array(gj["events"], dtype=np.float32)
    hev8 = np.zeros((len(hev), 8), np.float32)
    hev8[:, 0] = hev[:, 0]
    hev8[:, 1] = hev[:, 0] ** 2
    hev8[:, 5:8] = hev[:, 1:4]
    he = orc.binmd_err(grid, np.array(gj["N"]), hev8, col_e=1, col_q=5)
    expect = np.zeros(grid.nbins)
    expect[0], expect[3], expect[57] = 4.0 + 9.0 + 9.0, 1.0, 0.0625
    np.testing.assert_array_equal(he, expect)
    norm = orc.mdnorm(g, wl.pix_dir[::97], wl.solid[::97], wl.flux_k, wl.flux_F,
                      orc.mdnorm_matrices(wl.R, wl.UB, wl.ops, wl.W), 1.0, wl.k_min, wl.k_max)
    x1, s1 = orc.cross_section(b, norm), orc.cross_section_err(e2, norm)
    x2, s2 = orc.cross_section(2 * b, 2 * norm), orc.cross_section_err(2 * e2, 2 * norm)
    ok = ~np.isnan(x1)
    assert np.array_equal(np.isnan(s1), np.isnan(x1))
    np.testing.assert_allclose(x2[ok], x1[ok], rtol=1e-15)
    np.testing.assert_allclose(s2[ok], s1[ok] / math.sqrt(2.0), rtol=1e-15)


# ----------------------------------------------------------------------------- second pins (r02)


def test_segments_have_positive_length(orc):
    """Reading #7 (skip only k2 <= k1): on a diagonal trajectory whose H and K crossings
    coincide at every grid corner (v = (a, a, 0), square bins), L has tied entries; the oracle
    keeps exactly one segment per distinct pair of consecutive values, every one of positive
    value under a flux of positive density -- n_seg = distinct crossings + 1 (closed form)."""
    a = 0.37
    M = np.diag([a, a, 0.0]) / a  # v = M q; q = z - d with d chosen so q = (1, 1, 0) * s
    # pixel direction with q = z - d = (c, c, 0): d = (-c, -c, 1); not unit -- the oracle takes d as given
    c = 0.8
    d = np.array([-c, -c, 1.0])
    lo, hi, n = [0.0, 0.0, -1.0], [4.0, 4.0, 1.0], [8, 8, 1]
    grid = orc.Grid(lo, hi, n)
    fk, fF = np.array([0.1, 50.0]), np.array([0.0, 49.9])  # uniform density 1
    kmin, kmax = 0.3, 4.7
    nc, ns, bins, vals = orc.mdnorm_trajectory(grid, d, 1.0, fk, fF, M, 1.0, kmin, kmax)
    # x(k) = k c (1, 1, 0): inside for k c in [0, 4); every plane j * 0.5 crosses both axes at once
    kin, kout = kmin, min(kmax, 4.0 / c)
    distinct = [j * 0.5 / c for j in range(1, 8) if kin < j * 0.5 / c < kout]
    assert ns == len(distinct) + 1
    assert np.all(vals > 0)
    assert np.isclose(vals.sum(), kout - kin, rtol=1e-13)


def test_rotated_goniometer_bragg_trajectory(orc):
    """Second pin on the composition order M = (R UB S W)^-1 / 2 pi (reading #2) through the
    trajectory geometry: for a reflection h, the physics forward model gives Q_lab = R 2 pi UB h;
    the elastic pixel that sees it is d = z - Q_lab / k* with k* = |Q|^2 / (2 Q_z).  That pixel's
    trajectory (goniometer R, a narrow k window around k*) must cross the bin of x = W^-1 h."""
    wl = synth.make_workload("corelli")
    rng = np.random.default_rng(5)
    hits = 0
    for _ in range(40):
        h = rng.integers(-4, 5, 3).astype(float)
        h[2] = rng.integers(-2, 3)
        if not h.any():
            continue
        R = synth.rot_y(rng.uniform(0, 360)) @ synth.rot_x(rng.uniform(-20, 20))
        Q = R @ (2 * math.pi * wl.UB @ h)
        if Q[2] <= 1e-3:
            continue  # not reachable in the elastic geometry (needs Q_z > 0)
        kst = Q @ Q / (2 * Q[2])
        d = np.array([0.0, 0.0, 1.0]) - Q / kst
        x = np.linalg.solve(wl.W, h)
        # grid of 1e-3-wide bins centred on x
        w = 1e-3
        lo = x - 1.5 * w
        grid = orc.Grid(lo, lo + 3 * w, [3, 3, 3])
        M = orc.compose_mdnorm(R, wl.UB, np.eye(3), wl.W)
        fk, fF = np.array([0.01, 1e4]), np.array([0.0, 1e4])
        nc, ns, bins, vals = orc.mdnorm_trajectory(grid, d, 1.0, fk, fF, M, 1.0, kst * (1 - 1e-6), kst * (1 + 1e-6))
        assert ns > 0, (h, kst)
        assert 13 in bins.tolist(), (h, bins)  # the centre bin (1, 1, 1) of the 3x3x3 grid
        hits += 1
    assert hits >= 10
