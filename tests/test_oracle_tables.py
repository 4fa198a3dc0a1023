"""Pins of the oracle's per-bank flux tables (S§8(f) NEXT #1: pixel -> flux-table index)."""
import numpy as np

import synth
from tests.test_oracle_pins import _closed_form_axis2


def _setup(orc):
    wl = synth.make_workload("corelli")
    g = orc.Grid(wl.lo, wl.hi, [60, 60, 1])
    d, s = wl.pix_dir[::499], wl.solid[::499]
    M = orc.mdnorm_matrices(wl.R, wl.UB, wl.ops[:6], wl.W)
    return wl, g, d, s, M


def test_identical_tables_equal_single_table(orc):
    wl, g, d, s, M = _setup(orc)
    rng = np.random.default_rng(41)
    pt = rng.integers(0, 3, len(s)).astype(np.int32)
    tabs = [(wl.flux_k, wl.flux_F)] * 3
    one = orc.mdnorm(g, d, s, wl.flux_k, wl.flux_F, M, 1.0, wl.k_min, wl.k_max)
    three = orc.mdnorm_tables(g, d, s, tabs, pt, M, 1.0, wl.k_min, wl.k_max)
    assert one.sum() > 0 and np.array_equal(one, three)
    none = orc.mdnorm_tables(g, d, s, tabs[:1], None, M, 1.0, wl.k_min, wl.k_max)
    assert np.array_equal(one, none)


def test_doubled_table_equals_doubled_solid_angle(orc):
    """F -> 2F is exact through interpolation and differencing, so a pixel reading a doubled table
    contributes exactly what it would with 2 Omega on the original table."""
    wl, g, d, s, M = _setup(orc)
    rng = np.random.default_rng(42)
    pt = rng.integers(0, 2, len(s)).astype(np.int32)
    tabs = [(wl.flux_k, wl.flux_F), (wl.flux_k, 2.0 * wl.flux_F)]
    a = orc.mdnorm_tables(g, d, s, tabs, pt, M, 1.0, wl.k_min, wl.k_max)
    b = orc.mdnorm(g, d, np.where(pt == 1, 2.0 * s, s), wl.flux_k, wl.flux_F, M, 1.0, wl.k_min, wl.k_max)
    assert np.array_equal(a, b)


def test_uniform_tables_closed_form(orc):
    """Axis-aligned trajectories, each pixel on its own uniform table of slope phi_t."""
    rng = np.random.default_rng(43)
    d = rng.normal(size=(10, 3))
    d /= np.linalg.norm(d, axis=1)[:, None]
    d = d[1 - d[:, 2] > 0.1]
    s = rng.uniform(0.5, 2.0, len(d))
    slopes = [1.0, 2.5, 0.3]
    tabs = [(np.array([0.5, 30.0]), np.array([0.0, ph * 29.5])) for ph in slopes]
    pt = rng.integers(0, 3, len(d)).astype(np.int32)
    n2, lo2, hi2, alpha, kmin, kmax = 13, 0.5, 20.0, 0.9, 1.5, 16.0
    g = orc.Grid([-1e3, -1e3, lo2], [1e3, 1e3, hi2], [1, 1, n2])
    h = orc.mdnorm_tables(g, d, s, tabs, pt, (alpha * np.eye(3))[None], [1.0], kmin, kmax)
    expect = sum(_closed_form_axis2(lo2, hi2, n2, alpha * (1 - dp[2]), kmin, kmax, sp, slopes[t])
                 for dp, sp, t in zip(d, s, pt))
    np.testing.assert_allclose(h, expect, rtol=1e-12, atol=1e-12 * expect.max())
