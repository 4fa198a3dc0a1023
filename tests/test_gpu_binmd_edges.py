"""B2/B3 at bin edges: events whose grid coordinates fall on, or within a few fp32 ulps of, bin
planes and grid faces -- exactly where the fp32 decisions of binmd_kernel cannot decide and the
exact fp64 formula per axis (member_bin's fallback, the first axis' -2 path) has to.  Unit weights
make every bin an exact count, so the bar is bit-exact: the histogram equals the oracle's
(Listing 3; DESIGN.md §4 "Decisions") and binmd_debug_bins equals oracle.binmd_bins."""
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


def edge_events(N, lo, hi, n, count, rng):
    """Unit-weight float4 events (w, Q) whose coordinates x = N_s Q (for a random op s) sit on
    random bin planes or grid faces of every axis, nudged by -3..3 fp32 ulps of Q."""
    lo, hi, n = (np.asarray(a, float) for a in (lo, hi, n))
    w = (hi - lo) / n
    j = np.stack([rng.integers(0, n[a] + 1, count) for a in range(3)], 1)  # plane index 0..n
    x = lo + j * w
    # some coordinates strictly inside a bin (so a pair can land inside on the other axes)
    inner = rng.random((count, 3)) < 0.3
    x = np.where(inner, lo + (rng.integers(0, n, (count, 3)) + rng.random((count, 3))) * w, x)
    s = rng.integers(0, len(N), count)
    q = np.einsum("eij,ej->ei", np.linalg.inv(N)[s], x).astype(np.float32)
    steps = rng.integers(-3, 4, (count, 3))
    steps[rng.random((count, 3)) < 0.25] = 0  # a quarter exactly as rounded
    up, down = np.float32(np.inf), np.float32(-np.inf)
    for _ in range(3):
        q = np.where(steps > 0, np.nextafter(q, up), np.where(steps < 0, np.nextafter(q, down), q))
        steps = steps - np.sign(steps)
    ev = np.empty((count, 4), np.float32)
    ev[:, 0] = 1.0
    ev[:, 1:] = q
    return ev


@pytest.mark.parametrize("cfg", ["corelli", "topaz"])
def test_binmd_events_on_bin_planes(mdn, cfg):
    import torch
    wl = synth.make_workload(cfg, nops=48) if cfg == "topaz" else synth.make_workload(cfg)
    N = oracle.binmd_matrices(wl.UB, wl.ops, wl.W)
    rng = np.random.default_rng(21)
    ev = edge_events(N, wl.lo, wl.hi, wl.nbins, 400_000, rng)
    og = oracle.workload_grid(wl)
    g = mdn.mdnorm_create_grid(0, wl.lo, wl.hi, wl.nbins, wl.W, mdn.MDN_ACC_F64)
    mdn.mdnorm_set_privatization(g, 0)
    mdn.binmd_accumulate(g, wl.UB, wl.ops, torch.from_numpy(ev).cuda())
    torch.cuda.synchronize()
    bm = mdn.packed_histograms(g).cpu().numpy()[g.nbins_total:2 * g.nbins_total]
    obm = oracle.binmd(og, N, ev)
    assert np.array_equal(bm, obm)
    assert obm.sum() > 10_000  # plenty of in-grid pairs
    # the per-pair decisions, including those of pairs outside the grid
    sub = ev[::7]
    Ns = N[:: max(1, len(N) // 12)]
    gb = mdn.binmd_debug_bins(g, Ns, sub)
    ob = oracle.binmd_bins(og, Ns, sub)
    assert np.array_equal(gb, ob)
    # the events really sit on planes: many pairs are within 1e-6 of a bin edge in fp64
    x = np.einsum("mij,ej->mei", Ns, sub[:, 1:].astype(np.float64))
    t = (x - np.asarray(wl.lo)) / ((np.asarray(wl.hi) - np.asarray(wl.lo)) / np.asarray(wl.nbins))
    assert (np.abs(t - np.round(t)) < 1e-6).mean() > 0.1


def test_binmd_edges_privatised(mdn):
    """The same edge events into a coarse grid that fits shared memory (private histograms)."""
    import torch
    wl = synth.make_workload("corelli")
    lo, hi, n = [-7.5, -7.5, -0.1], [7.5, 7.5, 0.1], [60, 60, 1]
    N = oracle.binmd_matrices(wl.UB, wl.ops, wl.W)
    ev = edge_events(N, lo, hi, n, 300_000, np.random.default_rng(4))
    g = mdn.mdnorm_create_grid(0, lo, hi, n, wl.W, mdn.MDN_ACC_F64)
    mdn.mdnorm_set_privatization(g, 1)
    mdn.binmd_accumulate(g, wl.UB, wl.ops, torch.from_numpy(ev).cuda())
    torch.cuda.synchronize()
    assert mdn.mdnorm_accumulation_paths(g)[1] != "global"
    bm = mdn.packed_histograms(g).cpu().numpy()[g.nbins_total:2 * g.nbins_total]
    assert np.array_equal(bm, oracle.binmd(oracle.Grid(lo, hi, n), N, ev))
