"""GPU parity: the CUDA path (through the C ABI) against the fp64 CPU oracle, on the same seeded
synthetic inputs (BASELINE.json configs).  Bar (BASELINE north_star):
  * crossing counts, segment bin indices and event bin indices: bit-exact;
  * histogram values (MDN_ACC_F64): |gpu - oracle| <= 1e-12 |oracle| per bin, zero <=> zero;
  * xs NaN masks identical.
"""
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


def make_grid(mdn, wl, lo=None, hi=None, nbins=None):
    g = mdn.mdnorm_create_grid(0, wl.lo if lo is None else lo, wl.hi if hi is None else hi,
                               wl.nbins if nbins is None else nbins, wl.W, mdn.MDN_ACC_F64)
    mdn.mdnorm_set_instrument(g, wl.pix_dir, wl.solid)
    mdn.mdnorm_set_flux(g, wl.flux_k, wl.flux_F)
    return g


def hist(mdn, g):
    import torch
    torch.cuda.synchronize()
    t = mdn.packed_histograms(g).cpu().numpy()
    n = g.nbins_total
    return t[:n].copy(), t[n:2 * n].copy()


def assert_rel(gpu, ref, rel=REL64, what="hist"):
    assert gpu.shape == ref.shape
    assert np.array_equal(gpu == 0, ref == 0), f"{what}: zero pattern differs"
    err = np.abs(gpu - ref)
    bad = err > rel * np.abs(ref)
    assert not bad.any(), f"{what}: {bad.sum()} bins off, worst rel {(err / np.maximum(np.abs(ref), 1e-300)).max():.3e}"


def dev_events(ev):
    import torch
    return torch.from_numpy(ev).cuda()


# ----------------------------------------------------------------------------- M0 / B0


@pytest.mark.parametrize("cfg", ["tiny", "corelli", "topaz", "multirun"])
def test_compose_bit_exact(mdn, cfg):
    wl = synth.make_workload(cfg, nruns=5) if cfg == "multirun" else synth.make_workload(cfg)
    g = make_grid(mdn, wl)
    R = wl.R[:5]
    M, N = mdn.mdnorm_debug_compose(g, wl.UB, R, wl.ops)
    assert np.array_equal(M, oracle.mdnorm_matrices(R, wl.UB, wl.ops, wl.W))
    assert np.array_equal(N, oracle.binmd_matrices(wl.UB, wl.ops, wl.W))


# ----------------------------------------------------------------------------- tiny (configs[0])


def test_tiny_full_parity(mdn):
    wl = synth.make_workload("tiny")
    g = make_grid(mdn, wl)
    ev = synth.events_for_run(wl, 0)
    mdn.mdnorm_accumulate(g, wl.UB, wl.R[0], wl.ops, wl.k_min, wl.k_max, wl.charge[0])
    mdn.binmd_accumulate(g, wl.UB, wl.ops, dev_events(ev))
    norm, bm = hist(mdn, g)
    onorm, obm, oxs = oracle.run_workload(wl, events={0: ev})
    assert_rel(norm, onorm, what="norm")
    assert np.array_equal(bm, obm), "unit-weight BinMD counts must be exact"
    xs = mdn.mdnorm_cross_section(g)
    assert np.array_equal(np.isnan(xs), np.isnan(oxs))
    ok = ~np.isnan(oxs)
    assert np.all(np.abs(xs[ok] - oxs[ok]) <= 3e-12 * np.abs(oxs[ok]))


def _traj_check(mdn, g, wl, M, charge, ids, orc_grid, max_segs=1024):
    nc, ns, bins, vals = mdn.mdnorm_debug_trajectories(g, M, charge, wl.k_min, wl.k_max, ids, max_segs)
    npix = wl.npix
    for t, tid in enumerate(ids):
        m, p = divmod(int(tid), npix)
        onc, ons, obins, ovals = oracle.mdnorm_trajectory(orc_grid, wl.pix_dir[p], wl.solid[p], wl.flux_k,
                                                          wl.flux_F, M[m], charge[m], wl.k_min, wl.k_max,
                                                          max_segs)
        assert nc[t] == onc, (tid, nc[t], onc)
        assert ns[t] == ons, (tid, ns[t], ons)
        k = min(ons, max_segs)
        assert np.array_equal(bins[t, :k], obins), tid
        assert np.array_equal(vals[t, :k], ovals), tid  # same IEEE operations -> same bits
    return nc, ns


@pytest.mark.parametrize("cfg", ["tiny", "corelli", "topaz", "stress"])
def test_debug_trajectories_bit_exact(mdn, cfg):
    wl = synth.make_workload(cfg)
    g = make_grid(mdn, wl)
    og = oracle.workload_grid(wl)
    M = oracle.mdnorm_matrices(wl.R[:1], wl.UB, wl.ops[:min(wl.nops, 64)], wl.W)
    charge = np.full(len(M), 1.25)
    rng = np.random.default_rng(7)
    n = 64 if cfg == "tiny" else 3000
    ids = rng.integers(0, len(M) * wl.npix, size=n)
    if cfg == "corelli":  # make sure plenty of hitters are included (3.9% hit the slab)
        nc, _ = _traj_check(mdn, g, wl, M, charge, ids, og)
        assert (nc > 0).sum() > 50
        return
    nc, ns = _traj_check(mdn, g, wl, M, charge, ids, og)
    assert (nc > 0).sum() > 0


def test_debug_trajectory_truncation_and_golden(mdn):
    """max_segs smaller than n_seg keeps the first segments; golden backscatter example."""
    import json, os
    gj = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "mdnorm_backscatter_axis2.json")))
    g = mdn.mdnorm_create_grid(0, gj["grid"]["lo"], gj["grid"]["hi"], gj["grid"]["n"], np.eye(3))
    mdn.mdnorm_set_instrument(g, np.array([gj["dir"]]), np.array([gj["solid"]]))
    mdn.mdnorm_set_flux(g, np.array(gj["flux_k"]), np.array(gj["flux_F"]))
    M = np.array(gj["M"])[None]
    nc, ns, bins, vals = mdn.mdnorm_debug_trajectories(g, M, [gj["charge"]], gj["k_min"], gj["k_max"], [0], 2)
    assert nc[0] == gj["expect_n_cross"] and ns[0] == 4
    assert bins[0].tolist() == gj["expect_seg_bins"][:2]
    assert vals[0].tolist() == gj["expect_seg_vals"][:2]
    mdn.mdnorm_accumulate_matrices(g, M, [gj["charge"]], gj["k_min"], gj["k_max"])
    norm, _ = hist(mdn, g)
    assert norm.tolist() == gj["expect_seg_vals"]


# ----------------------------------------------------------------------------- CORELLI (configs[1])


@pytest.fixture(scope="module")
def corelli():
    wl = synth.make_workload("corelli")
    ev = synth.events_for_run(wl, 0)
    return wl, ev


def test_corelli_full_size_parity(mdn, corelli):
    """The bench launch configuration at full size: 24 ops x 372,736 pixels, 10^7 events."""
    wl, ev = corelli
    g = make_grid(mdn, wl)
    mdn.mdnorm_accumulate(g, wl.UB, wl.R[0], wl.ops, wl.k_min, wl.k_max, wl.charge[0])
    mdn.binmd_accumulate(g, wl.UB, wl.ops, dev_events(ev))
    norm, bm = hist(mdn, g)
    onorm, obm, oxs = oracle.run_workload(wl, events={0: ev})
    assert_rel(norm, onorm, what="norm")
    assert_rel(bm, obm, what="binmd")
    xs = mdn.mdnorm_cross_section(g)
    assert np.array_equal(np.isnan(xs), np.isnan(oxs))
    ok = ~np.isnan(oxs)
    assert np.all(np.abs(xs[ok] - oxs[ok]) <= 3e-12 * np.abs(oxs[ok]))


def test_corelli_unit_weight_counts_exact(mdn, corelli):
    """Unit weights make every BinMD bin an exact integer count: bit-exact event bin indices."""
    wl, _ = corelli
    ev = synth.events_for_run(wl, 0, n=2_000_000, unit_weights=True)
    g = make_grid(mdn, wl)
    mdn.binmd_accumulate(g, wl.UB, wl.ops, dev_events(ev))
    _, bm = hist(mdn, g)
    obm = oracle.binmd(oracle.workload_grid(wl), oracle.binmd_matrices(wl.UB, wl.ops, wl.W), ev)
    assert np.array_equal(bm, obm)
    N = oracle.binmd_matrices(wl.UB, wl.ops[:8], wl.W)
    sub = ev[::97]
    assert np.array_equal(mdn.binmd_debug_bins(g, N, sub), oracle.binmd_bins(oracle.workload_grid(wl), N, sub))


def test_corelli_strided_and_host_events(mdn, corelli):
    """8-column strided events (P:188 layout: weight col 1, Q cols 6-8) and host (pageable and
    pinned) event buffers give the same histogram as packed device float4 events."""
    import torch
    wl, ev = corelli
    ev = ev[:3_000_001]  # ragged
    ops = wl.ops[:6]
    ev8 = np.zeros((len(ev), 8), np.float32)
    ev8[:, 0] = ev[:, 0]
    ev8[:, 1] = ev[:, 0] ** 2
    ev8[:, 5:8] = ev[:, 1:4]
    outs = []
    for src, kw in [(dev_events(ev), {}), (ev, {}), (torch.from_numpy(ev).pin_memory(), {}),
                    (dev_events(ev8), dict(col_w=0, col_q=5)), (ev8, dict(col_w=0, col_q=5))]:
        g = make_grid(mdn, wl)
        mdn.binmd_accumulate(g, wl.UB, ops, src, **kw)
        outs.append(hist(mdn, g)[1])
    obm = oracle.binmd(oracle.workload_grid(wl), oracle.binmd_matrices(wl.UB, ops, wl.W), ev)
    for o in outs:
        assert_rel(o, obm, what="binmd")


def test_shard_sum_on_one_gpu(mdn, corelli):
    """T3 emulation: G grids each taking pixels p = g mod G and event block g sum to the
    single-grid result (P:100 per-rank histograms + reduce)."""
    from paper_conf_sc_hahnfgmmshvvs24_b200 import plan_shards
    wl, ev = corelli
    ev = ev[:1_000_000]
    g1 = make_grid(mdn, wl)
    mdn.mdnorm_accumulate(g1, wl.UB, wl.R[0], wl.ops, wl.k_min, wl.k_max, 1.0)
    mdn.binmd_accumulate(g1, wl.UB, wl.ops, dev_events(ev))
    ref_n, ref_b = hist(mdn, g1)
    for G in (2, 3, 8):
        tot_n, tot_b = 0, 0
        for r in range(G):
            p = plan_shards(G, r, 1, wl.npix, len(ev))
            g = make_grid(mdn, wl)
            mdn.mdnorm_accumulate(g, wl.UB, wl.R[0], wl.ops, wl.k_min, wl.k_max, 1.0,
                                  pix_begin=p.pix_begin, pix_stride=p.pix_stride)
            b, e = p.event_ranges[0]
            mdn.binmd_accumulate(g, wl.UB, wl.ops, dev_events(ev[b:e]))
            n_, b_ = hist(mdn, g)
            tot_n, tot_b = tot_n + n_, tot_b + b_
        assert_rel(tot_n, ref_n, rel=1e-12, what=f"norm G={G}")
        assert_rel(tot_b, ref_b, rel=1e-12, what=f"binmd G={G}")


def test_determinism_and_reset(mdn, corelli):
    wl, ev = corelli
    g = make_grid(mdn, wl)
    outs = []
    for _ in range(2):
        mdn.mdnorm_reset(g)
        mdn.mdnorm_accumulate(g, wl.UB, wl.R[0], wl.ops[:4], wl.k_min, wl.k_max, 1.0)
        outs.append(hist(mdn, g)[0])
    assert_rel(outs[0], outs[1], rel=1e-13, what="repeat")


# ----------------------------------------------------------------------------- TOPAZ (configs[2])


@pytest.mark.parametrize("nops", [1, 8, 48])
def test_topaz_pixel_subsample_parity(mdn, nops):
    """TOPAZ-shaped 200^3 grid, op sweep: every 2003rd pixel through the production kernel."""
    wl = synth.make_workload("topaz", nops=nops)
    g = make_grid(mdn, wl)
    stride = 2003
    mdn.mdnorm_accumulate(g, wl.UB, wl.R[0], wl.ops, wl.k_min, wl.k_max, 1.0, pix_stride=stride)
    norm, _ = hist(mdn, g)
    M = oracle.mdnorm_matrices(wl.R, wl.UB, wl.ops, wl.W)
    onorm = oracle.mdnorm(oracle.workload_grid(wl), wl.pix_dir, wl.solid, wl.flux_k, wl.flux_F, M, 1.0,
                          wl.k_min, wl.k_max, pix_stride=stride)
    assert_rel(norm, onorm, what="norm")


def test_topaz_full_size_properties(mdn):
    """Full TOPAZ-shaped launch (1.64M px x 8 ops): linearity over pixel shards (a property that
    holds at any size: four interleaved shards sum to the one launch) and 2M of its events
    through BinMD against the oracle.  The full launch itself is compared with the oracle bin by
    bin in tests/test_gpu_fullsize.py::test_topaz_8ops_full_pixels."""
    wl = synth.make_workload("topaz", nops=8)
    g = make_grid(mdn, wl)
    mdn.mdnorm_accumulate(g, wl.UB, wl.R[0], wl.ops, wl.k_min, wl.k_max, 1.0)
    full, _ = hist(mdn, g)
    parts = 0
    for r in range(4):
        gg = make_grid(mdn, wl)
        mdn.mdnorm_accumulate(gg, wl.UB, wl.R[0], wl.ops, wl.k_min, wl.k_max, 1.0, pix_begin=r, pix_stride=4)
        parts = parts + hist(mdn, gg)[0]
    assert_rel(parts, full, rel=1e-12, what="shards")
    events = synth.events_for_run(wl, 0, n=2_000_000)
    mdn.binmd_accumulate(g, wl.UB, wl.ops, dev_events(events))
    _, bm = hist(mdn, g)
    obm = oracle.binmd(oracle.workload_grid(wl), oracle.binmd_matrices(wl.UB, wl.ops, wl.W), events)
    assert_rel(bm, obm, what="binmd")


# ----------------------------------------------------------------------------- stress (configs[4])


def test_stress_500_cubed(mdn):
    """BASELINE configs[4] grid (500^3 = 1.25e8 bins, 1 GB fp64 histograms: the global-reduction
    path) with 48 ops, in the bench's launch configuration: every 4099th pixel through the
    production kernels against the oracle per bin, and 10^6 of its events through BinMD."""
    wl = synth.make_workload("stress", events_per_run=1_000_000)
    g = make_grid(mdn, wl)
    stride = 4099
    mdn.mdnorm_accumulate(g, wl.UB, wl.R[0], wl.ops, wl.k_min, wl.k_max, 1.0, pix_stride=stride)
    ev = synth.events_for_run(wl, 0)
    mdn.binmd_accumulate(g, wl.UB, wl.ops, dev_events(ev))
    assert mdn.mdnorm_accumulation_paths(g) == ("global", "global")
    norm, bm = hist(mdn, g)
    og = oracle.workload_grid(wl)
    M = oracle.mdnorm_matrices(wl.R, wl.UB, wl.ops, wl.W)
    onorm = oracle.mdnorm(og, wl.pix_dir, wl.solid, wl.flux_k, wl.flux_F, M, 1.0, wl.k_min, wl.k_max,
                          pix_stride=stride)
    assert_rel(norm, onorm, what="norm")
    del onorm, norm
    obm = oracle.binmd(og, oracle.binmd_matrices(wl.UB, wl.ops, wl.W), ev)
    assert_rel(bm, obm, what="binmd")


# ----------------------------------------------------------------------------- multi-run (configs[3])


def test_multirun_batched_parity(mdn):
    """Rotation scan: 20 runs x 24 ops through mdnorm_accumulate_runs (two launches) on every
    37th pixel, and 2 runs' events, against Algorithm 1 on the oracle."""
    wl = synth.make_workload("multirun", nruns=20, events_per_run=300_000)
    g = make_grid(mdn, wl)
    stride = 37
    mdn.mdnorm_accumulate_runs(g, wl.UB, wl.R, wl.charge, wl.ops, wl.k_min, wl.k_max, pix_stride=stride)
    evs = {r: synth.events_for_run(wl, r) for r in range(2)}
    for r in range(2):
        mdn.binmd_accumulate(g, wl.UB, wl.ops, dev_events(evs[r]))
    norm, bm = hist(mdn, g)
    M = oracle.mdnorm_matrices(wl.R, wl.UB, wl.ops, wl.W)
    charge = np.repeat(wl.charge, wl.nops)
    og = oracle.workload_grid(wl)
    onorm = oracle.mdnorm(og, wl.pix_dir, wl.solid, wl.flux_k, wl.flux_F, M, charge, wl.k_min, wl.k_max,
                          pix_stride=stride)
    N = oracle.binmd_matrices(wl.UB, wl.ops, wl.W)
    acc = oracle.Accumulator(og.nbins)
    for r in range(2):
        oracle.binmd(og, N, evs[r], acc=acc)
    assert_rel(norm, onorm, what="norm")
    assert_rel(bm, acc.value(), what="binmd")


# ----------------------------------------------------------------------------- edge cases


def test_edge_cases(mdn):
    wl = synth.make_workload("tiny")
    g = make_grid(mdn, wl)
    # empty event list and empty pixel shard are no-ops
    mdn.binmd_accumulate(g, wl.UB, wl.ops, np.zeros((0, 4), np.float32))
    mdn.mdnorm_accumulate(g, wl.UB, wl.R[0], wl.ops, wl.k_min, wl.k_max, 1.0, pix_begin=10, pix_end=10)
    norm, bm = hist(mdn, g)
    assert not norm.any() and not bm.any()
    # k range that misses the grid entirely
    mdn.mdnorm_accumulate(g, wl.UB, wl.R[0], wl.ops, 1000.0, 2000.0, 1.0)
    assert not hist(mdn, g)[0].any()
    # errors: state, arguments
    g2 = mdn.mdnorm_create_grid(0, wl.lo, wl.hi, wl.nbins, wl.W)
    with pytest.raises(mdn.MdnError, match="MDN_ESTATE"):
        mdn.mdnorm_accumulate(g2, wl.UB, wl.R[0], wl.ops, 2.0, 3.0, 1.0)
    with pytest.raises(mdn.MdnError, match="MDN_EINVAL"):
        mdn.mdnorm_set_flux(g2, np.array([1.0, 1.0]), np.array([0.0, 1.0]))
    with pytest.raises(mdn.MdnError, match="MDN_EINVAL"):
        mdn.mdnorm_set_flux(g2, np.array([1.0, 2.0]), np.array([1.0, 0.0]))
    with pytest.raises(mdn.MdnError, match="MDN_EINVAL"):
        mdn.mdnorm_set_instrument(g2, wl.pix_dir, -wl.solid)
    with pytest.raises(mdn.MdnError, match="MDN_EINVAL"):
        mdn.mdnorm_accumulate(g, wl.UB, wl.R[0], wl.ops, 3.0, 2.0, 1.0)
    with pytest.raises(mdn.MdnError, match="MDN_EINVAL"):
        mdn.mdnorm_accumulate(g, wl.UB, wl.R[0], np.zeros((1, 3, 3)), 2.0, 3.0, 1.0)
    with pytest.raises(mdn.MdnError, match="MDN_EINVAL"):
        mdn.binmd_accumulate(g, wl.UB, wl.ops, np.zeros((4, 4), np.float32), col_q=2)


def test_masked_and_beam_axis_pixels(mdn):
    """Omega = 0 (masked) contributes nothing; a pixel with v_a = 0 on some axis (backscatter,
    M with zero rows) follows reading #17: the whole trajectory stays on that axis' plane."""
    d = np.array([[0.0, 0.0, -1.0], [0.3, 0.4, np.sqrt(1 - 0.25)], [0.0, 0.6, 0.8]])
    s = np.array([1.0, 0.0, 2.0])
    lo, hi, n = [-3.0, -3.0, 0.0], [3.0, 3.0, 12.0], [5, 7, 9]
    g = mdn.mdnorm_create_grid(0, lo, hi, n, np.eye(3))
    mdn.mdnorm_set_instrument(g, d, s)
    fk, fF = np.array([0.5, 8.0]), np.array([0.0, 3.0])
    mdn.mdnorm_set_flux(g, fk, fF)
    M = np.stack([np.eye(3), np.diag([0.0, 1.0, 1.0]), np.diag([1.0, 0.0, 0.5])])
    c = np.array([1.0, 2.0, 0.5])
    mdn.mdnorm_accumulate_matrices(g, M, c, 1.0, 6.0)
    norm, _ = hist(mdn, g)
    og = oracle.Grid(lo, hi, n)
    onorm = oracle.mdnorm(og, d, s, fk, fF, M, c, 1.0, 6.0)
    assert_rel(norm, onorm, what="norm")
    ids = np.arange(9)
    _traj_check(mdn, g, type("W", (), dict(npix=3, pix_dir=d, solid=s, flux_k=fk, flux_F=fF, k_min=1.0,
                                           k_max=6.0))(), M, c, ids, og)


def test_many_planes_ragged_grid(mdn):
    """A 3-D grid with odd, unequal bin counts and a pixel count that is not a multiple of the
    block size (ragged tails), including an op list of 64 matrices (maximum per call)."""
    wl = synth.make_workload("topaz", nops=48)
    rng = np.random.default_rng(9)
    sel = np.sort(rng.choice(wl.npix, 1001, replace=False))
    d, s = wl.pix_dir[sel], wl.solid[sel]
    lo, hi, n = [-9.3, -7.1, -11.0], [8.2, 10.4, 9.9], [101, 37, 253]
    g = mdn.mdnorm_create_grid(0, lo, hi, n, np.eye(3))
    mdn.mdnorm_set_instrument(g, d, s)
    mdn.mdnorm_set_flux(g, wl.flux_k, wl.flux_F)
    M = np.concatenate([oracle.mdnorm_matrices(wl.R, wl.UB, wl.ops, wl.W)[:48],
                        oracle.mdnorm_matrices(wl.R, wl.UB, wl.ops[:16], np.diag([1.0, -1.0, 2.0]))])
    c = rng.uniform(0.5, 1.5, len(M))
    mdn.mdnorm_accumulate_matrices(g, M, c, wl.k_min, wl.k_max)
    norm, _ = hist(mdn, g)
    onorm = oracle.mdnorm(oracle.Grid(lo, hi, n), d, s, wl.flux_k, wl.flux_F, M, c, wl.k_min, wl.k_max)
    assert_rel(norm, onorm, what="norm")
