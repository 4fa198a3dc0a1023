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


def test_binmd_l2_slabs_boundaries(mdn):
    """BinMD on a grid larger than L2 (binmd part 154 MB: two L2 slabs of the last axis, one
    launch each with an axis window, DESIGN.md §4 "BinMD on grids larger than L2"): edge events
    on every bin plane plus events whose op image sits on the slab boundary plane itself (+-3
    fp32 ulps), unit weights -- the histogram equals the oracle's exactly (no pair dropped or
    counted twice at the seam), and the (event, op) pair counter counts each event once."""
    import torch
    wl = synth.make_workload("topaz", nops=48, events_per_run=1000)
    lo, hi, n = [-6.0, -6.0, -3.0], [6.0, 6.0, 3.0], [400, 400, 120]
    N = oracle.binmd_matrices(wl.UB, wl.ops, wl.W)
    rng = np.random.default_rng(33)
    ev = edge_events(N, lo, hi, n, 300_000, rng)
    # the seam: z plane 60 (the slab boundary for two slabs) on the op images' last axis
    seam = edge_events(N, lo, hi, n, 200_000, rng)
    s = rng.integers(0, len(N), seam.shape[0])
    x = np.einsum("eij,ej->ei", N[s], seam[:, 1:].astype(np.float64))
    x[:, 2] = lo[2] + 60 * (hi[2] - lo[2]) / n[2]
    q = np.einsum("eij,ej->ei", np.linalg.inv(N)[s], x).astype(np.float32)
    steps = rng.integers(-3, 4, q.shape[0])
    for _ in range(3):
        q[:, 2] = np.where(steps > 0, np.nextafter(q[:, 2], np.float32(np.inf)),
                           np.where(steps < 0, np.nextafter(q[:, 2], np.float32(-np.inf)), q[:, 2]))
        steps = steps - np.sign(steps)
    seam[:, 1:] = q
    ev = np.concatenate([ev, seam])
    g = mdn.mdnorm_create_grid(0, lo, hi, n, wl.W, mdn.MDN_ACC_F64)
    assert 8 * g.nbins_total > 120 * 2**20  # above the L2-slab threshold
    mdn.mdnorm_stats(g, 1, read=False)
    mdn.binmd_accumulate(g, wl.UB, wl.ops, torch.from_numpy(ev).cuda())
    st = mdn.mdnorm_stats(g, 0)
    torch.cuda.synchronize()
    bm = mdn.packed_histograms(g).cpu().numpy()[g.nbins_total:2 * g.nbins_total]
    obm = oracle.binmd(oracle.Grid(lo, hi, n), N, ev)
    assert np.array_equal(bm, obm)
    assert st["event_op_pairs"] == ev.shape[0] * len(N)
    assert st["event_op_inside"] == int(obm.sum())
    # pairs on both sides of the seam
    z = obm.reshape(n[2], n[1], n[0]).sum(axis=(1, 2))
    assert z[59] > 1000 and z[60] > 1000


def test_binmd_l2_slabs_host_vs_device(mdn):
    """On a grid above the L2-slab threshold, host events (staging ring, one pass) and device
    events (two L2 slabs) give the same unit-weight histogram, equal to the oracle's."""
    import torch
    wl = synth.make_workload("topaz", nops=24, events_per_run=200_000)
    lo, hi, n = [-6.0, -6.0, -3.0], [6.0, 6.0, 3.0], [400, 400, 120]
    ev = synth.events_for_run(wl, 0)
    N = oracle.binmd_matrices(wl.UB, wl.ops, wl.W)
    out = []
    for src in (ev, torch.from_numpy(ev).cuda()):
        g = mdn.mdnorm_create_grid(0, lo, hi, n, wl.W, mdn.MDN_ACC_F64)
        mdn.binmd_accumulate(g, wl.UB, wl.ops, src)
        torch.cuda.synchronize()
        out.append(mdn.packed_histograms(g).cpu().numpy()[g.nbins_total:2 * g.nbins_total].copy())
        g.close()
    obm = oracle.binmd(oracle.Grid(lo, hi, n), N, ev)
    assert obm.sum() > 100_000
    assert np.array_equal(out[0], obm) and np.array_equal(out[1], obm)
