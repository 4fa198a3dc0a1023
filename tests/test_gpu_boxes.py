"""NEXT #4, hierarchical-box BinMD: events grouped in
MDBoxes of equal event counts with known Q extents.  binmd_accumulate_boxes must give exactly
binmd_accumulate's histogram (unit weights: equal integer counts, i.e. bit-exact event bins) and
the oracle's within 1e-12, for any box size, ragged last boxes, boxes that all miss the grid and
NaN events; binmd_box_bounds must be the true per-box extents."""
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


def _grid(mdn, wl, nbins=None):
    return mdn.mdnorm_create_grid(0, wl.lo, wl.hi, wl.nbins if nbins is None else nbins, wl.W)


def _binmd(mdn, g):
    import torch
    torch.cuda.synchronize()
    n = g.nbins_total
    return mdn.packed_histograms(g)[n:2 * n].cpu().numpy().copy()


def test_box_bounds_are_extents(mdn):
    import torch
    wl = synth.make_workload("corelli", events_per_run=100_003)
    ev = synth.events_for_run(wl, 0)
    ev[5, 1:] = np.nan  # a NaN event does not enter the extents
    g = _grid(mdn, wl)
    for B in (32, 256, 1024):
        b = mdn.binmd_box_bounds(g, torch.from_numpy(ev).cuda(), B).cpu().numpy()
        nb = -(-len(ev) // B)
        assert b.shape == (nb, 6)
        for i in (0, 1, nb // 2, nb - 1):
            q = ev[i * B:(i + 1) * B, 1:]
            q = q[np.isfinite(q).all(axis=1)]
            assert np.array_equal(b[i, :3], q.min(axis=0)) and np.array_equal(b[i, 3:], q.max(axis=0))


@pytest.mark.parametrize("cfg,B", [("corelli", 32), ("corelli", 256), ("corelli", 1024), ("topaz", 256)])
def test_boxes_equal_plain_binmd(mdn, cfg, B):
    import torch
    wl = synth.make_workload(cfg, nops=8 if cfg == "topaz" else None, events_per_run=1_000_003)
    ev = synth.events_for_run(wl, 0, unit_weights=True)
    d = torch.from_numpy(ev).cuda()
    g1, g2 = _grid(mdn, wl), _grid(mdn, wl)
    mdn.binmd_accumulate(g1, wl.UB, wl.ops, d)
    bounds = mdn.binmd_box_bounds(g2, d, B)
    mdn.binmd_accumulate_boxes(g2, wl.UB, wl.ops, d, B, bounds)
    a, b = _binmd(mdn, g1), _binmd(mdn, g2)
    assert np.array_equal(a, b)  # unit weights: integer counts, bit-exact bins
    o = oracle.binmd(oracle.workload_grid(wl), oracle.binmd_matrices(wl.UB, wl.ops, wl.W), ev)
    assert np.array_equal(b, o)
    g1.close()
    g2.close()


def test_boxes_weighted_and_err_free_parity(mdn):
    """Weighted CORELLI events (Bragg weights) through boxes: oracle within 1e-12 per bin."""
    import torch
    wl = synth.make_workload("corelli", events_per_run=2_000_000)
    ev = synth.events_for_run(wl, 0)
    d = torch.from_numpy(ev).cuda()
    g = _grid(mdn, wl)
    bounds = mdn.binmd_box_bounds(g, d, 1024)
    mdn.binmd_accumulate_boxes(g, wl.UB, wl.ops, d, 1024, bounds)
    b = _binmd(mdn, g)
    o = oracle.binmd(oracle.workload_grid(wl), oracle.binmd_matrices(wl.UB, wl.ops, wl.W), ev)
    assert np.array_equal(b == 0, o == 0)
    assert np.all(np.abs(b - o) <= 1e-12 * np.abs(o))
    g.close()


def test_boxes_all_miss_and_edge_cases(mdn):
    import torch
    wl = synth.make_workload("corelli", events_per_run=50_000)
    ev = synth.events_for_run(wl, 0)
    ev[:, 1:] += 1000.0  # every event far outside the grid: every box dropped
    d = torch.from_numpy(ev).cuda()
    g = _grid(mdn, wl)
    bounds = mdn.binmd_box_bounds(g, d, 256)
    mdn.binmd_accumulate_boxes(g, wl.UB, wl.ops, d, 256, bounds)
    assert not _binmd(mdn, g).any()
    with pytest.raises(mdn.MdnError, match="MDN_EINVAL"):
        mdn.binmd_accumulate_boxes(g, wl.UB, wl.ops, d, 100, bounds)  # not a power of two
    with pytest.raises(mdn.MdnError, match="MDN_EINVAL"):
        mdn.binmd_box_bounds(g, d, 16)
    g.close()
