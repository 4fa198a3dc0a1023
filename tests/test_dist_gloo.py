"""N > 1 host logic on CPU: world_size-2 gloo processes follow the shard plan,
compute their partial histograms (with the oracle standing in for the GPU kernels -- test
only), pack the library's [norm | binmd | err2] layout and make ONE reduce; rank 0 must obtain
the single-process result."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_sc_hahnfgmmshvvs24_b200.dist import plan_shards, reduce_packed, reduce_scatter_packed


def test_plan_covers_everything_once():
    for world in (1, 2, 3, 8):
        # multi-run: run blocks
        runs = sorted(r for k in range(world) for r in plan_shards(world, k, 120, 1000, 10).runs)
        assert runs == list(range(120))
        # single run: interleaved pixels and contiguous event blocks
        pix = sorted(p for k in range(world) for p in range(plan_shards(world, k, 1, 1000, 10).pix_begin,
                                                                   1000, plan_shards(world, k, 1, 1000, 10).pix_stride))
        assert pix == list(range(1000))
        ev = [plan_shards(world, k, 1, 1000, 1001).event_ranges[0] for k in range(world)]
        assert ev[0][0] == 0 and ev[-1][1] == 1001
        assert all(ev[i][1] == ev[i + 1][0] for i in range(world - 1))
    with pytest.raises(ValueError):
        plan_shards(2, 2, 1, 10, 10)


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, out):
    import oracle
    import synth
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    wl = synth.make_workload("tiny", events_per_run=5000)
    wl.ops = synth.hex_6mmm_ops()[:4]
    g = oracle.workload_grid(wl)
    ev = synth.events_for_run(wl, 0)
    p = plan_shards(world, rank, wl.nruns, wl.npix, len(ev))
    M = oracle.mdnorm_matrices(wl.R, wl.UB, wl.ops, wl.W)
    norm = oracle.mdnorm(g, wl.pix_dir, wl.solid, wl.flux_k, wl.flux_F, M, 1.0, wl.k_min, wl.k_max,
                         pix_begin=p.pix_begin, pix_stride=p.pix_stride)
    b, e = p.event_ranges[0]
    bm = oracle.binmd(g, oracle.binmd_matrices(wl.UB, wl.ops, wl.W), ev[b:e])
    # the library's layout: [norm | binmd | err2]; err2 was not accumulated (zeros on every rank,
    # a marker value here to prove that the collective leaves it alone)
    packed = torch.from_numpy(np.concatenate([norm, bm, np.full(g.nbins, 7.0)]))
    reduce_packed(packed, dst=0)
    # with_err: the whole buffer travels
    packed_e = torch.from_numpy(np.concatenate([norm, bm, 0.5 * bm]))
    reduce_packed(packed_e, dst=None, with_err=True)
    if rank == 0:
        full_n, full_b, _ = oracle.run_workload(wl, events={0: ev})
        n = g.nbins
        out.put((np.abs(packed[:n].numpy() - full_n).max() / full_n.max(),
                 float(np.abs(packed[n:2 * n].numpy() - full_b).max()),
                 bool(np.all(packed[2 * n:].numpy() == 7.0)),
                 float(np.abs(packed_e[2 * n:].numpy() - 0.5 * full_b).max())))
    dist.destroy_process_group()


def test_gloo_world2_reduce_matches_single_process():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    rel_n, abs_b, err_untouched, abs_e = q.get(timeout=300)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert rel_n < 1e-14
    assert abs_b == 0.0  # unit weights: integer counts add exactly
    assert err_untouched  # err2 not accumulated -> not sent (2 nbins doubles travel, not 3)
    assert abs_e == 0.0


def _rs_worker(rank, world, port, out):
    """reduce_scatter path (SURVEY.md §8(e), 500^3 stress grid): every rank gets the summed norm
    and binmd of its own bin block; dividing the blocks reproduces the single-process xs."""
    import oracle
    import synth
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    wl = synth.make_workload("tiny", events_per_run=3000)
    wl.nbins = np.array([7, 5, 3])  # 105 bins: not a multiple of the world size (padded blocks)
    g = oracle.workload_grid(wl)
    ev = synth.events_for_run(wl, 0)
    p = plan_shards(world, rank, wl.nruns, wl.npix, len(ev))
    M = oracle.mdnorm_matrices(wl.R, wl.UB, wl.ops, wl.W)
    norm = oracle.mdnorm(g, wl.pix_dir, wl.solid, wl.flux_k, wl.flux_F, M, 1.0, wl.k_min, wl.k_max,
                         pix_begin=p.pix_begin, pix_stride=p.pix_stride)
    b, e = p.event_ranges[0]
    bm = oracle.binmd(g, oracle.binmd_matrices(wl.UB, wl.ops, wl.W), ev[b:e])
    # the library's 3-part layout [norm | binmd | err2], err2 = 0.25 binmd (halves + 1/4: exact)
    packed = torch.from_numpy(np.concatenate([norm, bm, 0.25 * bm]))
    ns, bs, es, (b0, b1) = reduce_scatter_packed(packed, nbins=g.nbins, with_err=True)
    ns2, bs2, (c0, c1) = reduce_scatter_packed(packed, nbins=g.nbins)
    full_n, full_b, full_x = oracle.run_workload(wl, events={0: ev})
    with np.errstate(invalid="ignore", divide="ignore"):
        xs = np.where(ns.numpy() > 0, bs.numpy() / ns.numpy(), np.nan)
    ok = (np.allclose(ns.numpy(), full_n[b0:b1], rtol=1e-14, atol=0) and np.array_equal(bs.numpy(), full_b[b0:b1])
          and np.array_equal(es.numpy(), 0.25 * full_b[b0:b1]) and (c0, c1) == (b0, b1)
          and np.array_equal(ns2.numpy(), ns.numpy()) and np.array_equal(bs2.numpy(), bs.numpy())
          and np.array_equal(np.isnan(xs), np.isnan(full_x[b0:b1]))
          and np.allclose(xs[~np.isnan(xs)], full_x[b0:b1][~np.isnan(xs)], rtol=1e-13))
    out.put((rank, b0, b1, g.nbins, bool(ok)))
    dist.destroy_process_group()


def test_gloo_world2_reduce_scatter_blocks():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_rs_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = sorted(q.get(timeout=300) for _ in range(2))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert all(r[4] for r in res)
    # the two blocks tile [0, nbins) exactly
    assert res[0][1] == 0 and res[0][2] == res[1][1] and res[1][2] == res[0][3]


def test_packed_layout_checks():
    """The collectives take the library's 3-part buffer; a 2-part buffer is refused."""
    import torch
    buf = torch.zeros(10, dtype=torch.float64)
    with pytest.raises(ValueError):
        reduce_packed(buf, nbins=4)
    n, bs, (b0, b1) = reduce_scatter_packed(torch.arange(12, dtype=torch.float64))[0], \
        reduce_scatter_packed(torch.arange(12, dtype=torch.float64))[1], (0, 4)
    assert n.tolist() == [0, 1, 2, 3] and bs.tolist() == [4, 5, 6, 7]
