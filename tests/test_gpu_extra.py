"""More GPU parity cases: flux tables off the fast path, work counters, and the N > 1 code path
(two processes sharing one GPU, gloo reduce) -- all through the C ABI against the fp64 oracle."""
import json
import os
import socket
import subprocess
import sys

import numpy as np
import pytest

import oracle
import synth

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def mdn():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    import paper_conf_sc_hahnfgmmshvvs24_b200 as m
    from paper_conf_sc_hahnfgmmshvvs24_b200 import build
    build.build()
    return m


def _hist(mdn, g):
    import torch
    torch.cuda.synchronize()
    t = mdn.packed_histograms(g).cpu().numpy()
    n = g.nbins_total
    return t[:n].copy(), t[n:2 * n].copy()


def _assert_rel(a, b, rel=1e-12):
    assert np.array_equal(a == 0, b == 0)
    assert np.all(np.abs(a - b) <= rel * np.abs(b))


def _weird_flux(n=6000):
    """Non-uniform table larger than the shared-memory limit (4096 knots): a dense cluster of 60
    knots inside one search cell, and knots placed exactly on plane-crossing values."""
    rng = np.random.default_rng(11)
    k = np.sort(np.concatenate([np.linspace(1.0, 12.0, n - 64), 5.0 + 1e-5 * np.arange(1, 61),
                                [2.5, 5.0, 7.5, 3.75]]))
    k = np.unique(k)
    F = np.concatenate([[0.0], np.cumsum(rng.uniform(0.1, 1.0, len(k) - 1))])
    return k, F


@pytest.mark.parametrize("nflux", [6000, 300])
def test_flux_table_paths(mdn, nflux):
    k, F = _weird_flux(nflux)
    wl = synth.make_workload("tiny")
    d = np.concatenate([wl.pix_dir, [[0.0, 0.0, -1.0]]])
    s = np.concatenate([wl.solid, [1.0]])
    lo, hi, n = [-8.0, -8.0, 0.0], [8.0, 8.0, 20.0], [16, 16, 4]
    g = mdn.mdnorm_create_grid(0, lo, hi, n, np.eye(3))
    mdn.mdnorm_set_instrument(g, d, s)
    mdn.mdnorm_set_flux(g, k, F)
    rng = np.random.default_rng(12)
    M = np.concatenate([np.eye(3)[None], rng.normal(size=(7, 3, 3)) * 0.6])
    c = rng.uniform(0.5, 2.0, len(M))
    mdn.mdnorm_accumulate_matrices(g, M, c, 2.0, 9.0)
    norm, _ = _hist(mdn, g)
    og = oracle.Grid(lo, hi, n)
    onorm = oracle.mdnorm(og, d, s, k, F, M, c, 2.0, 9.0)
    assert onorm.sum() > 0
    _assert_rel(norm, onorm)
    ids = np.arange(len(M) * len(s))
    nc, ns, bins, vals = mdn.mdnorm_debug_trajectories(g, M, c, 2.0, 9.0, ids, 256)
    for t in ids:
        m, p = divmod(int(t), len(s))
        onc, ons, ob, ov = oracle.mdnorm_trajectory(og, d[p], s[p], k, F, M[m], c[m], 2.0, 9.0, 256)
        assert (nc[t], ns[t]) == (onc, ons)
        assert np.array_equal(bins[t, :ons], ob) and np.array_equal(vals[t, :ons], ov)


def test_work_counters_match_oracle(mdn):
    wl = synth.make_workload("corelli")
    g = mdn.mdnorm_create_grid(0, wl.lo, wl.hi, wl.nbins, wl.W)
    mdn.mdnorm_set_instrument(g, wl.pix_dir, wl.solid)
    mdn.mdnorm_set_flux(g, wl.flux_k, wl.flux_F)
    mdn.mdnorm_stats(g, 1, read=False)
    stride = 211
    mdn.mdnorm_accumulate(g, wl.UB, wl.R[0], wl.ops, wl.k_min, wl.k_max, 1.0, pix_stride=stride)
    ev = synth.events_for_run(wl, 0, n=100_000)
    import torch
    mdn.binmd_accumulate(g, wl.UB, wl.ops, torch.from_numpy(ev).cuda())
    st = mdn.mdnorm_stats(g, 0)
    og = oracle.workload_grid(wl)
    M = oracle.mdnorm_matrices(wl.R, wl.UB, wl.ops, wl.W)
    pix = np.arange(0, wl.npix, stride)
    hits = segs = cross = 0
    for m in range(len(M)):
        for p in pix:
            if wl.solid[p] == 0:
                continue  # masked pixels are skipped by the kernel (reading #16)
            nc, ns, _, _ = oracle.mdnorm_trajectory(og, wl.pix_dir[p], wl.solid[p], wl.flux_k, wl.flux_F,
                                                    M[m], 1.0, wl.k_min, wl.k_max, 1)
            hits += nc > 0
            cross += max(nc - 2, 0)
            segs += ns
    assert st["trajectories"] == len(pix) * len(M)
    assert st["hit_trajectories"] == hits
    assert st["crossings"] == cross
    assert st["segments"] == segs
    assert st["event_op_pairs"] == len(ev) * len(wl.ops)
    inside = (oracle.binmd_bins(og, oracle.binmd_matrices(wl.UB, wl.ops, wl.W), ev) >= 0).sum()
    assert st["event_op_inside"] == inside


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _dist_worker(rank, world, port, q):
    import torch
    import torch.distributed as dist
    sys.path.insert(0, ROOT)
    import paper_conf_sc_hahnfgmmshvvs24_b200 as m
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    wl = synth.make_workload("corelli", events_per_run=400_000)
    ev = synth.events_for_run(wl, 0)
    plan = m.plan_shards(world, rank, 1, wl.npix, len(ev))
    g = m.mdnorm_create_grid(0, wl.lo, wl.hi, wl.nbins, wl.W)
    m.mdnorm_set_instrument(g, wl.pix_dir, wl.solid)
    m.mdnorm_set_flux(g, wl.flux_k, wl.flux_F)
    m.mdnorm_accumulate(g, wl.UB, wl.R[0], wl.ops, wl.k_min, wl.k_max, 1.0,
                        pix_begin=plan.pix_begin, pix_stride=plan.pix_stride * 13)
    b, e = plan.event_ranges[0]
    m.binmd_accumulate(g, wl.UB, wl.ops, torch.from_numpy(ev[b:e]).cuda())
    packed = m.packed_histograms(g)
    m.reduce_packed(packed, dst=0)
    if rank == 0:
        xs = m.mdnorm_cross_section(g)
        torch.cuda.synchronize()
        q.put((packed.cpu().numpy(), xs))
    dist.barrier()
    g.close()
    dist.destroy_process_group()


def test_two_processes_one_gpu_reduce(mdn):
    """N > 1 path on real kernels: plan_shards + per-rank library histograms + one reduce; the
    pixel stride 2*13 of the two ranks covers every 13th pixel exactly once."""
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_dist_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    packed, xs = q.get(timeout=600)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    wl = synth.make_workload("corelli", events_per_run=400_000)
    ev = synth.events_for_run(wl, 0)
    og = oracle.workload_grid(wl)
    M = oracle.mdnorm_matrices(wl.R, wl.UB, wl.ops, wl.W)
    onorm = oracle.Accumulator(og.nbins)
    for r in range(2):
        oracle.mdnorm(og, wl.pix_dir, wl.solid, wl.flux_k, wl.flux_F, M, 1.0, wl.k_min, wl.k_max,
                      pix_begin=r, pix_stride=26, acc=onorm)
    obm = oracle.binmd(og, oracle.binmd_matrices(wl.UB, wl.ops, wl.W), ev)
    n = og.nbins
    _assert_rel(packed[:n], onorm.value())
    _assert_rel(packed[n:2 * n], obm)
    oxs = oracle.cross_section(obm, onorm.value())
    assert np.array_equal(np.isnan(xs), np.isnan(oxs))


def _rs_dist_worker(rank, world, port, q):
    """reduce_scatter of the library's real 3-part buffer [norm | binmd | err2] (err2 written by
    binmd_accumulate_err), then mdn_divide on each rank's own bin block."""
    import torch
    import torch.distributed as dist
    sys.path.insert(0, ROOT)
    import paper_conf_sc_hahnfgmmshvvs24_b200 as m
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    wl = synth.make_workload("corelli", events_per_run=300_000)
    ev = synth.events_for_run(wl, 0)
    ev8 = np.zeros((len(ev), 8), np.float32)
    ev8[:, 0] = ev[:, 0]
    ev8[:, 1] = 0.5 * ev[:, 0] + 0.25
    ev8[:, 5:8] = ev[:, 1:4]
    nb = [61, 47, 1]  # 2867 bins: not a multiple of the world size (padded blocks)
    plan = m.plan_shards(world, rank, 1, wl.npix, len(ev))
    g = m.mdnorm_create_grid(0, wl.lo, wl.hi, nb, wl.W)
    m.mdnorm_set_privatization(g, m.MDN_PRIV_OFF)
    m.mdnorm_set_instrument(g, wl.pix_dir, wl.solid)
    m.mdnorm_set_flux(g, wl.flux_k, wl.flux_F)
    m.mdnorm_accumulate(g, wl.UB, wl.R[0], wl.ops, wl.k_min, wl.k_max, 1.0,
                        pix_begin=plan.pix_begin, pix_stride=plan.pix_stride * 7)
    b, e = plan.event_ranges[0]
    m.binmd_accumulate_err(g, wl.UB, wl.ops, torch.from_numpy(ev8[b:e]).cuda(), col_w=0, col_e=1, col_q=5)
    packed = m.packed_histograms(g)
    ns, bs, es, (b0, b1) = m.reduce_scatter_packed(packed, nbins=g.nbins_total, with_err=True)
    xs = m.mdn_divide(ns.contiguous(), bs.contiguous())
    torch.cuda.synchronize()
    q.put((rank, b0, b1, ns.cpu().numpy(), bs.cpu().numpy(), es.cpu().numpy(), xs.cpu().numpy()))
    dist.barrier()
    g.close()
    dist.destroy_process_group()


def test_two_processes_reduce_scatter_real_buffer(mdn):
    """The reduce_scatter path (grids too large to gather) on the library's own
    packed [norm | binmd | err2] buffer: every rank's norm, binmd and err2 blocks equal the
    oracle's, and its divided block equals the oracle's xs (NaN masks equal)."""
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_rs_dist_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = sorted(q.get(timeout=600) for _ in range(2))
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    wl = synth.make_workload("corelli", events_per_run=300_000)
    ev = synth.events_for_run(wl, 0)
    ev8 = np.zeros((len(ev), 8), np.float32)
    ev8[:, 0] = ev[:, 0]
    ev8[:, 1] = 0.5 * ev[:, 0] + 0.25
    ev8[:, 5:8] = ev[:, 1:4]
    og = oracle.Grid(wl.lo, wl.hi, [61, 47, 1])
    M = oracle.mdnorm_matrices(wl.R, wl.UB, wl.ops, wl.W)
    onorm = oracle.Accumulator(og.nbins)
    for r in range(2):
        oracle.mdnorm(og, wl.pix_dir, wl.solid, wl.flux_k, wl.flux_F, M, 1.0, wl.k_min, wl.k_max,
                      pix_begin=r, pix_stride=14, acc=onorm)
    N = oracle.binmd_matrices(wl.UB, wl.ops, wl.W)
    obm = oracle.binmd(og, N, ev8, col_w=0, col_q=5)
    oe2 = oracle.binmd_err(og, N, ev8, col_e=1, col_q=5)
    onorm = onorm.value()
    oxs = oracle.cross_section(obm, onorm)
    assert res[0][1] == 0 and res[0][2] == res[1][1] and res[1][2] == og.nbins
    for rank, b0, b1, ns, bs, es, xs in res:
        _assert_rel(ns, onorm[b0:b1])
        _assert_rel(bs, obm[b0:b1])
        _assert_rel(es, oe2[b0:b1])
        assert np.array_equal(np.isnan(xs), np.isnan(oxs[b0:b1]))
        fin = ~np.isnan(xs)
        assert np.all(np.abs(xs[fin] - oxs[b0:b1][fin]) <= 3e-12 * np.abs(oxs[b0:b1][fin]))


def test_bench_multi_rank_code_path():
    """`bench.py --gpus 2` without torchrun launches its own 2 ranks (MDN_BENCH_SHARED_GPU=1: both
    on GPU 0 over gloo): the N > 1 code path runs and rank 0 prints one JSON line with n_gpus = 2
    (a code-path check, not a performance number)."""
    env = dict(os.environ, MDN_BENCH_SHARED_GPU="1")
    env.pop("WORLD_SIZE", None)
    cmd = [sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--steps", "2", "--warmup", "3",
           "--no-cpu-baseline"]
    r = subprocess.run(cmd, env=env, capture_output=True, text=True, timeout=900, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["scaling"] == "weak" and d["value"] > 0
    assert d["config"]["trajectories_per_gpu"] == 372736 * 24


def test_divide_on_bin_shards(mdn):
    """X2 per bin block (the reduce_scatter path of SURVEY.md §8(e)): mdn_divide on each block
    of the summed histograms equals the grid's own cross-section (bit-exact: same IEEE division)
    and the oracle's xs (NaN masks equal)."""
    import torch
    wl = synth.make_workload("tiny")
    g = mdn.mdnorm_create_grid(0, wl.lo, wl.hi, wl.nbins, wl.W)
    mdn.mdnorm_set_instrument(g, wl.pix_dir, wl.solid)
    mdn.mdnorm_set_flux(g, wl.flux_k, wl.flux_F)
    ev = synth.events_for_run(wl, 0)
    mdn.mdnorm_accumulate(g, wl.UB, wl.R[0], wl.ops, wl.k_min, wl.k_max, wl.charge[0])
    mdn.binmd_accumulate(g, wl.UB, wl.ops, torch.from_numpy(ev).cuda())
    n = g.nbins_total
    packed = mdn.packed_histograms(g)
    full = mdn.mdnorm_cross_section(g)
    world = 3
    chunk = -(-n // world)
    parts = []
    for r in range(world):
        b0, b1 = min(n, r * chunk), min(n, (r + 1) * chunk)
        xs = mdn.mdn_divide(packed[b0:b1].contiguous(), packed[n + b0:n + b1].contiguous())
        parts.append(xs.cpu().numpy())
    got = np.concatenate(parts)
    assert np.array_equal(np.isnan(got), np.isnan(full))
    assert np.array_equal(got[~np.isnan(got)], full[~np.isnan(full)])
    _, _, oxs = oracle.run_workload(wl, events={0: ev})
    assert np.array_equal(np.isnan(got), np.isnan(oxs))
    fin = ~np.isnan(oxs)
    assert np.all(np.abs(got[fin] - oxs[fin]) <= 3e-12 * np.abs(oxs[fin]))
    with pytest.raises(ValueError):
        mdn.mdn_divide(packed[:4].cpu(), packed[:4].cpu())
    g.close()


def _nccl_world1_worker(port, q):
    """The X1 collectives over the NCCL backend itself (world size 1: this environment has one
    GPU per call, and NCCL refuses two ranks on one device): reduce, all_reduce and
    reduce_scatter_tensor on the library's own [norm | binmd | err2] device buffer."""
    import torch
    import torch.distributed as dist
    sys.path.insert(0, ROOT)
    import paper_conf_sc_hahnfgmmshvvs24_b200 as m
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.cuda.set_device(0)
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    assert dist.get_backend() == "nccl"
    wl = synth.make_workload("corelli", events_per_run=200_000)
    ev = synth.events_for_run(wl, 0)
    ev8 = np.zeros((len(ev), 8), np.float32)
    ev8[:, 0] = ev[:, 0]
    ev8[:, 1] = 0.5 * ev[:, 0] + 0.25
    ev8[:, 5:8] = ev[:, 1:4]
    g = m.mdnorm_create_grid(0, wl.lo, wl.hi, [61, 47, 1], wl.W)
    m.mdnorm_set_instrument(g, wl.pix_dir, wl.solid)
    m.mdnorm_set_flux(g, wl.flux_k, wl.flux_F)
    m.mdnorm_accumulate(g, wl.UB, wl.R[0], wl.ops, wl.k_min, wl.k_max, 1.0, pix_stride=11)
    m.binmd_accumulate_err(g, wl.UB, wl.ops, torch.from_numpy(ev8).cuda(), col_w=0, col_e=1, col_q=5)
    packed = m.packed_histograms(g)
    n = g.nbins_total
    before = packed.clone()
    m.reduce_packed(packed, dst=0, nbins=n)          # NCCL reduce of [norm | binmd]
    m.reduce_packed(packed, dst=None, nbins=n, with_err=True)  # NCCL all_reduce of all three parts
    ns, bs, es, (b0, b1) = m.reduce_scatter_packed(packed, nbins=n, with_err=True)  # NCCL reduce_scatter
    torch.cuda.synchronize()
    q.put((before.cpu().numpy(), packed.cpu().numpy(), ns.cpu().numpy(), bs.cpu().numpy(), es.cpu().numpy(),
           b0, b1, n))
    g.close()
    dist.destroy_process_group()


def test_nccl_backend_collectives_world1(mdn):
    """dist.py's collectives executed by NCCL on the library's device buffer (a one-rank sum is
    the identity, so every part must come back bit-identical)."""
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    p = ctx.Process(target=_nccl_world1_worker, args=(_free_port(), q))
    p.start()
    before, after, ns, bs, es, b0, b1, n = q.get(timeout=600)
    p.join(timeout=120)
    assert p.exitcode == 0
    assert np.array_equal(before, after)
    assert (b0, b1) == (0, n)
    assert np.array_equal(ns, before[:n]) and np.array_equal(bs, before[n:2 * n]) and np.array_equal(es, before[2 * n:])
    assert before[:n].any() and before[n:2 * n].any() and before[2 * n:].any()
