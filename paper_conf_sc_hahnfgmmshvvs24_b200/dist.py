"""Multi-GPU layer: one process per GPU, shard plan + one collective.

Algorithm 1 gives every MPI rank a block of files (runs), private histograms and one
MPI_Reduce before the divide ("Each process allocates its own histogram, and the MPI reduce
function is used to add histograms").  Here:
  * several runs  -> contiguous run blocks per rank (range(rank, size));
  * a single run  -> pixels interleaved by rank (p = rank, rank + G, ...) so every GPU sees every
    detector region (balances the CORELLI slab, where only ~4% of trajectories hit the grid),
    and that run's events split into contiguous ranges;
  * exchange      -> ONE collective over the packed fp64 [norm | binmd (| err2)] buffer (sum); rank 0
    (or every rank for all_reduce) then divides -- or, for grids too large to gather on one
    GPU (the 500^3 stress grid: 2 GB packed), ONE reduce_scatter that leaves every rank the summed
    norm and binmd of its own contiguous bin block, which it divides locally (mdn_divide).
The plan is pure Python (tested on CPU with gloo); the reduce works on any torch process group
(NCCL over NVLink/NVSwitch on B200s).
"""
from __future__ import annotations

from dataclasses import dataclass, field


@dataclass
class RankPlan:
    rank: int
    world: int
    runs: list = field(default_factory=list)      # run indices this rank processes
    pix_begin: int = 0
    pix_stride: int = 1
    # per run: (event_begin, event_end) of that run's events handled by this rank
    event_ranges: dict = field(default_factory=dict)


def _block(n: int, world: int, rank: int) -> tuple[int, int]:
    """Contiguous block [b, e) of n items for rank (first n % world ranks get one extra)."""
    base, extra = divmod(n, world)
    b = rank * base + min(rank, extra)
    return b, b + base + (1 if rank < extra else 0)


def plan_shards(world: int, rank: int, nruns: int, npix: int, events_per_run) -> RankPlan:
    """Shard plan for `rank` of `world`.  events_per_run: int or list."""
    if not (0 <= rank < world):
        raise ValueError("rank outside [0, world)")
    ev = events_per_run if isinstance(events_per_run, (list, tuple)) else [events_per_run] * nruns
    p = RankPlan(rank=rank, world=world)
    if nruns >= world:
        b, e = _block(nruns, world, rank)
        p.runs = list(range(b, e))
        p.pix_begin, p.pix_stride = 0, 1
        p.event_ranges = {r: (0, int(ev[r])) for r in p.runs}
    else:
        p.runs = list(range(nruns))
        p.pix_begin, p.pix_stride = rank, world
        p.event_ranges = {r: _block(int(ev[r]), world, rank) for r in p.runs}
    if p.pix_begin >= npix:
        p.pix_begin = npix  # empty pixel shard (more ranks than pixels)
    return p


def _halves(packed, nbins: int | None, with_err: bool):
    """The prefix of the packed [norm | binmd | err2] buffer one collective must cover: norm and
    binmd (2 nbins doubles), plus err2 only when the error column was accumulated."""
    n = packed.numel() // 3 if nbins is None else int(nbins)
    if packed.numel() < 3 * n:
        raise ValueError(f"packed buffer holds {packed.numel()} doubles, need 3 * nbins = {3 * n}")
    return n, packed[: (3 if with_err else 2) * n]


def reduce_packed(packed, group=None, dst: int | None = 0, nbins: int | None = None,
                  with_err: bool = False):
    """Sum the library's packed [norm | binmd | err2] histograms (3 * nbins doubles, as
    `packed_histograms` returns them) of all ranks with ONE collective, in place.

    Only [norm | binmd] travels unless with_err (binmd_accumulate_err was used): err2 is
    otherwise all zero.  dst=None -> all_reduce (every rank gets the sum); otherwise reduce to
    rank `dst`.  nbins defaults to numel // 3."""
    import torch.distributed as dist
    n, view = _halves(packed, nbins, with_err)
    if not dist.is_available() or not dist.is_initialized() or dist.get_world_size(group) == 1:
        return packed
    buf = view
    if view.is_cuda and dist.get_backend(group) == "gloo":  # gloo (CPU tests): host staging
        buf = view.cpu()
    if dst is None:
        dist.all_reduce(buf, op=dist.ReduceOp.SUM, group=group)
    else:
        dist.reduce(buf, dst=dst, op=dist.ReduceOp.SUM, group=group)
    if buf is not view:
        view.copy_(buf)
    return packed


def reduce_scatter_packed(packed, group=None, nbins: int | None = None, with_err: bool = False):
    """Sum the library's packed [norm | binmd | err2] histograms of all ranks with ONE
    reduce_scatter; rank r gets bins [b0, b1) (contiguous blocks of ceil(nbins / world)) of norm
    and binmd (and err2 when with_err).

    Returns (norm_shard, binmd_shard, (b0, b1)), or (norm_shard, binmd_shard, err2_shard, (b0, b1))
    when with_err -- views of a new buffer; divide them with mdn_divide.  The bin blocks are laid
    out rank-major ([rank][part][block], zero padded) before the collective so that each rank's
    output is [norm block | binmd block (| err2 block)]."""
    import torch.distributed as dist
    n, _ = _halves(packed, nbins, with_err)
    parts = 3 if with_err else 2
    if not dist.is_available() or not dist.is_initialized() or dist.get_world_size(group) == 1:
        views = tuple(packed[i * n:(i + 1) * n] for i in range(parts))
        return (*views, (0, n))
    world, rank = dist.get_world_size(group), dist.get_rank(group)
    chunk = -(-n // world)
    tmp = packed.new_zeros(parts, world * chunk)
    for i in range(parts):
        tmp[i, :n] = packed[i * n:(i + 1) * n]
    src = tmp.view(parts, world, chunk).transpose(0, 1).contiguous().view(-1)  # [rank][part][block]
    out = packed.new_empty(parts * chunk)
    if dist.get_backend(group) == "gloo":  # gloo (CPU tests) has no reduce_scatter: all_reduce + slice
        buf = src.cpu() if src.is_cuda else src
        dist.all_reduce(buf, op=dist.ReduceOp.SUM, group=group)
        out.copy_(buf.view(world, parts * chunk)[rank])
    else:
        dist.reduce_scatter_tensor(out, src, op=dist.ReduceOp.SUM, group=group)
    b0 = min(n, rank * chunk)
    b1 = min(n, b0 + chunk)
    views = tuple(out[i * chunk: i * chunk + b1 - b0] for i in range(parts))
    return (*views, (b0, b1))
