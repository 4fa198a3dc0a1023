"""Thin Python binding of include/mdnorm.h: same names, argument marshalling only.

Inputs may be numpy arrays (host) or torch tensors (host or CUDA); every computation happens
in libmdnorm.so's CUDA kernels.  Streams default to torch's current stream on the grid's device.
"""
from __future__ import annotations

import ctypes as C

import numpy as np

from . import _native
from ._native import (MDN_ACC_F32, MDN_ACC_F64, MDN_PRIV_AUTO, MDN_PRIV_OFF, MDN_PRIV_ON,  # noqa: F401
                      MdnError, check, load)


def _is_torch(x) -> bool:
    return type(x).__module__.startswith("torch")


def _arg(x, dtype, n=None, name="arg"):
    """(pointer, keepalive) for a host numpy-compatible or torch input of 'dtype'."""
    if x is None:
        return None, None
    if _is_torch(x):
        import torch
        tdt = {np.float64: torch.float64, np.float32: torch.float32, np.int64: torch.int64,
               np.int32: torch.int32}[dtype]
        if x.dtype != tdt or not x.is_contiguous():
            x = x.to(tdt).contiguous()
        if n is not None and x.numel() < n:
            raise ValueError(f"{name}: need {n} elements, got {x.numel()}")
        return x.data_ptr(), x
    a = np.ascontiguousarray(x, dtype=dtype)
    if n is not None and a.size < n:
        raise ValueError(f"{name}: need {n} elements, got {a.size}")
    return a.ctypes.data, a


def _stream(stream, device: int):
    if stream is None:
        import torch
        if torch.cuda.is_available():
            return torch.cuda.current_stream(device).cuda_stream
        return None
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


class Grid:
    """Owner of an mdn_grid* handle (mdnorm_create_grid / mdnorm_destroy)."""

    def __init__(self, handle: int, device: int, nbins):
        self.handle = handle
        self.device = device
        self.nbins = tuple(int(x) for x in nbins)

    @property
    def nbins_total(self) -> int:
        return self.nbins[0] * self.nbins[1] * self.nbins[2]

    def close(self):
        if self.handle:
            check(load().mdnorm_destroy(self.handle), "mdnorm_destroy")
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()


# ------------------------------------------------------------------------------ user entry points


def mdnorm_create_grid(device, lo, hi, nbins, W, acc=MDN_ACC_F64) -> Grid:
    lib = load()
    lo_p, lo_k = _arg(lo, np.float64, 3, "lo")
    hi_p, hi_k = _arg(hi, np.float64, 3, "hi")
    nb_p, nb_k = _arg(nbins, np.int64, 3, "nbins")
    W_p, W_k = _arg(W, np.float64, 9, "W")
    h = C.c_void_p()
    check(lib.mdnorm_create_grid(int(device), lo_p, hi_p, nb_p, W_p, int(acc), C.byref(h)),
          "mdnorm_create_grid")
    return Grid(h.value, int(device), np.asarray(nbins).ravel())


def mdnorm_destroy(g: Grid) -> None:
    g.close()


def mdnorm_set_instrument(g: Grid, dir, solid) -> None:
    n = len(solid)
    d_p, d_k = _arg(dir, np.float64, 3 * n, "dir")
    s_p, s_k = _arg(solid, np.float64, n, "solid")
    check(load().mdnorm_set_instrument(g.handle, n, d_p, s_p), "mdnorm_set_instrument")


def mdnorm_set_flux(g: Grid, k, F) -> None:
    n = len(k)
    k_p, k_k = _arg(k, np.float64, n, "k")
    F_p, F_k = _arg(F, np.float64, n, "F")
    check(load().mdnorm_set_flux(g.handle, n, k_p, F_p), "mdnorm_set_flux")


def mdnorm_accumulate(g: Grid, UB, R, ops, k_min, k_max, proton_charge, pix_begin=0, pix_end=-1,
                      pix_stride=1, stream=None) -> None:
    ops = np.ascontiguousarray(ops, dtype=np.float64).reshape(-1, 9)
    UB_p, UB_k = _arg(UB, np.float64, 9, "UB")
    R_p, R_k = _arg(R, np.float64, 9, "R")
    check(load().mdnorm_accumulate(
        g.handle, UB_p, R_p, len(ops), ops.ctypes.data,
        float(k_min), float(k_max), float(proton_charge), int(pix_begin), int(pix_end),
        int(pix_stride), _stream(stream, g.device)), "mdnorm_accumulate")


def mdnorm_accumulate_runs(g: Grid, UB, R, charge, ops, k_min, k_max, pix_begin=0, pix_end=-1,
                           pix_stride=1, stream=None) -> None:
    R = np.ascontiguousarray(R, dtype=np.float64).reshape(-1, 9)
    charge = np.ascontiguousarray(charge, dtype=np.float64).reshape(-1)
    ops = np.ascontiguousarray(ops, dtype=np.float64).reshape(-1, 9)
    if len(charge) != len(R):
        raise ValueError("one charge per run")
    UB_p, UB_k = _arg(UB, np.float64, 9)
    check(load().mdnorm_accumulate_runs(
        g.handle, UB_p, len(R), R.ctypes.data, charge.ctypes.data, len(ops), ops.ctypes.data,
        float(k_min), float(k_max), int(pix_begin), int(pix_end), int(pix_stride),
        _stream(stream, g.device)), "mdnorm_accumulate_runs")


def _event_layout(events, stride_floats):
    shape = tuple(events.shape)
    if stride_floats is None:
        stride_floats = shape[1] if len(shape) == 2 else 4
    n = (shape[0] if len(shape) == 2 else int(np.prod(shape)) // stride_floats)
    return n, stride_floats


def binmd_accumulate(g: Grid, UB, ops, events, stride_floats=None, col_w=0, col_q=1,
                     stream=None, nevents=None) -> None:
    """events: [n, stride] float32 (numpy/torch, host or CUDA)."""
    n, stride_floats = _event_layout(events, stride_floats)
    n = n if nevents is None else int(nevents)
    ops = np.ascontiguousarray(ops, dtype=np.float64).reshape(-1, 9)
    ev_p, ev_k = _arg(events, np.float32, n * stride_floats, "events")
    UB_p, UB_k = _arg(UB, np.float64, 9)
    check(load().binmd_accumulate(g.handle, UB_p, len(ops), ops.ctypes.data, n, ev_p,
                                  int(stride_floats), int(col_w), int(col_q),
                                  _stream(stream, g.device)), "binmd_accumulate")


def binmd_accumulate_err(g: Grid, UB, ops, events, stride_floats=None, col_w=0, col_e=1, col_q=5,
                         stream=None) -> None:
    """BinMD plus the error-squared column (8-column rows: signal 0, error^2 1, Q 5-7)."""
    n, stride_floats = _event_layout(events, stride_floats)
    ops = np.ascontiguousarray(ops, dtype=np.float64).reshape(-1, 9)
    ev_p, ev_k = _arg(events, np.float32, n * stride_floats, "events")
    UB_p, UB_k = _arg(UB, np.float64, 9)
    check(load().binmd_accumulate_err(g.handle, UB_p, len(ops), ops.ctypes.data, n, ev_p,
                                      int(stride_floats), int(col_w), int(col_e), int(col_q),
                                      _stream(stream, g.device)), "binmd_accumulate_err")


def mdnorm_set_flux_tables(g: Grid, tables, pixel_table=None) -> None:
    """Per-bank flux tables: tables = [(k, F), ...]; pixel_table[p] = table index of pixel p."""
    k = np.ascontiguousarray(np.concatenate([np.asarray(t[0], dtype=np.float64) for t in tables]))
    F = np.ascontiguousarray(np.concatenate([np.asarray(t[1], dtype=np.float64) for t in tables]))
    offs = np.ascontiguousarray(np.concatenate([[0], np.cumsum([len(t[0]) for t in tables])]), dtype=np.int64)
    pt_p, pt_k = _arg(pixel_table, np.int32) if pixel_table is not None else (None, None)
    npix = 0 if pixel_table is None else len(pixel_table)
    check(load().mdnorm_set_flux_tables(g.handle, len(tables), offs.ctypes.data, k.ctypes.data, F.ctypes.data,
                                        npix, pt_p), "mdnorm_set_flux_tables")


def mdnorm_set_pixel_krange(g: Grid, kmin, kmax) -> None:
    """Per-pixel momentum limits (None, None removes them)."""
    if kmin is None and kmax is None:
        check(load().mdnorm_set_pixel_krange(g.handle, 0, None, None), "mdnorm_set_pixel_krange")
        return
    n = len(kmin)
    lo_p, lo_k = _arg(kmin, np.float64, n, "kmin")
    hi_p, hi_k = _arg(kmax, np.float64, n, "kmax")
    check(load().mdnorm_set_pixel_krange(g.handle, n, lo_p, hi_p), "mdnorm_set_pixel_krange")


def mdnorm_error_histogram(g: Grid) -> int:
    """Borrowed device pointer of the error-squared histogram."""
    p = C.c_void_p()
    check(load().mdnorm_error_histogram(g.handle, C.byref(p)), "mdnorm_error_histogram")
    return p.value


def mdnorm_cross_section_err(g: Grid, xs=None, xs_err=None, stream=None):
    """(xs, xs_err) as host numpy arrays (allocated if None) or CUDA tensors."""
    if xs is None:
        xs = np.empty(g.nbins_total, dtype=np.float64)
    if xs_err is None:
        xs_err = np.empty(g.nbins_total, dtype=np.float64)
    a_p, _ = _arg(xs, np.float64, g.nbins_total, "xs")
    b_p, _ = _arg(xs_err, np.float64, g.nbins_total, "xs_err")
    check(load().mdnorm_cross_section_err(g.handle, a_p, b_p, _stream(stream, g.device)),
          "mdnorm_cross_section_err")
    return xs, xs_err


def mdnorm_histograms(g: Grid):
    """(norm_ptr, binmd_ptr, nbins_total) -- borrowed device pointers."""
    a, b, n = C.c_void_p(), C.c_void_p(), C.c_int64()
    check(load().mdnorm_histograms(g.handle, C.byref(a), C.byref(b), C.byref(n)), "mdnorm_histograms")
    return a.value, b.value, n.value


def mdnorm_cross_section(g: Grid, xs=None, stream=None):
    """Writes xs (host numpy or CUDA tensor); allocates a host array if xs is None."""
    if xs is None:
        xs = np.empty(g.nbins_total, dtype=np.float64)
    xs_p, _ = _arg(xs, np.float64, g.nbins_total, "xs")
    if not _is_torch(xs) and xs_p != xs.ctypes.data:
        raise ValueError("xs must be a contiguous float64 array")
    check(load().mdnorm_cross_section(g.handle, xs_p, _stream(stream, g.device)), "mdnorm_cross_section")
    return xs


def mdn_divide(norm, binmd, xs=None, stream=None):
    """X2 on device tensors (a bin shard after a reduce_scatter): xs = binmd / norm, NaN where
    norm == 0.  norm, binmd (and xs, allocated if None) are contiguous float64 CUDA tensors."""
    import torch
    for name, t in (("norm", norm), ("binmd", binmd)):
        if not (_is_torch(t) and t.is_cuda and t.dtype == torch.float64 and t.is_contiguous()):
            raise ValueError(f"{name} must be a contiguous float64 CUDA tensor")
    n = norm.numel()
    if binmd.numel() != n:
        raise ValueError("norm and binmd differ in length")
    if xs is None:
        xs = torch.empty_like(norm)
    dev = norm.device.index or 0
    check(load().mdn_divide(dev, norm.data_ptr(), binmd.data_ptr(), xs.data_ptr(), n, _stream(stream, dev)),
          "mdn_divide")
    return xs


def mdnorm_reset(g: Grid, stream=None) -> None:
    check(load().mdnorm_reset(g.handle, _stream(stream, g.device)), "mdnorm_reset")


STAT_NAMES = ("trajectories", "hit_trajectories", "crossings", "segments", "event_op_pairs",
              "event_op_inside")


def mdnorm_stats(g: Grid, enable: int = -1, read: bool = True):
    """Toggle work counters (enable 1/0, -1 = unchanged); returns a dict of counts if read."""
    out = np.zeros(6, np.int64)
    check(load().mdnorm_stats(g.handle, int(enable), out.ctypes.data if read else None), "mdnorm_stats")
    return dict(zip(STAT_NAMES, (int(x) for x in out))) if read else None


def mdnorm_set_privatization(g: Grid, mode: int) -> None:
    """Shared-memory privatised histograms: MDN_PRIV_AUTO (-1), MDN_PRIV_OFF (0), MDN_PRIV_ON (1)."""
    check(load().mdnorm_set_privatization(g.handle, int(mode)), "mdnorm_set_privatization")


PATH_NAMES = {0: "global", 1: "smem_f64", 2: "smem_f32"}


def mdnorm_accumulation_paths(g: Grid) -> tuple[str, str]:
    """Accumulation path of the last (MDNorm, BinMD) launch: 'global', 'smem_f64' or 'smem_f32'."""
    out = np.zeros(2, np.int32)
    check(load().mdnorm_accumulation_paths(g.handle, out.ctypes.data), "mdnorm_accumulation_paths")
    return PATH_NAMES[int(out[0])], PATH_NAMES[int(out[1])]


def mdn_last_error() -> str:
    return load().mdn_last_error().decode(errors="replace")


def mdn_version() -> str:
    return load().mdn_version().decode()


# ------------------------------------------------------------------------------ torch views


class _CudaArray:
    def __init__(self, ptr: int, n: int):
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": "<f8", "data": (ptr, False),
                                         "version": 3, "strides": None, "stream": None}


def packed_histograms(g: Grid):
    """torch float64 CUDA view of the library-owned packed [norm | binmd | err2] buffer
    (3*nbins), valid while g lives -- the buffer one collective reduces."""
    import torch
    a, _, n = mdnorm_histograms(g)
    return torch.as_tensor(_CudaArray(a, 3 * n), device=f"cuda:{g.device}")


# ------------------------------------------------------------------------------ parity entry points


def mdnorm_accumulate_matrices(g: Grid, M, charge, k_min, k_max, pix_begin=0, pix_end=-1,
                               pix_stride=1, stream=None) -> None:
    M = np.ascontiguousarray(M, dtype=np.float64).reshape(-1, 9)
    c = np.ascontiguousarray(np.broadcast_to(np.asarray(charge, dtype=np.float64), (len(M),)))
    check(load().mdnorm_accumulate_matrices(g.handle, len(M), M.ctypes.data, c.ctypes.data,
                                            float(k_min), float(k_max), int(pix_begin),
                                            int(pix_end), int(pix_stride),
                                            _stream(stream, g.device)), "mdnorm_accumulate_matrices")


def binmd_accumulate_matrices(g: Grid, N, events, stride_floats=None, col_w=0, col_q=1,
                              stream=None) -> None:
    n, stride_floats = _event_layout(events, stride_floats)
    N = np.ascontiguousarray(N, dtype=np.float64).reshape(-1, 9)
    ev_p, ev_k = _arg(events, np.float32, n * stride_floats, "events")
    check(load().binmd_accumulate_matrices(g.handle, len(N), N.ctypes.data, n, ev_p,
                                           int(stride_floats), int(col_w), int(col_q),
                                           _stream(stream, g.device)), "binmd_accumulate_matrices")


def mdnorm_debug_trajectories(g: Grid, M, charge, k_min, k_max, traj_ids, max_segs=1024):
    """-> (n_cross[int32], n_seg[int32], seg_bins[ntraj, max_segs], seg_vals[ntraj, max_segs])"""
    M = np.ascontiguousarray(M, dtype=np.float64).reshape(-1, 9)
    c = np.ascontiguousarray(np.broadcast_to(np.asarray(charge, dtype=np.float64), (len(M),)))
    ids = np.ascontiguousarray(traj_ids, dtype=np.int64)
    nt = len(ids)
    nc = np.zeros(nt, np.int32)
    ns = np.zeros(nt, np.int32)
    bins = np.full((nt, max_segs), -1, np.int64)
    vals = np.zeros((nt, max_segs), np.float64)
    check(load().mdnorm_debug_trajectories(g.handle, len(M), M.ctypes.data, c.ctypes.data,
                                           float(k_min), float(k_max), nt, ids.ctypes.data,
                                           nc.ctypes.data, ns.ctypes.data, bins.ctypes.data,
                                           vals.ctypes.data, int(max_segs)),
          "mdnorm_debug_trajectories")
    return nc, ns, bins, vals


def binmd_debug_bins(g: Grid, N, events, stride_floats=None, col_w=0, col_q=1):
    n, stride_floats = _event_layout(events, stride_floats)
    N = np.ascontiguousarray(N, dtype=np.float64).reshape(-1, 9)
    ev_p, ev_k = _arg(events, np.float32, n * stride_floats, "events")
    out = np.empty((len(N), n), np.int64)
    check(load().binmd_debug_bins(g.handle, len(N), N.ctypes.data, n, ev_p, int(stride_floats),
                                  int(col_w), int(col_q), out.ctypes.data), "binmd_debug_bins")
    return out


def mdnorm_debug_compose(g: Grid, UB, R, ops):
    R = np.ascontiguousarray(R, dtype=np.float64).reshape(-1, 9)
    ops = np.ascontiguousarray(ops, dtype=np.float64).reshape(-1, 9)
    M = np.empty((len(R) * len(ops), 9))
    N = np.empty((len(ops), 9))
    UB_p, UB_k = _arg(UB, np.float64, 9)
    check(load().mdnorm_debug_compose(g.handle, UB_p, len(R), R.ctypes.data, len(ops),
                                      ops.ctypes.data, M.ctypes.data, N.ctypes.data),
          "mdnorm_debug_compose")
    return M.reshape(-1, 3, 3), N.reshape(-1, 3, 3)


def mdnorm_debug_set_max_slab(g: Grid, max_traj: int) -> None:
    """Trajectories per cull/walk slab of later MDNorm calls (0 = default 2^27)."""
    check(load().mdnorm_debug_set_max_slab(g.handle, int(max_traj)), "mdnorm_debug_set_max_slab")


def mdnorm_debug_last_launch(g: Grid) -> dict:
    """{slabs, hitters (last slab), big_claim_threshold, slab_limit} of the last MDNorm call."""
    out = np.zeros(4, np.int64)
    check(load().mdnorm_debug_last_launch(g.handle, out.ctypes.data), "mdnorm_debug_last_launch")
    return dict(zip(("slabs", "hitters", "big_claim_threshold", "slab_limit"), (int(x) for x in out)))


def mdnorm_debug_flux_guess(g: Grid, table: int = 0) -> dict:
    """{mode, hit}: the flux interval guess chosen for a table (0 none, 1 uniform in k, 2 in 1/k)."""
    out = np.zeros(2, np.float64)
    check(load().mdnorm_debug_flux_guess(g.handle, int(table), out.ctypes.data), "mdnorm_debug_flux_guess")
    return {"mode": int(out[0]), "hit": float(out[1])}


def binmd_box_bounds(g: Grid, events, box_events=1024, bounds=None, stream=None):
    """MDBox extents (NEXT #4) of packed float4 CUDA events: a CUDA float32 tensor [nboxes, 6]
    (allocated if None) of (min Qx, Qy, Qz, max Qx, Qy, Qz) per box of box_events events."""
    import torch
    if not (_is_torch(events) and events.is_cuda and events.dtype == torch.float32 and events.is_contiguous()):
        raise ValueError("events must be a contiguous float32 CUDA tensor [n, 4]")
    n = events.numel() // 4
    nboxes = -(-n // int(box_events))
    if bounds is None:
        bounds = torch.empty((nboxes, 6), dtype=torch.float32, device=events.device)
    check(load().binmd_box_bounds(g.handle, n, events.data_ptr(), int(box_events), bounds.data_ptr(),
                                  _stream(stream, g.device)), "binmd_box_bounds")
    return bounds


def binmd_accumulate_boxes(g: Grid, UB, ops, events, box_events, bounds, stream=None) -> None:
    """BinMD over MDBoxes with known extents: boxes that cannot reach the grid are not read."""
    ops = np.ascontiguousarray(ops, dtype=np.float64).reshape(-1, 9)
    n = events.numel() // 4
    UB_p, UB_k = _arg(UB, np.float64, 9)
    check(load().binmd_accumulate_boxes(g.handle, UB_p, len(ops), ops.ctypes.data, n, events.data_ptr(),
                                        int(box_events), bounds.data_ptr(), _stream(stream, g.device)),
          "binmd_accumulate_boxes")
