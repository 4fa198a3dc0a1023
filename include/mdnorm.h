/*
 * mdnorm.h -- C ABI of the B200-native MDNorm + BinMD cross-section hot path.
 *
 * Library: paper_conf_sc_hahnfgmmshvvs24_b200/libmdnorm.so (CUDA, sm_100a).  Every entry point is
 * extern "C", takes plain pointers and sizes, and returns an mdn_status (MDN_OK == 0); on any
 * other status mdn_last_error() holds a message for the calling thread.
 *
 * The operation (PAPER.md = "P:"; the hot path of Algorithm 1):
 *   norm[b]  += c_r * Omega_p * integral_{k_min}^{k_max} 1[k * v_{r,s,p} in b] dF(k)     (MDNorm,
 *               Listing 1: plane intersections, sort, linear_interpolation of the
 *               integrated flux, append_to_histogram)
 *   binmd[b] += w_e * 1[N_s * Q_e in b]                                                    (BinMD,
 *               Listings 2-3 P:126-158: transform each event by each op, push its weight)
 *   xs[b]     = binmd[b] / norm[b]   ("sum of all histograms over the sum of all
 *               normalizations"; NaN where norm[b] == 0)
 * with v_{r,s,p} = M_{r,s} (z - d_p), M_{r,s} = (R_r UB S_s W)^-1 / (2 pi), N_s = (UB S_s W)^-1 /
 * (2 pi) (DESIGN.md §3 readings #1-#2).  k is |k_i| = |k_f| in 1/Angstrom; the beam is +z.
 *
 * Grid: nbins[a] uniform half-open bins on [lo[a], hi[a]) per axis a, linear bin index
 * b = i0 + n0 * (i1 + n1 * i2) (first axis fastest).  A segment of a trajectory belongs to the
 * bin of its midpoint (reading #8); segments of zero length are skipped (reading #7).
 *
 * Conventions
 *  - Matrices are row-major double[9].  W's COLUMNS are the projection vectors in HKL
 *    (e.g. CORELLI [H,H,0],[H,-H,0],[0,0,L]).  ops are integer-valued HKL-space symmetry
 *    matrices S_s (at most MDN_MAX_OPS per call).
 *  - Ownership: the caller owns every input.  set_* calls copy their (host or device) inputs
 *    into library-owned device memory and may be freed on return.  The histograms are
 *    library-owned; mdnorm_histograms() returns borrowed device pointers valid until
 *    mdnorm_destroy().  The grid owns ONE packed fp64 buffer [norm | binmd | err2] of
 *    3 * nbins_total doubles: binmd_dev == norm_dev + nbins_total and err2_dev == binmd_dev +
 *    nbins_total always, so one collective covers all of them.
 *  - Streams: 'stream' is a cudaStream_t (NULL = legacy default stream).  Work is enqueued
 *    stream-ordered; only calls that write to a HOST pointer synchronise.  All calls on one grid
 *    must be issued on one stream, or be ordered by the caller.
 *  - Host or device: 'events' and 'xs' may be host or device pointers (detected with
 *    cudaPointerGetAttributes).  Host events are streamed to the GPU in chunks (pinned host
 *    memory makes the copy asynchronous and overlapped with the scatter).
 *  - Errors: arguments are validated before any side effect, so a failed call changes nothing.
 *    MDN_EINVAL: bad argument (lo >= hi, nbins < 1, non-finite values, k not strictly
 *    increasing, F decreasing, singular UB/R/W composition, nops outside [1, MDN_MAX_OPS],
 *    k_min >= k_max or k_min <= 0, negative charge or solid angle, bad shard or column
 *    arguments).  MDN_ESTATE: accumulate before set_instrument / set_flux.  MDN_ENOMEM: device
 *    allocation failed.  MDN_ECUDA: any other CUDA error (message from cudaGetErrorString).
 *  - Precision: geometry (matrices, clip, crossings, midpoints, bin indices, flux
 *    interpolation) is IEEE fp64 without FMA contraction, so crossing counts and bin indices are
 *    bit-identical to the fp64 oracle.  Global histograms are fp64.  mdn_acc selects the
 *    precision of the privatised partial sums (mdnorm_set_privatization): MDN_ACC_F64 = fp64
 *    end to end; MDN_ACC_F32 = fp32 shared-memory partials folded into the fp64 histogram
 *    (BASELINE north_star fp32 mode: 1e-5 relative per bin).  Launches that accumulate
 *    straight into the global histogram (grids larger than shared memory) are fp64 in both
 *    modes.
 */
#ifndef MDNORM_H
#define MDNORM_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define MDN_MAX_OPS 48        /* largest crystallographic point group (m-3m), "~6 and 24" */
#define MDN_MAX_MATS 64       /* matrices per *_matrices / debug call                          */

typedef struct mdn_grid mdn_grid; /* opaque: one grid + histograms + instrument + flux, one GPU */

typedef enum { MDN_OK = 0, MDN_EINVAL = 1, MDN_ENOMEM = 2, MDN_ECUDA = 3, MDN_ESTATE = 4 } mdn_status;
typedef enum { MDN_ACC_F32 = 0, MDN_ACC_F64 = 1 } mdn_acc;

/* Create a grid on CUDA device 'device' (P:177-178 bin counts and projections).
 * lo, hi: double[3] extents in projection coordinates; nbins: int64[3] >= 1; W: double[9];
 * *out receives the handle.  Histograms start at zero. */
mdn_status mdnorm_create_grid(int device, const double lo[3], const double hi[3],
                              const int64_t nbins[3], const double W[9], mdn_acc acc,
                              mdn_grid **out);

/* Free every device and host resource of g (synchronises the device).  NULL is a no-op. */
mdn_status mdnorm_destroy(mdn_grid *g);

/* Detector table ("CORELLI 372K and TOPAZ 1.6M"; VanadiumFile P:428).
 * dir: double[npix][3] unit vectors sample->pixel, lab frame, beam = +z (host or device; any
 * finite vectors are accepted and used as given, q_p = z - d_p);
 * solid: double[npix] solid angle x vanadium factor, >= 0, 0 == masked pixel. */
mdn_status mdnorm_set_instrument(mdn_grid *g, int64_t npix, const double *dir, const double *solid);

/* Per-pixel momentum limits (Mantid's MDNorm_low/high): pixel p's
 * trajectory then runs over [max(k_min, kmin[p]), min(k_max, kmax[p])] in every later
 * mdnorm_accumulate*.  kmin, kmax: double[npix] (host or device), npix must equal the
 * instrument's; kmin == kmax == NULL removes the limits.  set_instrument also removes them. */
mdn_status mdnorm_set_pixel_krange(mdn_grid *g, int64_t npix, const double *kmin, const double *kmax);

/* Integrated (cumulative) flux table F(k) (FluxFile; linear_interpolation):
 * k: double[n] strictly increasing, 1/Angstrom; F: double[n] non-decreasing; n >= 2.
 * F is clamped to F[0] below k[0] and to F[n-1] above k[n-1]. */
mdn_status mdnorm_set_flux(mdn_grid *g, int64_t n, const double *k, const double *F);

/* Per-bank flux tables: ntables cumulative-flux tables concatenated in
 * k/F (host or device), table t = [offsets[t], offsets[t+1]) (offsets: int64[ntables+1], host,
 * offsets[0] == 0, every table >= 2 knots with the rules of mdnorm_set_flux), and pixel_table:
 * int32[npix] (host or device) giving each pixel's table (required when ntables > 1; npix must
 * equal the instrument's).  Replaces any earlier flux; a later set_instrument drops a pixel map
 * (the tables must then be set again).  mdnorm_set_flux(n, k, F) == one table, no map. */
mdn_status mdnorm_set_flux_tables(mdn_grid *g, int32_t ntables, const int64_t *offsets, const double *k,
                                  const double *F, int64_t npix, const int32_t *pixel_table);

/* MDNorm of one run (Algorithm 1 line "mdnorm += MDNorm"): all nops symmetry ops
 * (ops: double[nops][9], host) x pixels p = pix_begin, pix_begin + pix_stride, ... < pix_end
 * (the shard; pix_end = -1 means npix).  UB, R: double[9] host (R = goniometer rotation of the
 * run, "rotations" P:80); proton_charge = c_r ("charge" P:80) >= 0; 0 < k_min < k_max. */
mdn_status mdnorm_accumulate(mdn_grid *g, const double UB[9], const double R[9], int32_t nops,
                             const double *ops, double k_min, double k_max, double proton_charge,
                             int64_t pix_begin, int64_t pix_end, int64_t pix_stride, void *stream);

/* Batched form for a rotation scan: nruns runs (R: double[nruns][9], charge: double[nruns],
 * host) in as few launches as possible; same result as nruns mdnorm_accumulate calls. */
mdn_status mdnorm_accumulate_runs(mdn_grid *g, const double UB[9], int32_t nruns, const double *R,
                                  const double *charge, int32_t nops, const double *ops,
                                  double k_min, double k_max, int64_t pix_begin, int64_t pix_end,
                                  int64_t pix_stride, void *stream);

/* BinMD of one run's events (Algorithm 1 "binmd += BinMD(events)"; Listing 3).
 * events: float[nevents * stride_floats] (host or device; device pointers are borrowed until the
 * stream reaches the work), event e has weight events[e*stride + col_w] (column 1 of the
 * paper's 8-column array) and Q_sample = events[e*stride + col_q + 0..2] (columns 6-8,
 * P:149-150).  Fast path: stride 4, col_w 0, col_q 1 (packed float4 (w, Qx, Qy, Qz)).
 * Grids whose fp64 histogram exceeds what the L2 holds (> 120 MB) are binned from device events
 * in L2-sized slabs of the last axis, one kernel pass each (the events are read once per slab;
 * the result is the same); host events are binned in one pass. */
mdn_status binmd_accumulate(mdn_grid *g, const double UB[9], int32_t nops, const double *ops,
                            int64_t nevents, const float *events, int64_t stride_floats,
                            int32_t col_w, int32_t col_q, void *stream);

/* BinMD that also accumulates the error-squared column (Mantid MDEvent signal + error^2; the
 * paper's 8-column rows): err2[b] += events[e*stride + col_e] for every (op, event)
 * inside the grid, besides binmd[b] += weight.  col_e = -1 is plain binmd_accumulate. */
mdn_status binmd_accumulate_err(mdn_grid *g, const double UB[9], int32_t nops, const double *ops,
                                int64_t nevents, const float *events, int64_t stride_floats,
                                int32_t col_w, int32_t col_e, int32_t col_q, void *stream);

/* MDBox extents ("Mantid's BinMD uses a hierarchy of boxes with equal numbers
 * of events"; the SaveMD files the workflow reads store them): events (DEVICE,
 * packed float4 (w, Qx, Qy, Qz), 16-byte aligned) are cut into boxes of box_events consecutive
 * events (a power of two >= 32; the last box may be shorter) and bounds (DEVICE float[6 * nboxes],
 * nboxes = ceil(nevents / box_events)) receives each box's (min Qx, min Qy, min Qz, max Qx, max Qy,
 * max Qz) over its events with finite Q.  One pass over the events, stream-ordered; the extents
 * belong to the event list and serve every later binmd_accumulate_boxes of it. */
mdn_status binmd_box_bounds(mdn_grid *g, int64_t nevents, const float *events, int32_t box_events,
                            float *bounds, void *stream);

/* BinMD of one run's events grouped in MDBoxes with known extents (binmd_box_bounds, or the file's
 * own): a box whose extent cannot reach the grid under any op (fp64 interval arithmetic on the
 * extent, widened far beyond rounding) is not read at all; the events of the other boxes take the
 * binmd_accumulate path.  The result equals binmd_accumulate's on the same events provided every
 * event's Q lies inside its box's bounds (the caller's contract).  events, bounds: DEVICE
 * (borrowed until the stream reaches the work); packed float4 layout only. */
mdn_status binmd_accumulate_boxes(mdn_grid *g, const double UB[9], int32_t nops, const double *ops,
                                  int64_t nevents, const float *events, int32_t box_events,
                                  const float *bounds, void *stream);

/* Borrowed device pointers to the fp64 histograms (each nbins_total doubles). */
mdn_status mdnorm_histograms(mdn_grid *g, void **norm_dev, void **binmd_dev, int64_t *nbins_total);

/* Borrowed device pointer to the error-squared histogram (== binmd_dev + nbins_total). */
mdn_status mdnorm_error_histogram(mdn_grid *g, void **err2_dev);

/* xs[b] = binmd[b] / norm[b] (NaN where norm[b] == 0) into xs (double[nbins_total], host or
 * device).  A host xs synchronises the stream before returning. */
mdn_status mdnorm_cross_section(mdn_grid *g, double *xs, void *stream);

/* Cross-section and its error: xs as above and xs_err[b] = sqrt(err2[b]) / norm[b] (the
 * normalization is computed, so it carries no error; NaN where norm[b] == 0).  xs and xs_err
 * are both host or both device arrays of nbins_total doubles. */
mdn_status mdnorm_cross_section_err(mdn_grid *g, double *xs, double *xs_err, void *stream);

/* X2 on a bin shard (after a reduce_scatter of the histograms each GPU divides
 * its own bins; "the sum of all histograms over the sum of all normalizations", P:72, P:84,
 * P:100): xs[b] = binmd[b] / norm[b] for b in [0, n), NaN where norm[b] == 0 (reading #12).
 * norm, binmd and xs are DEVICE arrays of n doubles on `device` (caller-owned; xs may alias
 * neither input); stream-ordered on `stream`.  MDN_EINVAL for n < 0, NULL or host pointers. */
mdn_status mdn_divide(int device, const double *norm, const double *binmd, double *xs, int64_t n,
                      void *stream);

/* Zero all histograms (stream-ordered) and start an accumulation epoch: host events passed to
 * later binmd_accumulate* calls are copied to the device only after the stream reaches this
 * point (the copies still overlap the MDNorm kernels enqueued after it). */
mdn_status mdnorm_reset(mdn_grid *g, void *stream);

/* Work counters (tracing).  enable = 1 turns counting on for later kernels, 0 turns it off,
 * -1 leaves it unchanged (counting costs one warp-aggregated atomic per warp per launch).
 * out (HOST int64[6], may be NULL) receives the counts accumulated since the last mdnorm_reset:
 * {trajectories (pixel x op x run, masked pixels included), trajectories that hit the grid,
 *  plane crossings kept (M3), segments appended (M7), (event, op) pairs (B2),
 *  (event, op) pairs inside the grid (B3)}.  Synchronises the device when out != NULL. */
mdn_status mdnorm_stats(mdn_grid *g, int enable, int64_t out[6]);

/* Shared-memory privatisation of the histograms (BASELINE north_star "shared-memory privatised
 * sub-histograms ... falling back to global red.add when the grid exceeds shared memory";
 * S§2.8 G2/G3).  Each CTA accumulates into its own copy of the grid in shared memory (fp64, or
 * fp32 with MDN_ACC_F32) and folds it into the global fp64 histogram with one red.add per
 * touched bin when it finishes.  mode: -1 = auto (default: privatise when the grid fits and the
 * launch has more work units than the flush touches bins), 0 = never (always global red.add),
 * 1 = whenever the grid fits.  Grids that do not fit always use global red.add.  Takes effect
 * for later accumulate calls; no device work.  MDN_EINVAL: NULL grid or mode outside [-1, 1]. */
mdn_status mdnorm_set_privatization(mdn_grid *g, int32_t mode);

/* Accumulation path taken by the last MDNorm (out[0]) and BinMD (out[1]) launch on this grid:
 * 0 = global fp64 red.add, 1 = fp64 shared-memory partials, 2 = fp32 shared-memory partials
 * (tracing and tests; host only, no synchronisation).  MDN_EINVAL: NULL argument. */
mdn_status mdnorm_accumulation_paths(mdn_grid *g, int32_t out[2]);

/* Message of the last non-OK status on this thread ("" if none).  Never NULL. */
const char *mdn_last_error(void);

/* Library build identification, e.g. "mdnorm sm_100a <version>". */
const char *mdn_version(void);

/* ---------------- parity / test entry points (same kernels; not for users) ---------------- */

/* MDNorm with final matrices M: double[nmat][9] (host, nmat <= MDN_MAX_MATS) and per-matrix
 * charge: double[nmat]; same kernel as mdnorm_accumulate with the composition step skipped. */
mdn_status mdnorm_accumulate_matrices(mdn_grid *g, int32_t nmat, const double *M,
                                      const double *charge, double k_min, double k_max,
                                      int64_t pix_begin, int64_t pix_end, int64_t pix_stride,
                                      void *stream);

/* BinMD with final matrices N: double[nmat][9] (host, nmat <= MDN_MAX_MATS). */
mdn_status binmd_accumulate_matrices(mdn_grid *g, int32_t nmat, const double *N, int64_t nevents,
                                     const float *events, int64_t stride_floats, int32_t col_w,
                                     int32_t col_q, void *stream);

/* Per-trajectory geometry through the production device code.  traj_ids[t] = m * npix + p
 * selects matrix m of M (double[nmat][9], host) and pixel p.  Outputs (HOST arrays):
 * n_cross[t] = |L| (clip endpoints + kept plane crossings, 0 if the trajectory misses the grid),
 * n_seg[t] = segments appended, seg_bins/seg_vals[t * max_segs + i] = bin and value of segment
 * i (first max_segs only; values use Omega_p * charge[m]).  Synchronous. */
mdn_status mdnorm_debug_trajectories(mdn_grid *g, int32_t nmat, const double *M,
                                     const double *charge, double k_min, double k_max,
                                     int64_t ntraj, const int64_t *traj_ids, int32_t *n_cross,
                                     int32_t *n_seg, int64_t *seg_bins, double *seg_vals,
                                     int64_t max_segs);

/* Bin index (-1 = outside) of every (matrix, event) pair through the production BinMD decision
 * (the same device functions as binmd_accumulate: op-class test, fp32 per-axis bins inside the
 * proven error band, the exact fp64 formula for pairs within the band of a bin edge):
 * bins[m * nevents + e] (HOST int64 array).  Synchronous. */
mdn_status binmd_debug_bins(mdn_grid *g, int32_t nmat, const double *N, int64_t nevents,
                            const float *events, int64_t stride_floats, int32_t col_w,
                            int32_t col_q, int64_t *bins);

/* Largest number of trajectories (matrix x pixel) per cull/walk slab of later MDNorm calls
 * (max_traj in [1, 2^27]; 0 restores the default 2^27), so small inputs can exercise the
 * multi-slab path.  No device work.  MDN_EINVAL: NULL grid or max_traj out of range. */
mdn_status mdnorm_debug_set_max_slab(mdn_grid *g, int64_t max_traj);

/* Launch facts of the last MDNorm call on g (HOST int64[4]): {slabs of its last launch block,
 * hitters written by the cull of its last slab, the walk's large-launch threshold (hitters above
 * which warps claim 32 hitters at a time with no static per-CTA blocks), the slab limit}.
 * Synchronises the device. */
mdn_status mdnorm_debug_last_launch(mdn_grid *g, int64_t out[4]);

/* The interval guess mdnorm_set_flux[_tables] chose for flux table `table` (HOST double[2]):
 * {mode: 0 none, 1 knots near-uniform in k, 2 near-uniform in 1/k (wavelength); the fraction of
 * the table's k range on which the fp32 guess names the interval (0 for mode 0)}.  The guess only
 * proposes an interval that the exact comparisons kappa_i <= x < kappa_{i+1} then accept or
 * reject, so it never changes a value.  MDN_EINVAL: NULL argument or no such table. */
mdn_status mdnorm_debug_flux_guess(mdn_grid *g, int32_t table, double out[2]);

/* M_{r,s} / N_s exactly as the kernels compose them (device code; HOST outputs).  M: double
 * [nruns*nops][9] run-major; N: double[nops][9].  Synchronous (test entry point). */
mdn_status mdnorm_debug_compose(mdn_grid *g, const double UB[9], int32_t nruns, const double *R,
                                int32_t nops, const double *ops, double *M, double *N);

#ifdef __cplusplus
}
#endif
#endif /* MDNORM_H */
