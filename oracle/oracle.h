/*
 * oracle.h -- plain, slow, double-precision CPU oracle for MDNorm + BinMD + cross-section.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load or call this library.  The product path (the CUDA C-ABI library
 * in paper_conf_sc_hahnfgmmshvvs24_b200/) never includes, links or calls it, and this file shares
 * no code, header, table or constant generator with it.
 *
 * What it computes (PAPER.md = "P:"):
 *   norm[b]  = sum_r sum_s sum_p c_r * Omega_p * integral_{k_min}^{k_max} 1[k*v_{r,s,p} in b] dF(k)
 *   binmd[b] = sum_s sum_e w_e * 1[N_s * q_e in b]
 *   xs[b]    = binmd[b] / norm[b]     ("sum of all histograms over the sum of all
 *                                        normalizations", Algorithm 1)
 * evaluated step by step in the order of Listing 1: for each op, for each detector,
 * loop over the H, K and L bin planes collecting intersections, sort them,
 * linearly interpolate the integrated flux and append to the histogram;
 * BinMD follows Listing 2/3: transform each event by each op, push its weight.
 *
 * Conventions (readings listed in DESIGN.md §3): no FMA contraction (compile with
 * -ffp-contract=off), IEEE double, Neumaier-compensated accumulation into (sum, comp) pairs
 * whose final value is sum + comp.
 */
#ifndef MDN_ORACLE_H
#define MDN_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct {
  double lo[3], hi[3];
  int64_t n[3];
} orc_grid;

/* M = inv(R*UB*S*W) * (1/(2*pi));  N = inv(UB*S*W) * (1/(2*pi)).  Row-major 3x3. 0 on success,
 * -1 if the composed matrix is singular. */
int orc_compose_mdnorm(const double R[9], const double UB[9], const double S[9], const double W[9],
                       double M[9]);
int orc_compose_binmd(const double UB[9], const double S[9], const double W[9], double N[9]);

/* F(x) from the cumulative flux table (P:116 linear_interpolation, P:428 FluxFile). */
double orc_flux(int64_t nflux, const double *fk, const double *fF, double x);

/* MDNorm over trajectories (m, p) for m in [0, nmat), p = pix_begin, pix_begin+stride, ...
 * < pix_end.  Adds into norm_sum/norm_comp (nbins each).  charge[m] = c_r of matrix m.
 * Returns the number of trajectories processed. */
int64_t orc_mdnorm(const orc_grid *g, int64_t npix, const double *dir, const double *solid,
                   int64_t nflux, const double *fk, const double *fF,
                   int32_t nmat, const double *M, const double *charge,
                   double k_min, double k_max,
                   int64_t pix_begin, int64_t pix_end, int64_t pix_stride,
                   double *norm_sum, double *norm_comp);

/* orc_mdnorm with optional per-pixel momentum limits (NULL = none): pixel p runs over
 * [max(k_min, pix_kmin[p]), min(k_max, pix_kmax[p])] (S§8(f) NEXT #1, Mantid MDNorm_low/high). */
int64_t orc_mdnorm_krange(const orc_grid *g, int64_t npix, const double *dir, const double *solid,
                          const double *pix_kmin, const double *pix_kmax,
                          int64_t nflux, const double *fk, const double *fF,
                          int32_t nmat, const double *M, const double *charge,
                          double k_min, double k_max,
                          int64_t pix_begin, int64_t pix_end, int64_t pix_stride,
                          double *norm_sum, double *norm_comp);

/* Most general form: per-bank flux tables.  Table t = fk/fF[offsets[t] .. offsets[t+1]); pixel p
 * uses table pixel_table[p] (NULL: table 0).  Optional per-pixel limits as above. */
int64_t orc_mdnorm_tables(const orc_grid *g, int64_t npix, const double *dir, const double *solid,
                          const double *pix_kmin, const double *pix_kmax, int32_t ntables,
                          const int64_t *offsets, const double *fk, const double *fF,
                          const int32_t *pixel_table, int32_t nmat, const double *M,
                          const double *charge, double k_min, double k_max, int64_t pix_begin,
                          int64_t pix_end, int64_t pix_stride, double *norm_sum, double *norm_comp);

/* One trajectory, for bit-exact debug checks: n_cross = |L| (endpoints + kept crossings),
 * n_seg = number of segments appended, seg_bins/seg_vals = the first max_segs of them in order.
 * Returns n_seg. */
int32_t orc_mdnorm_trajectory(const orc_grid *g, const double dir[3], double solid,
                              int64_t nflux, const double *fk, const double *fF,
                              const double M[9], double charge, double k_min, double k_max,
                              int32_t *n_cross, int64_t *seg_bins, double *seg_vals,
                              int64_t max_segs);

/* BinMD: events[e*stride + col_w] = weight, events[e*stride + col_q + 0..2] = Q_sample.
 * Adds into binmd_sum/binmd_comp.  Returns the number of (op, event) pairs inside the grid. */
int64_t orc_binmd(const orc_grid *g, int32_t nmat, const double *N, int64_t nevents,
                  const float *events, int64_t stride, int32_t col_w, int32_t col_q,
                  double *binmd_sum, double *binmd_comp);

/* Bin index of every (op, event) pair, op-major: bins[m*nevents + e]; -1 = outside. */
void orc_binmd_bins(const orc_grid *g, int32_t nmat, const double *N, int64_t nevents,
                    const float *events, int64_t stride, int32_t col_w, int32_t col_q,
                    int64_t *bins);

/* Error-squared histogram: err2[b] += events[e*stride + col_e] per (op, event) inside. */
int64_t orc_binmd_err(const orc_grid *g, int32_t nmat, const double *N, int64_t nevents,
                      const float *events, int64_t stride, int32_t col_e, int32_t col_q,
                      double *err_sum, double *err_comp);

/* xs[b] = binmd[b] / norm[b] if norm[b] > 0 else NaN. */
void orc_cross_section(int64_t nbins, const double *binmd, const double *norm, double *xs);

/* xs_err[b] = sqrt(err2[b]) / norm[b] if norm[b] > 0 else NaN. */
void orc_cross_section_err(int64_t nbins, const double *err2, const double *norm, double *xs_err);

#ifdef __cplusplus
}
#endif
#endif
