/*
 * oracle.c -- plain fp64 CPU oracle for MDNorm + BinMD + cross-section.
 *
 * TEST INFRASTRUCTURE ONLY (see oracle.h): loaded by tests/, __graft_entry__.smoke() and the
 * bench.py cpu_baseline / --impl reference legs; never by the product path.
 *
 * Every function follows the paper's algorithm in the paper's order, with the readings of
 * SURVEY.md §8(c) (listed again in DESIGN.md §3).  Nothing is blocked, fused or reordered: a
 * trajectory loops over ALL bin planes of each axis (Listing 1), the kept
 * intersections are sorted with qsort, the flux is interpolated at each intersection
 * and each segment is appended to the histogram.
 *
 * Build: gcc -O2 -std=c11 -ffp-contract=off -fno-fast-math -fPIC -shared (x86-64 SSE2 doubles:
 * every +,-,*,/ below is one IEEE-754 round-to-nearest operation, no FMA contraction).
 */
#include "oracle.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>

static const double ORC_PI = 3.14159265358979323846;

/* ------------------------------------------------------------------ Neumaier accumulation */

static void neu_add(double *sum, double *comp, int64_t b, double x) {
  double s = sum[b];
  double t = s + x;
  if (fabs(s) >= fabs(x))
    comp[b] += (s - t) + x;
  else
    comp[b] += (x - t) + s;
  sum[b] = t;
}

/* ------------------------------------------------------------------ M0 / B0: matrices      */
/* C = A * B, row-major 3x3, each element ((a0*b0 + a1*b1) + a2*b2). */
static void matmul3(const double *A, const double *B, double *C) {
  for (int i = 0; i < 3; ++i)
    for (int j = 0; j < 3; ++j)
      C[3 * i + j] = (A[3 * i + 0] * B[0 + j] + A[3 * i + 1] * B[3 + j]) + A[3 * i + 2] * B[6 + j];
}

/* out = inverse(C) * scale via the adjugate: out_ij = (cof_ji / det) * scale. */
static int inv3_scaled(const double *C, double scale, double *out) {
  double cof[9];
  cof[0] = C[4] * C[8] - C[5] * C[7];
  cof[1] = C[5] * C[6] - C[3] * C[8];
  cof[2] = C[3] * C[7] - C[4] * C[6];
  cof[3] = C[2] * C[7] - C[1] * C[8];
  cof[4] = C[0] * C[8] - C[2] * C[6];
  cof[5] = C[1] * C[6] - C[0] * C[7];
  cof[6] = C[1] * C[5] - C[2] * C[4];
  cof[7] = C[2] * C[3] - C[0] * C[5];
  cof[8] = C[0] * C[4] - C[1] * C[3];
  double det = (C[0] * cof[0] + C[1] * cof[1]) + C[2] * cof[2];
  if (det == 0.0 || !isfinite(det)) return -1;
  for (int i = 0; i < 3; ++i)
    for (int j = 0; j < 3; ++j) out[3 * i + j] = (cof[3 * j + i] / det) * scale;
  return 0;
}

static double inv_two_pi(void) { return 1.0 / (2.0 * ORC_PI); }

/* M_{r,s} = (R_r * UB * S_s * W)^-1 / (2 pi): maps a lab-frame Q to grid coordinates
 * (reading #1-#2: Q_sample = R^-1 Q_lab = 2 pi UB h, h = S W x). */
int orc_compose_mdnorm(const double R[9], const double UB[9], const double S[9], const double W[9],
                       double M[9]) {
  double A[9], B[9], C[9];
  matmul3(R, UB, A);
  matmul3(A, S, B);
  matmul3(B, W, C);
  return inv3_scaled(C, inv_two_pi(), M);
}

/* N_s = (UB * S_s * W)^-1 / (2 pi): events are already in Q_sample. */
int orc_compose_binmd(const double UB[9], const double S[9], const double W[9], double N[9]) {
  double B[9], C[9];
  matmul3(UB, S, B);
  matmul3(B, W, C);
  return inv3_scaled(C, inv_two_pi(), N);
}

/* ------------------------------------------------------------------ M5: flux               */
/* F(x): clamp outside the table; otherwise i = max{i : kappa_i <= x} and linear interpolation
 * Phi_i + (Phi_{i+1} - Phi_i) * ((x - kappa_i) / (kappa_{i+1} - kappa_i)). */
double orc_flux(int64_t nflux, const double *fk, const double *fF, double x) {
  if (x <= fk[0]) return fF[0];
  if (x >= fk[nflux - 1]) return fF[nflux - 1];
  int64_t lo = 0, hi = nflux - 1; /* invariant: fk[lo] <= x < fk[hi] */
  while (hi - lo > 1) {
    int64_t mid = lo + (hi - lo) / 2;
    if (fk[mid] <= x)
      lo = mid;
    else
      hi = mid;
  }
  return fF[lo] + (fF[lo + 1] - fF[lo]) * ((x - fk[lo]) / (fk[lo + 1] - fk[lo]));
}

/* ------------------------------------------------------------------ grid constants         */
typedef struct {
  double lo[3], hi[3], w[3], s[3];
  int64_t n[3];
} gconst;

static void grid_consts(const orc_grid *g, gconst *c) {
  for (int a = 0; a < 3; ++a) {
    c->lo[a] = g->lo[a];
    c->hi[a] = g->hi[a];
    c->n[a] = g->n[a];
    c->w[a] = (g->hi[a] - g->lo[a]) / (double)g->n[a];
    c->s[a] = 1.0 / c->w[a];
  }
}

/* interior bin edge e_{a,j} = lo_a + j * w_a (product rounded, then sum rounded) */
static double edge(const gconst *c, int a, int64_t j) { return c->lo[a] + (double)j * c->w[a]; }

static int cmp_double(const void *x, const void *y) {
  double a = *(const double *)x, b = *(const double *)y;
  return (a > b) - (a < b);
}

/* ------------------------------------------------------------------ M1-M7: one trajectory  */
/* Returns n_seg; segments are reported through seg_bins / seg_vals (first max_segs) and, when
 * sum/comp are given, appended to the histogram.  'buf' holds >= n0 + n1 + n2 + 2 doubles. */
static int32_t trajectory(const gconst *c, const double d[3], double omega_c,
                          int64_t nflux, const double *fk, const double *fF, const double M[9],
                          double k_min, double k_max, double *buf, int32_t *n_cross,
                          int64_t *seg_bins, double *seg_vals, int64_t max_segs,
                          double *sum, double *comp) {
  /* M1: q_p = z - d_p (k_i along +z, k_f along d_p; reading #1), v = M q_p */
  double q[3] = {-d[0], -d[1], 1.0 - d[2]};
  double v[3];
  for (int a = 0; a < 3; ++a) v[a] = (M[3 * a + 0] * q[0] + M[3 * a + 1] * q[1]) + M[3 * a + 2] * q[2];

  /* M2: clip [k_min, k_max] to the box, one slab per axis */
  double k_in = k_min, k_out = k_max;
  for (int a = 0; a < 3; ++a) {
    double lk, hk;
    if (v[a] > 0.0) {
      double r = 1.0 / v[a];
      lk = c->lo[a] * r;
      hk = c->hi[a] * r;
    } else if (v[a] < 0.0) {
      double r = 1.0 / v[a];
      lk = c->hi[a] * r;
      hk = c->lo[a] * r;
    } else {
      if (c->lo[a] <= 0.0 && 0.0 < c->hi[a]) continue;
      *n_cross = 0;
      return 0;
    }
    if (lk > k_in) k_in = lk;
    if (hk < k_out) k_out = hk;
  }
  if (!(k_in < k_out)) {
    *n_cross = 0;
    return 0;
  }

  /* M3: the three plane loops of Listing 1, interior planes j = 1 .. n_a - 1 */
  int64_t nk = 0;
  buf[nk++] = k_in;
  for (int a = 0; a < 3; ++a) {
    if (v[a] == 0.0) continue;
    double r = 1.0 / v[a];
    for (int64_t j = 1; j < c->n[a]; ++j) {
      double k = edge(c, a, j) * r;
      if (k_in < k && k < k_out) buf[nk++] = k;
    }
  }
  /* M4: sort; endpoints stay first/last because every kept k is strictly inside */
  qsort(buf + 1, (size_t)(nk - 1), sizeof(double), cmp_double);
  buf[nk++] = k_out;
  *n_cross = (int32_t)nk;

  /* M5-M7: interpolate and append each segment, midpoint rule */
  int32_t nseg = 0;
  double F1 = orc_flux(nflux, fk, fF, buf[0]);
  for (int64_t i = 0; i + 1 < nk; ++i) {
    double k1 = buf[i], k2 = buf[i + 1];
    if (!(k2 > k1)) continue;
    double F2 = orc_flux(nflux, fk, fF, k2);
    double km = 0.5 * (k1 + k2);
    int inside = 1;
    int64_t idx[3];
    for (int a = 0; a < 3; ++a) {
      double t = (km * v[a] - c->lo[a]) * c->s[a];
      if (!(0.0 <= t && t < (double)c->n[a])) {
        inside = 0;
        break;
      }
      idx[a] = (int64_t)floor(t);
    }
    if (inside) {
      int64_t b = idx[0] + c->n[0] * (idx[1] + c->n[1] * idx[2]);
      double val = (F2 - F1) * omega_c;
      if (nseg < max_segs) {
        if (seg_bins) seg_bins[nseg] = b;
        if (seg_vals) seg_vals[nseg] = val;
      }
      if (sum) neu_add(sum, comp, b, val);
      ++nseg;
    }
    F1 = F2;
  }
  return nseg;
}

int32_t orc_mdnorm_trajectory(const orc_grid *g, const double dir[3], double solid,
                              int64_t nflux, const double *fk, const double *fF,
                              const double M[9], double charge, double k_min, double k_max,
                              int32_t *n_cross, int64_t *seg_bins, double *seg_vals,
                              int64_t max_segs) {
  gconst c;
  grid_consts(g, &c);
  double *buf = (double *)malloc(sizeof(double) * (size_t)(c.n[0] + c.n[1] + c.n[2] + 2));
  int32_t ns = trajectory(&c, dir, solid * charge, nflux, fk, fF, M, k_min, k_max, buf, n_cross,
                          seg_bins, seg_vals, max_segs, NULL, NULL);
  free(buf);
  return ns;
}

/* Listing 1: for each op (matrix m = run * nops + op), for each detector p. */
int64_t orc_mdnorm(const orc_grid *g, int64_t npix, const double *dir, const double *solid,
                   int64_t nflux, const double *fk, const double *fF,
                   int32_t nmat, const double *M, const double *charge,
                   double k_min, double k_max,
                   int64_t pix_begin, int64_t pix_end, int64_t pix_stride,
                   double *norm_sum, double *norm_comp) {
  return orc_mdnorm_krange(g, npix, dir, solid, NULL, NULL, nflux, fk, fF, nmat, M, charge, k_min,
                           k_max, pix_begin, pix_end, pix_stride, norm_sum, norm_comp);
}

/* Same, with optional per-pixel momentum limits (S§8(f) NEXT #1; Mantid's MDNorm_low/high):
 * pixel p's trajectory runs over [max(k_min, pix_kmin[p]), min(k_max, pix_kmax[p])]. */
int64_t orc_mdnorm_krange(const orc_grid *g, int64_t npix, const double *dir, const double *solid,
                          const double *pix_kmin, const double *pix_kmax,
                          int64_t nflux, const double *fk, const double *fF,
                          int32_t nmat, const double *M, const double *charge,
                          double k_min, double k_max,
                          int64_t pix_begin, int64_t pix_end, int64_t pix_stride,
                          double *norm_sum, double *norm_comp) {
  const int64_t offsets[2] = {0, nflux};
  return orc_mdnorm_tables(g, npix, dir, solid, pix_kmin, pix_kmax, 1, offsets, fk, fF, NULL, nmat,
                           M, charge, k_min, k_max, pix_begin, pix_end, pix_stride, norm_sum,
                           norm_comp);
}

/* Most general form: per-bank flux tables (S§8(f) NEXT #1).  Table t is fk/fF[offsets[t] ..
 * offsets[t+1]); pixel p uses table pixel_table[p] (NULL: table 0 for every pixel). */
int64_t orc_mdnorm_tables(const orc_grid *g, int64_t npix, const double *dir, const double *solid,
                          const double *pix_kmin, const double *pix_kmax, int32_t ntables,
                          const int64_t *offsets, const double *fk, const double *fF,
                          const int32_t *pixel_table, int32_t nmat, const double *M,
                          const double *charge, double k_min, double k_max, int64_t pix_begin,
                          int64_t pix_end, int64_t pix_stride, double *norm_sum, double *norm_comp) {
  (void)ntables;
  gconst c;
  grid_consts(g, &c);
  if (pix_end > npix) pix_end = npix;
  double *buf = (double *)malloc(sizeof(double) * (size_t)(c.n[0] + c.n[1] + c.n[2] + 2));
  int64_t ntraj = 0;
  for (int32_t m = 0; m < nmat; ++m) {
    for (int64_t p = pix_begin; p < pix_end; p += pix_stride) {
      int32_t ncross;
      double lo = k_min, hi = k_max;
      if (pix_kmin && pix_kmin[p] > lo) lo = pix_kmin[p];
      if (pix_kmax && pix_kmax[p] < hi) hi = pix_kmax[p];
      const int32_t t = pixel_table ? pixel_table[p] : 0;
      const int64_t o = offsets[t], nf = offsets[t + 1] - offsets[t];
      trajectory(&c, dir + 3 * p, solid[p] * charge[m], nf, fk + o, fF + o, M + 9 * m, lo, hi, buf,
                 &ncross, NULL, NULL, 0, norm_sum, norm_comp);
      ++ntraj;
    }
  }
  free(buf);
  return ntraj;
}

/* ------------------------------------------------------------------ B1-B3: BinMD           */
static int64_t event_bin(const gconst *c, const double *N, const float *ev, int32_t col_q) {
  double q[3] = {(double)ev[col_q], (double)ev[col_q + 1], (double)ev[col_q + 2]};
  int64_t idx[3];
  for (int a = 0; a < 3; ++a) {
    double x = (N[3 * a + 0] * q[0] + N[3 * a + 1] * q[1]) + N[3 * a + 2] * q[2];
    double t = (x - c->lo[a]) * c->s[a];
    if (!(0.0 <= t && t < (double)c->n[a])) return -1;
    idx[a] = (int64_t)floor(t);
  }
  return idx[0] + c->n[0] * (idx[1] + c->n[1] * idx[2]);
}

/* Listing 2/3: for each op, for each event, v = op * Q; push weight (column 1). */
int64_t orc_binmd(const orc_grid *g, int32_t nmat, const double *N, int64_t nevents,
                  const float *events, int64_t stride, int32_t col_w, int32_t col_q,
                  double *binmd_sum, double *binmd_comp) {
  gconst c;
  grid_consts(g, &c);
  int64_t inside = 0;
  for (int32_t m = 0; m < nmat; ++m)
    for (int64_t e = 0; e < nevents; ++e) {
      const float *ev = events + e * stride;
      int64_t b = event_bin(&c, N + 9 * m, ev, col_q);
      if (b >= 0) {
        neu_add(binmd_sum, binmd_comp, b, (double)ev[col_w]);
        ++inside;
      }
    }
  return inside;
}

void orc_binmd_bins(const orc_grid *g, int32_t nmat, const double *N, int64_t nevents,
                    const float *events, int64_t stride, int32_t col_w, int32_t col_q,
                    int64_t *bins) {
  (void)col_w;
  gconst c;
  grid_consts(g, &c);
  for (int32_t m = 0; m < nmat; ++m)
    for (int64_t e = 0; e < nevents; ++e)
      bins[m * nevents + e] = event_bin(&c, N + 9 * m, events + e * stride, col_q);
}

/* Error histogram (S§8(f) NEXT #1: Mantid's MDEvent carries signal and error squared, P:188's
 * 8 columns): err2[b] += events[e*stride + col_e] for every (op, event) inside the grid. */
int64_t orc_binmd_err(const orc_grid *g, int32_t nmat, const double *N, int64_t nevents,
                      const float *events, int64_t stride, int32_t col_e, int32_t col_q,
                      double *err_sum, double *err_comp) {
  gconst c;
  grid_consts(g, &c);
  int64_t inside = 0;
  for (int32_t m = 0; m < nmat; ++m)
    for (int64_t e = 0; e < nevents; ++e) {
      const float *ev = events + e * stride;
      int64_t b = event_bin(&c, N + 9 * m, ev, col_q);
      if (b >= 0) {
        neu_add(err_sum, err_comp, b, (double)ev[col_e]);
        ++inside;
      }
    }
  return inside;
}

/* ------------------------------------------------------------------ X2: divide             */
void orc_cross_section(int64_t nbins, const double *binmd, const double *norm, double *xs) {
  for (int64_t b = 0; b < nbins; ++b) xs[b] = norm[b] > 0.0 ? binmd[b] / norm[b] : NAN;
}

/* Error of the cross-section: the normalization carries no error (it is computed, not
 * counted), so sigma_xs = sqrt(err2) / norm; NaN where norm == 0. */
void orc_cross_section_err(int64_t nbins, const double *err2, const double *norm, double *xs_err) {
  for (int64_t b = 0; b < nbins; ++b) xs_err[b] = norm[b] > 0.0 ? sqrt(err2[b]) / norm[b] : NAN;
}
