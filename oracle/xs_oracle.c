/*
 * xs_oracle.c — CPU ORACLE (TEST INFRASTRUCTURE ONLY; see xs_oracle.h).
 *
 * Plain C, fp64, one serial function per step.  Build:
 *   gcc -O2 -ffp-contract=off -fno-fast-math -fPIC -shared
 * No blocking, fusion or reordering: every loop runs in the order the
 * readings (R1-R17) state.  Shares no code with the CUDA path;
 * the only shared module is the input generator gen/xs_gen.h.
 */
#include "xs_oracle.h"

#include <math.h>
#include <pthread.h>
#include <stdlib.h>
#include <string.h>

#include "../gen/xs_gen.h"

/* ------------------------------------------------------------------ RNG --
 * R2: 63-bit LCG, m = 2^63, a = 2806196910506780709, c = 1; a draw is
 * s / 2^63 (XSBench v20 LCG_random_double).                              */
static const uint64_t LCG_A = 2806196910506780709ULL;
static const uint64_t LCG_C = 1ULL;
static const uint64_t LCG_M = 9223372036854775808ULL; /* 2^63 */

uint64_t oracle_lcg_step(uint64_t s) { return (LCG_A * s + LCG_C) % LCG_M; }

double oracle_lcg_to_double(uint64_t s) { return (double)s / (double)LCG_M; }

/* R2: FF(s, n) = LCG^n(s) by square-and-multiply of the affine map
 * x -> a x + c (XSBench fast_forward_LCG): for each bit of n from the LSB,
 * if set (A, C) <- (A a, C a + c); then (c, a) <- (c (a + 1), a^2); all mod
 * 2^63.  Result (A s + C) mod 2^63.                                        */
uint64_t oracle_fast_forward(uint64_t s, uint64_t n) {
  uint64_t a = LCG_A, c = LCG_C, A = 1, C = 0;
  n = n % LCG_M;
  while (n > 0) {
    if (n & 1ULL) {
      A = A * a;
      C = C * a + c;
    }
    c = c * (a + 1);
    a = a * a;
    n >>= 1;
  }
  return (A * s + C) % LCG_M;
}

/* R3: pick_mat.  dist[] is the XSBench core-volume fraction table; the
 * threshold for material m is the running sum dist[m] + dist[m-1] + ... +
 * dist[1] taken in that (descending j) order.                              */
static const double MAT_DIST[12] = {0.140, 0.052, 0.275, 0.134, 0.154, 0.064,
                                    0.066, 0.055, 0.008, 0.015, 0.025, 0.013};

void oracle_thresholds(double T[12]) {
  for (int m = 0; m < 12; m++) {
    double running = 0;
    for (int j = m; j > 0; j--) running += MAT_DIST[j];
    T[m] = running;
  }
}

int32_t oracle_pick_mat(double roll) {
  double T[12];
  oracle_thresholds(T);
  for (int m = 0; m < 12; m++)
    if (roll < T[m]) return m;
  return 0;
}

/* R4: lookup id -> (p, mat): s = FF(seed, 2 id); p = draw(s); roll =
 * draw(s); mat = pick_mat(roll).  (XSBench event kernel, 2 draws/lookup.) */
void oracle_sample(uint64_t lookup_seed, uint64_t id, double* p, int32_t* mat) {
  uint64_t s = oracle_fast_forward(lookup_seed, 2 * id);
  s = oracle_lcg_step(s);
  double pe = oracle_lcg_to_double(s);
  s = oracle_lcg_step(s);
  double roll = oracle_lcg_to_double(s);
  if (p) *p = pe;
  if (mat) *mat = oracle_pick_mat(roll);
}

/* --------------------------------------------------------------- search --
 * XSBench grid_search shape on A[lo..hi]: while (hi - lo > 1) probe the
 * midpoint; A[mid] > q moves hi, else lo.  Returns lo.                    */
int64_t oracle_grid_search(const double* A, int64_t lo, int64_t hi, double q) {
  int64_t length = hi - lo;
  while (length > 1) {
    int64_t mid = lo + length / 2;
    if (A[mid] > q)
      hi = mid;
    else
      lo = mid;
    length = hi - lo;
  }
  return lo;
}

/* ub(A, q) = #{x in A : x <= q} for sorted A (plain binary search). */
int64_t oracle_upper_bound(const double* A, int64_t n, double q) {
  int64_t lo = 0, hi = n; /* answer in [lo, hi] */
  while (lo < hi) {
    int64_t mid = lo + (hi - lo) / 2;
    if (A[mid] <= q)
      lo = mid + 1;
    else
      hi = mid;
  }
  return lo;
}

/* Strided view: ub over the energies of nuclide n (stride 6 doubles). */
static int64_t ub_nuclide(const double* grid, int64_t N, int32_t n, double q) {
  const double* E = grid + (int64_t)n * N * 6;
  int64_t lo = 0, hi = N;
  while (lo < hi) {
    int64_t mid = lo + (hi - lo) / 2;
    if (E[mid * 6] <= q)
      lo = mid + 1;
    else
      hi = mid;
  }
  return lo;
}

static int64_t clamp64(int64_t x, int64_t lo, int64_t hi) { return x < lo ? lo : (x > hi ? hi : x); }

/* ---------------------------------------------------------------- ctx -- */
struct oracle_ctx {
  int32_t I;
  int64_t N;
  double* grid; /* [I][N][6] */
  int32_t n_mats, max_nucs;
  int32_t* num_nucs;
  int32_t* mats;
  double* concs;
  uint64_t lookup_seed;
  int64_t NU;
  double* U; /* [NU] sorted multiset of all energies (R6) */
  int32_t B;  /* hash bins (0 = none) */
  double du;
  int32_t* HG; /* [B][I] (R7) */
};

static int cmp_double(const void* a, const void* b) {
  double x = *(const double*)a, y = *(const double*)b;
  return (x > y) - (x < y);
}

static int finish_ctx(oracle_ctx* c, int32_t hash_bins) {
  /* R6: U = all I*N energies, sorted ascending (a library sort is a step). */
  c->NU = (int64_t)c->I * c->N;
  c->U = (double*)malloc((size_t)c->NU * sizeof(double));
  if (!c->U) return 2;
  for (int64_t g = 0; g < c->NU; g++) c->U[g] = c->grid[g * 6];
  qsort(c->U, (size_t)c->NU, sizeof(double), cmp_double);
  /* R7: the hash grid, by definition, one entry at a time. */
  c->B = hash_bins > 0 ? hash_bins : 0;
  c->HG = NULL;
  if (c->B > 0) {
    c->du = 1.0 / (double)c->B;
    c->HG = (int32_t*)malloc((size_t)c->B * c->I * sizeof(int32_t));
    if (!c->HG) return 2;
    for (int64_t b = 0; b < c->B; b++)
      for (int32_t n = 0; n < c->I; n++) c->HG[b * c->I + n] = oracle_hash_entry(c, b, n);
  }
  return 0;
}

oracle_ctx* oracle_create_arrays(int32_t I, int64_t N, const double* grid, int32_t n_mats,
                                 int32_t max_nucs, const int32_t* num_nucs, const int32_t* mats,
                                 const double* concs, uint64_t lookup_seed, int32_t hash_bins,
                                 int* err) {
  int e = 0;
  oracle_ctx* c = NULL;
  if (I < 1 || N < 2 || !grid || n_mats < 1 || max_nucs < 1 || !num_nucs || !mats || !concs) {
    e = 1;
    goto out;
  }
  c = (oracle_ctx*)calloc(1, sizeof(oracle_ctx));
  if (!c) { e = 2; goto out; }
  c->I = I;
  c->N = N;
  c->n_mats = n_mats;
  c->max_nucs = max_nucs;
  c->lookup_seed = lookup_seed;
  c->grid = (double*)malloc((size_t)I * N * 6 * sizeof(double));
  c->num_nucs = (int32_t*)malloc((size_t)n_mats * sizeof(int32_t));
  c->mats = (int32_t*)malloc((size_t)n_mats * max_nucs * sizeof(int32_t));
  c->concs = (double*)malloc((size_t)n_mats * max_nucs * sizeof(double));
  if (!c->grid || !c->num_nucs || !c->mats || !c->concs) { e = 2; goto out; }
  memcpy(c->grid, grid, (size_t)I * N * 6 * sizeof(double));
  memcpy(c->num_nucs, num_nucs, (size_t)n_mats * sizeof(int32_t));
  memcpy(c->mats, mats, (size_t)n_mats * max_nucs * sizeof(int32_t));
  memcpy(c->concs, concs, (size_t)n_mats * max_nucs * sizeof(double));
  for (int32_t m = 0; m < n_mats; m++) {
    if (num_nucs[m] < 0 || num_nucs[m] > max_nucs) { e = 1; goto out; }
    for (int32_t j = 0; j < num_nucs[m]; j++)
      if (mats[m * max_nucs + j] < 0 || mats[m * max_nucs + j] >= I) { e = 1; goto out; }
  }
  /* R15: energies strictly increasing per nuclide. */
  for (int32_t n = 0; n < I; n++)
    for (int64_t k = 1; k < N; k++)
      if (!(grid[((int64_t)n * N + k - 1) * 6] < grid[((int64_t)n * N + k) * 6])) { e = 3; goto out; }
  e = finish_ctx(c, hash_bins);
out:
  if (err) *err = e;
  if (e && c) { oracle_free(c); c = NULL; }
  return c;
}

oracle_ctx* oracle_create_spec(int32_t I, int64_t N, uint64_t grid_seed, uint64_t conc_seed,
                               int32_t material_rule, uint64_t lookup_seed, int32_t hash_bins,
                               int nthreads, int* err) {
  int e = 0;
  oracle_ctx* c = NULL;
  int32_t num_nucs[12];
  int32_t mx = xsgen_max_num_nucs(I, material_rule);
  if (mx < 1 || N < 2) { if (err) *err = 1; return NULL; }
  c = (oracle_ctx*)calloc(1, sizeof(oracle_ctx));
  if (!c) { if (err) *err = 2; return NULL; }
  c->I = I;
  c->N = N;
  c->n_mats = 12;
  c->max_nucs = mx;
  c->lookup_seed = lookup_seed;
  c->grid = (double*)malloc((size_t)I * N * 6 * sizeof(double));
  c->num_nucs = (int32_t*)malloc(12 * sizeof(int32_t));
  c->mats = (int32_t*)malloc((size_t)12 * mx * sizeof(int32_t));
  c->concs = (double*)malloc((size_t)12 * mx * sizeof(double));
  if (!c->grid || !c->num_nucs || !c->mats || !c->concs) { e = 2; goto out; }
  if (xsgen_num_nucs(I, material_rule, num_nucs) || xsgen_mats(I, material_rule, mx, c->mats) ||
      xsgen_concs(conc_seed, num_nucs, mx, c->concs)) { e = 1; goto out; }
  memcpy(c->num_nucs, num_nucs, sizeof(num_nucs));
  {
    int ge = xsgen_nuclide_grid(I, N, grid_seed, c->grid, nthreads);
    if (ge == XSGEN_ERR_DUP_ENERGY) { e = 3; goto out; }
    if (ge) { e = 1; goto out; }
  }
  e = finish_ctx(c, hash_bins);
out:
  if (err) *err = e;
  if (e && c) { oracle_free(c); c = NULL; }
  return c;
}

void oracle_free(oracle_ctx* c) {
  if (!c) return;
  free(c->grid);
  free(c->num_nucs);
  free(c->mats);
  free(c->concs);
  free(c->U);
  free(c->HG);
  free(c);
}

int32_t oracle_n_isotopes(const oracle_ctx* c) { return c->I; }
int64_t oracle_n_gridpoints(const oracle_ctx* c) { return c->N; }
int32_t oracle_n_mats(const oracle_ctx* c) { return c->n_mats; }
int32_t oracle_max_num_nucs(const oracle_ctx* c) { return c->max_nucs; }
int64_t oracle_union_len(const oracle_ctx* c) { return c->NU; }
const double* oracle_grid(const oracle_ctx* c) { return c->grid; }
const double* oracle_union(const oracle_ctx* c) { return c->U; }
const int32_t* oracle_num_nucs(const oracle_ctx* c) { return c->num_nucs; }
const int32_t* oracle_mats(const oracle_ctx* c) { return c->mats; }
const double* oracle_concs(const oracle_ctx* c) { return c->concs; }

/* R5: the plain definition of the bracket of nuclide n at energy p. */
int64_t oracle_nuclide_bracket(const oracle_ctx* c, int32_t n, double p) {
  return clamp64(ub_nuclide(c->grid, c->N, n, p) - 1, 0, c->N - 2);
}

/* R6: unionized index u. */
int64_t oracle_union_index(const oracle_ctx* c, double p) {
  return clamp64(oracle_upper_bound(c->U, c->NU, p) - 1, 0, c->NU - 2);
}

/* R6: one entry of the unionized index grid, by definition. */
int32_t oracle_index_grid_entry(const oracle_ctx* c, int64_t e, int32_t n) {
  return (int32_t)clamp64(ub_nuclide(c->grid, c->N, n, c->U[e]) - 1, 0, c->N - 2);
}

/* R6 / pin P5: XSBench's incremental sweep over U (GridInit.c): idx_low[n]
 * starts at 0 and energy_high[n] at E_n[1]; for each e in order and each n,
 * if U[e] >= energy_high[n] and idx_low[n] < N-2 the index advances by one. */
int oracle_index_grid_sweep(const oracle_ctx* c, int32_t* out) {
  int32_t* idx_low = (int32_t*)calloc((size_t)c->I, sizeof(int32_t));
  double* energy_high = (double*)malloc((size_t)c->I * sizeof(double));
  if (!idx_low || !energy_high) { free(idx_low); free(energy_high); return 2; }
  for (int32_t n = 0; n < c->I; n++) energy_high[n] = c->grid[((int64_t)n * c->N + 1) * 6];
  for (int64_t e = 0; e < c->NU; e++) {
    double ue = c->U[e];
    for (int32_t n = 0; n < c->I; n++) {
      if (ue < energy_high[n]) {
        out[e * c->I + n] = idx_low[n];
      } else if (idx_low[n] == c->N - 2) {
        out[e * c->I + n] = idx_low[n];
      } else {
        idx_low[n]++;
        out[e * c->I + n] = idx_low[n];
        energy_high[n] = c->grid[((int64_t)n * c->N + idx_low[n] + 1) * 6];
      }
    }
  }
  free(idx_low);
  free(energy_high);
  return 0;
}

/* R8/R9: b = trunc(p / du), du = 1.0 / B, clamped to [0, B-1] (p = 1.0
 * gives B; explicit lookups may pass p < 0). */
int64_t oracle_hash_bin(const oracle_ctx* c, double p) {
  double q = p / c->du;
  if (!(q > 0.0)) return 0;
  if (q >= (double)c->B) return c->B - 1;
  return (int64_t)q;
}

/* R7: HG[b][n] = bracket of nuclide n at the bin's lower edge b du. */
int32_t oracle_hash_entry(const oracle_ctx* c, int64_t b, int32_t n) {
  double e = (double)b * c->du;
  return (int32_t)clamp64(ub_nuclide(c->grid, c->N, n, e) - 1, 0, c->N - 2);
}

/* R7: XSBench hash bracket.  u_lo = HG[b][n]; u_hi = N-1 for the last bin,
 * else HG[b+1][n] + 1.  p <= E[u_lo] -> u_lo (R7: XSBench writes 0 here,
 * which differs from the definition only when p equals a grid energy lying
 * on a bin edge); p >= E[u_hi] -> N-1; else grid_search on [u_lo, u_hi].
 * The result N-1 is clamped to N-2 (XSBench "low = lower - 1").          */
int64_t oracle_hash_bracket(const oracle_ctx* c, int64_t b, int32_t n, double p) {
  const double* E = c->grid + (int64_t)n * c->N * 6;
  int64_t u_lo = c->HG[b * c->I + n];
  int64_t u_hi = (b == c->B - 1) ? c->N - 1 : (int64_t)c->HG[(b + 1) * c->I + n] + 1;
  int64_t lower;
  if (p <= E[u_lo * 6])
    lower = u_lo;
  else if (p >= E[u_hi * 6])
    lower = c->N - 1;
  else {
    /* grid_search over the strided energies E[u_lo..u_hi] */
    int64_t lo = u_lo, hi = u_hi, length = hi - lo;
    while (length > 1) {
      int64_t mid = lo + length / 2;
      if (E[mid * 6] > p)
        hi = mid;
      else
        lo = mid;
      length = hi - lo;
    }
    lower = lo;
  }
  return lower == c->N - 1 ? c->N - 2 : lower;
}

/* R10: linear interpolation of the five channels between records k and k+1:
 *   f = (hi.E - p) / (hi.E - lo.E);  x_c = hi.c - f * (hi.c - lo.c).
 * Each operation is a separate IEEE binary64 op (no FMA).               */
void oracle_micro_xs(const oracle_ctx* c, int32_t n, int64_t k, double p, double xs[5]) {
  const double* lo = c->grid + ((int64_t)n * c->N + k) * 6;
  const double* hi = lo + 6;
  double f = (hi[0] - p) / (hi[0] - lo[0]);
  for (int ch = 0; ch < 5; ch++) {
    double d = hi[1 + ch] - lo[1 + ch];
    double t = f * d;
    xs[ch] = hi[1 + ch] - t;
  }
}

/* R5-R11: macroscopic XS of material mat at energy p.  M starts at +0.0;
 * nuclides are added in list order j = 0..num_nucs[mat]-1 as
 * M_c <- M_c + (x_c * conc_j).  grid_index receives u (UNIONIZED), b
 * (HASH) or -1 (NUCLIDE).                                                */
void oracle_macro_xs(const oracle_ctx* c, double p, int32_t mat, int mode, double M[5],
                     int64_t* grid_index) {
  int64_t idx = -1;
  for (int ch = 0; ch < 5; ch++) M[ch] = 0.0;
  if (mode == ORACLE_UNIONIZED) idx = oracle_union_index(c, p);
  if (mode == ORACLE_HASH) idx = oracle_hash_bin(c, p);
  for (int32_t j = 0; j < c->num_nucs[mat]; j++) {
    int32_t n = c->mats[mat * c->max_nucs + j];
    double conc = c->concs[mat * c->max_nucs + j];
    int64_t k;
    if (mode == ORACLE_UNIONIZED)
      k = oracle_index_grid_entry(c, idx, n);
    else if (mode == ORACLE_HASH)
      k = oracle_hash_bracket(c, idx, n, p);
    else
      k = oracle_nuclide_bracket(c, n, p);
    double xs[5];
    oracle_micro_xs(c, n, k, p, xs);
    for (int ch = 0; ch < 5; ch++) {
      double w = xs[ch] * conc;
      M[ch] = M[ch] + w;
    }
  }
  if (grid_index) *grid_index = idx;
}

/* R18 (fp32 variant, north_star "1e-5 if an fp32 variant is offered";
 * SURVEY §8(f) NEXT-2): energies stay binary64, so the search and every
 * bracket are those of R5-R9; f is the binary64 quotient of R10, rounded once
 * to binary32; the channel values and concentrations are the binary64 data
 * rounded once to binary32; then, in binary32, each operation rounded once
 * (fmaf is IEEE 754's fusedMultiplyAdd: one rounding for a product and a sum):
 *   d = hi.c - lo.c;  x = fmaf(-f, d, hi.c).
 * The accumulation is blocked so that the north_star's 1e-5 bound holds for
 * every material (R18): nuclides j = 0..n-1 in list order,
 *   B_c = fmaf(x_c, conc_j, B_c)        (block sum, from +0.0f)
 *   after j = 15, 31, 47, ... and after j = n-1:  M_c = M_c + B_c, B_c = +0.0f
 * (M from +0.0f).  Error against binary64: |M32 - M64| <= (K + ceil(n/K) + 4)
 * 2^-24 sum_j conc_j (|hi.c| + |f| (|hi.c| + |lo.c|)), K = 16: 2.4e-6 of that
 * scale for the 321-nuclide fuel.                                         */
enum { ORACLE_F32_BLOCK = 16 };

void oracle_micro_xs_f32(const oracle_ctx* c, int32_t n, int64_t k, double p, float xs[5]) {
  const double* lo = c->grid + ((int64_t)n * c->N + k) * 6;
  const double* hi = lo + 6;
  double f64 = (hi[0] - p) / (hi[0] - lo[0]);
  float f = (float)f64;
  for (int ch = 0; ch < 5; ch++) {
    float h = (float)hi[1 + ch];
    float l = (float)lo[1 + ch];
    float d = h - l;
    xs[ch] = fmaf(-f, d, h);
  }
}

void oracle_macro_xs_f32(const oracle_ctx* c, double p, int32_t mat, int mode, double M[5],
                         int64_t* grid_index) {
  int64_t idx = -1;
  float Mf[5] = {0.0f, 0.0f, 0.0f, 0.0f, 0.0f};
  float Bf[5] = {0.0f, 0.0f, 0.0f, 0.0f, 0.0f};
  if (mode == ORACLE_UNIONIZED) idx = oracle_union_index(c, p);
  if (mode == ORACLE_HASH) idx = oracle_hash_bin(c, p);
  const int32_t nn = c->num_nucs[mat];
  for (int32_t j = 0; j < nn; j++) {
    int32_t n = c->mats[mat * c->max_nucs + j];
    float conc = (float)c->concs[mat * c->max_nucs + j];
    int64_t k;
    if (mode == ORACLE_UNIONIZED)
      k = oracle_index_grid_entry(c, idx, n);
    else if (mode == ORACLE_HASH)
      k = oracle_hash_bracket(c, idx, n, p);
    else
      k = oracle_nuclide_bracket(c, n, p);
    float xs[5];
    oracle_micro_xs_f32(c, n, k, p, xs);
    for (int ch = 0; ch < 5; ch++) Bf[ch] = fmaf(xs[ch], conc, Bf[ch]);
    if ((j + 1) % ORACLE_F32_BLOCK == 0 || j == nn - 1) {
      for (int ch = 0; ch < 5; ch++) {
        Mf[ch] = Mf[ch] + Bf[ch];
        Bf[ch] = 0.0f;
      }
    }
  }
  for (int ch = 0; ch < 5; ch++) M[ch] = (double)Mf[ch]; /* exact widening */
  if (grid_index) *grid_index = idx;
}

/* Error scales of the binary64 result (test infrastructure for the
 * tolerances of SURVEY Q12 and R18), binary64, nuclides in list order:
 *   A_c = sum_j |x_c conc_j|                     (Q12's condition-aware scale)
 *   S_c = sum_j conc_j (|hi.c| + |f| (|hi.c| + |lo.c|))   (R18's a-priori scale)
 * with x_c, f, hi, lo those of R10 at the bracket of R5.                    */
void oracle_macro_scales(const oracle_ctx* c, double p, int32_t mat, double A[5], double S[5]) {
  for (int ch = 0; ch < 5; ch++) A[ch] = S[ch] = 0.0;
  for (int32_t j = 0; j < c->num_nucs[mat]; j++) {
    int32_t n = c->mats[mat * c->max_nucs + j];
    double conc = c->concs[mat * c->max_nucs + j];
    int64_t k = oracle_nuclide_bracket(c, n, p);
    const double* lo = c->grid + ((int64_t)n * c->N + k) * 6;
    const double* hi = lo + 6;
    double f = (hi[0] - p) / (hi[0] - lo[0]);
    double xs[5];
    oracle_micro_xs(c, n, k, p, xs);
    for (int ch = 0; ch < 5; ch++) {
      A[ch] += fabs(xs[ch] * conc);
      S[ch] += conc * (fabs(hi[1 + ch]) + fabs(f) * (fabs(hi[1 + ch]) + fabs(lo[1 + ch])));
    }
  }
}

/* R12: v = 1 + argmax_c M_c with max initialised to -1.0, strict '>', so the
 * first of equal maxima wins and all M_c <= -1 gives v = 1.             */
int oracle_verify(const double M[5]) {
  double mx = -1.0;
  int idx = 0;
  for (int ch = 0; ch < 5; ch++) {
    if (M[ch] > mx) {
      mx = M[ch];
      idx = ch;
    }
  }
  return idx + 1;
}

void oracle_lookup(const oracle_ctx* c, uint64_t id, int mode, double* p, int32_t* mat,
                   int64_t* grid_index, double M[5], int32_t* v) {
  double pe;
  int32_t m;
  double Ml[5];
  oracle_sample(c->lookup_seed, id, &pe, &m);
  if (mode & ORACLE_F32)
    oracle_macro_xs_f32(c, pe, m, mode & 0xF, Ml, grid_index);
  else
    oracle_macro_xs(c, pe, m, mode, Ml, grid_index);
  if (p) *p = pe;
  if (mat) *mat = m;
  if (M) memcpy(M, Ml, sizeof(Ml));
  if (v) *v = oracle_verify(Ml);
}

/* ---------------------------------------------------------------- runs -- */
typedef struct {
  const oracle_ctx* c;
  uint64_t first, begin, end;
  int mode;
  const double* in_p;
  const int32_t* in_mat;
  double* p;
  int32_t* mat;
  int64_t* gidx;
  double* M;
  int32_t* v;
  uint64_t sum;
} run_arg;

static void* run_range(void* va) {
  run_arg* a = (run_arg*)va;
  uint64_t s = 0;
  const int grid_mode = a->mode & 0xF;
  const int f32 = (a->mode & ORACLE_F32) != 0;
  for (uint64_t i = a->begin; i < a->end; i++) {
    double pe, Ml[5];
    int32_t m;
    int64_t gi;
    if (a->in_p) {
      pe = a->in_p[i];
      m = a->in_mat[i];
    } else {
      oracle_sample(a->c->lookup_seed, a->first + i, &pe, &m);
    }
    int vv;
    if (a->mode & (ORACLE_SCALE_A | ORACLE_SCALE_S)) {
      /* M receives an error scale instead of M (test infrastructure) */
      double As[5], Ss[5];
      oracle_macro_scales(a->c, pe, m, As, Ss);
      memcpy(Ml, (a->mode & ORACLE_SCALE_A) ? As : Ss, sizeof(Ml));
      gi = -1;
      vv = 0;
    } else {
      if (f32)
        oracle_macro_xs_f32(a->c, pe, m, grid_mode, Ml, &gi);
      else
        oracle_macro_xs(a->c, pe, m, grid_mode, Ml, &gi);
      vv = oracle_verify(Ml);
    }
    s += (uint64_t)vv;
    if (a->p) a->p[i] = pe;
    if (a->mat) a->mat[i] = m;
    if (a->gidx) a->gidx[i] = gi;
    if (a->M) memcpy(a->M + 5 * i, Ml, sizeof(Ml));
    if (a->v) a->v[i] = vv;
  }
  a->sum = s;
  return NULL;
}

static uint64_t run_common(const oracle_ctx* c, uint64_t first, uint64_t count, int mode,
                           int nthreads, const double* in_p, const int32_t* in_mat, double* p,
                           int32_t* mat, int64_t* gidx, double* M, int32_t* v) {
  if (nthreads < 1) nthreads = 1;
  if ((uint64_t)nthreads > count && count > 0) nthreads = (int)count;
  if (count == 0) return 0;
  run_arg* args = (run_arg*)calloc((size_t)nthreads, sizeof(run_arg));
  pthread_t* th = (pthread_t*)calloc((size_t)nthreads, sizeof(pthread_t));
  for (int t = 0; t < nthreads; t++) {
    args[t].c = c;
    args[t].first = first;
    args[t].begin = count * (uint64_t)t / (uint64_t)nthreads;
    args[t].end = count * (uint64_t)(t + 1) / (uint64_t)nthreads;
    args[t].mode = mode;
    args[t].in_p = in_p;
    args[t].in_mat = in_mat;
    args[t].p = p;
    args[t].mat = mat;
    args[t].gidx = gidx;
    args[t].M = M;
    args[t].v = v;
    if (t > 0) pthread_create(&th[t], NULL, run_range, &args[t]);
  }
  run_range(&args[0]);
  uint64_t S = args[0].sum;
  for (int t = 1; t < nthreads; t++) {
    pthread_join(th[t], NULL);
    S += args[t].sum;
  }
  free(args);
  free(th);
  return S;
}

uint64_t oracle_run(const oracle_ctx* c, uint64_t first, uint64_t count, int mode, int nthreads,
                    double* p, int32_t* mat, int64_t* grid_index, double* M, int32_t* v) {
  return run_common(c, first, count, mode, nthreads, NULL, NULL, p, mat, grid_index, M, v);
}

uint64_t oracle_run_explicit(const oracle_ctx* c, const double* p, const int32_t* mat,
                             uint64_t count, int mode, int nthreads, double* M, int32_t* v) {
  return run_common(c, 0, count, mode, nthreads, p, mat, NULL, NULL, NULL, M, v);
}

uint64_t oracle_hash_finalize(uint64_t S) { return S % 999983ULL; }

/* R6 by definition, rows [e0, e1) of IG: IG[e][n] = clamp(ub(E_n, U[e]) - 1,
 * 0, N-2).  ub(E_n, q) = #{x in E_n : x <= q} is non-decreasing in q and U is
 * sorted, so row e's count continues from row e-1's (table parity at scale;
 * test infrastructure).  out is [e1 - e0][I].                               */
void oracle_index_grid_rows(const oracle_ctx* c, int64_t e0, int64_t e1, int32_t* out) {
  for (int32_t n = 0; n < c->I; n++) {
    const double* E = c->grid + (int64_t)n * c->N * 6;
    int64_t u = e0 < e1 ? ub_nuclide(c->grid, c->N, n, c->U[e0]) : 0;
    for (int64_t e = e0; e < e1; e++) {
      while (u < c->N && E[u * 6] <= c->U[e]) u++;
      out[(e - e0) * c->I + n] = (int32_t)clamp64(u - 1, 0, c->N - 2);
    }
  }
}

/* R7: the whole hash grid HG[b][n] = k_n(b du), out is [B][I]. */
void oracle_hash_grid(const oracle_ctx* c, int32_t* out) {
  for (int64_t b = 0; b < c->B; b++)
    for (int32_t n = 0; n < c->I; n++) out[b * c->I + n] = oracle_hash_entry(c, b, n);
}

/* ------------------------------------------------- history mode (R19) --
 * XSBench's other driver ("-m history"; PAPER.md:835 names the event driver
 * the paper runs): particle q carries one stream
 * of the lookup LCG through `lookups` chained lookups.  In step order
 * (R19):
 *   s = FF(lookup_seed, 10 * lookups * q)      (2 draws per lookup + up to 5
 *                                               extra, inside 10 per lookup)
 *   p = draw(s); mat = pick_mat(draw(s))        (R2, R3)
 *   for i in 0 .. lookups-1:
 *     M = macro_xs(p, mat)                      (R5-R11)
 *     v = verify(M); S += v                     (R12)
 *     n = #{c : M_c > 1.0}; s = FF(s, n)        (the chain's data dependence)
 *     p = draw(s); mat = pick_mat(draw(s))
 * Per-lookup arrays are indexed [q * lookups + i] (relative to the first
 * particle of the call). */
typedef struct {
  const oracle_ctx* c;
  uint64_t first, begin, end;
  int32_t lookups;
  int mode;
  double* p;
  int32_t* mat;
  double* M;
  int32_t* v;
  uint64_t sum;
} hist_arg;

/* one draw: s <- LCG(s), return s / 2^63 (R2) */
static double draw(uint64_t* s) {
  *s = oracle_lcg_step(*s);
  return oracle_lcg_to_double(*s);
}

static void* hist_range(void* va) {
  hist_arg* a = (hist_arg*)va;
  uint64_t S = 0;
  const int grid_mode = a->mode & 0xF;
  const int f32 = (a->mode & ORACLE_F32) != 0;
  for (uint64_t q = a->begin; q < a->end; q++) {
    const uint64_t part = a->first + q;
    uint64_t s = oracle_fast_forward(a->c->lookup_seed, 10ULL * (uint64_t)a->lookups * part);
    double pe = draw(&s);
    int32_t m = oracle_pick_mat(draw(&s));
    for (int32_t i = 0; i < a->lookups; i++) {
      double Ml[5];
      int64_t gi;
      if (f32)
        oracle_macro_xs_f32(a->c, pe, m, grid_mode, Ml, &gi);
      else
        oracle_macro_xs(a->c, pe, m, grid_mode, Ml, &gi);
      const int vv = oracle_verify(Ml);
      S += (uint64_t)vv;
      const uint64_t o = q * (uint64_t)a->lookups + (uint64_t)i;
      if (a->p) a->p[o] = pe;
      if (a->mat) a->mat[o] = m;
      if (a->M) memcpy(a->M + 5 * o, Ml, sizeof(Ml));
      if (a->v) a->v[o] = vv;
      uint64_t n_forward = 0;
      for (int c = 0; c < 5; c++)
        if (Ml[c] > 1.0) n_forward++;
      if (n_forward > 0) s = oracle_fast_forward(s, n_forward);
      pe = draw(&s);
      m = oracle_pick_mat(draw(&s));
    }
  }
  a->sum = S;
  return NULL;
}

uint64_t oracle_run_history(const oracle_ctx* c, uint64_t first_particle, uint64_t n_particles,
                            int32_t lookups, int mode, int nthreads, double* p, int32_t* mat,
                            double* M, int32_t* v) {
  if (nthreads < 1) nthreads = 1;
  if (n_particles == 0 || lookups <= 0) return 0;
  if ((uint64_t)nthreads > n_particles) nthreads = (int)n_particles;
  hist_arg* args = (hist_arg*)calloc((size_t)nthreads, sizeof(hist_arg));
  pthread_t* th = (pthread_t*)calloc((size_t)nthreads, sizeof(pthread_t));
  for (int t = 0; t < nthreads; t++) {
    args[t].c = c;
    args[t].first = first_particle;
    args[t].begin = n_particles * (uint64_t)t / (uint64_t)nthreads;
    args[t].end = n_particles * (uint64_t)(t + 1) / (uint64_t)nthreads;
    args[t].lookups = lookups;
    args[t].mode = mode;
    args[t].p = p;
    args[t].mat = mat;
    args[t].M = M;
    args[t].v = v;
    if (t > 0) pthread_create(&th[t], NULL, hist_range, &args[t]);
  }
  hist_range(&args[0]);
  uint64_t S = args[0].sum;
  for (int t = 1; t < nthreads; t++) {
    pthread_join(th[t], NULL);
    S += args[t].sum;
  }
  free(args);
  free(th);
  return S;
}
