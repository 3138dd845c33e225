/*
 * rs_oracle.h — CPU ORACLE for the RSBench event-based multipole
 * macroscopic cross-section lookup (PAPER.md:929-937:
 * RSBench, "also a proxy application for the OpenMC project ... a
 * compute-bound implementation").  TEST INFRASTRUCTURE ONLY: only tests/,
 * __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference leg
 * may load or call this.  The product path never links or imports it; the
 * only shared module is the seeded input generator gen/rs_gen.h.
 *
 * Plain C, fp64, serial per lookup, -O2 -ffp-contract=off, libm sqrt, sin,
 * cos, atan.  PAPER.md says nothing about RSBench's arithmetic; every step
 * follows the recalled public RSBench v13 event kernel in its operation
 * order, as stated by the readings R20-R27 in DESIGN.md:
 *   R21 sampling   = XSBench's (oracle_sample: E = draw, mat = pick(draw))
 *   R22 window     w = (int)(E / (1.0 / n_windows)), w == n_windows -> w-1
 *   R23 phase      phi_l = K0RS[n][l]*sqrt(E); l=1: phi -= -atan(phi);
 *                  l=2: phi -= atan(3phi/(3-phi^2)); l=3: phi -= atan(phi
 *                  (15-phi^2)/(15-6phi^2)); phi *= 2; factor_l = (cos phi,
 *                  -sin phi)
 *   R24 Faddeeva   fast_nuclear_W: Abrarov series, N = 10, tau_m = 12 for
 *                  |Z| < 6 (exp via fast_exp = (1 + x/4096)^4096 by 12
 *                  squarings), else the 3-term asymptotic expansion
 *   R25 micro      doppler: sigT = E*T, sigA = E*A, sigF = E*F, then for
 *                  poles start <= i < end (end exclusive): Z = (E - EA)*0.5,
 *                  W = fast_nuclear_W(Z), sigT += Re(RT*(W*factor_l)),
 *                  sigA += Re(RA*W), sigF += Re(RF*W); sigE = sigT - sigA
 *                  non-doppler: CDUM = (i / (EA - sqrt E)) / E replaces W
 *   R26 macro      M_c += micro_c * conc_j, j in list order, M from +0.0
 *   R27 verify     max = -DBL_MAX, strict > over c = 0..3, v = idx + 1;
 *                  hash as XSBench (R13)
 *
 * Pins (tests/test_oracle_rs.py): fast_exp against exp with its closed-form
 * relative error; the Abrarov constants against their closed forms; W
 * against scipy.special.wofz (the Faddeeva function) within the series'
 * error; the phase factors against hard-sphere phase shifts from spherical
 * Bessel functions; zero-pole windows against sigma = E*coefficient; the
 * non-doppler pole term against its closed form; sampling, sums and shard
 * invariance.  See DESIGN.md "Oracle pins".
 */
#ifndef RS_ORACLE_H
#define RS_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct rs_oracle_ctx rs_oracle_ctx;

/* ---- building blocks (exposed for the pins) ---- */
double rs_oracle_fast_exp(double x);
void   rs_oracle_fast_cexp(double zr, double zi, double* outr, double* outi);
void   rs_oracle_faddeeva(double zr, double zi, double* wr, double* wi);
/* the two branches of fast_nuclear_W: the Abrarov series with the
 * exponential e = e^{i 12 z} given, and the 3-term asymptotic expansion */
void   rs_oracle_abrarov(double zr, double zi, double er, double ei, double* wr, double* wi);
void   rs_oracle_asymptotic(double zr, double zi, double* wr, double* wi);
/* the printed constants of the series (a_n, (-1)^n, (n pi)^2, tau^2/sqrt(pi)) */
void   rs_oracle_abrarov_constants(double an[10], double neg_1n[10], double denom_left[10],
                                   double* prefactor);
/* the four factors (cos 2phi_l, -sin 2phi_l) for K0RS values k0[l], l < 4 */
void   rs_oracle_sigT_factors(const double* k0, double E, double fr[4], double fi[4]);

rs_oracle_ctx* rs_oracle_create(int32_t n_nuclides, int32_t avg_n_poles, int32_t avg_n_windows,
                                int32_t numL, int32_t material_rule, uint64_t seed,
                                uint64_t lookup_seed, int32_t doppler, int* err);
void rs_oracle_free(rs_oracle_ctx* c);

int32_t rs_oracle_n_nuclides(const rs_oracle_ctx* c);
int32_t rs_oracle_max_num_nucs(const rs_oracle_ctx* c);
int32_t rs_oracle_max_poles(const rs_oracle_ctx* c);
int32_t rs_oracle_max_windows(const rs_oracle_ctx* c);
const int32_t* rs_oracle_num_nucs(const rs_oracle_ctx* c);
const int32_t* rs_oracle_mats(const rs_oracle_ctx* c);
const double*  rs_oracle_concs(const rs_oracle_ctx* c);
const int32_t* rs_oracle_n_poles(const rs_oracle_ctx* c);
const int32_t* rs_oracle_n_windows(const rs_oracle_ctx* c);
double*        rs_oracle_poles(rs_oracle_ctx* c);    /* [I][P][8] (writable for pins) */
int32_t*       rs_oracle_l_value(rs_oracle_ctx* c);  /* [I][P] */
double*        rs_oracle_windows(rs_oracle_ctx* c);  /* [I][W][3] */
int32_t*       rs_oracle_wrange(rs_oracle_ctx* c);   /* [I][W][2] */
double*        rs_oracle_k0rs(rs_oracle_ctx* c);     /* [I][numL] */

int32_t rs_oracle_window(const rs_oracle_ctx* c, int32_t nuc, double E);          /* R22 */
void rs_oracle_micro_xs(const rs_oracle_ctx* c, int32_t nuc, double E, double micro[4]);
void rs_oracle_macro_xs(const rs_oracle_ctx* c, double E, int32_t mat, double M[4]);
int  rs_oracle_verify(const double M[4]);                                          /* R27 */
void rs_oracle_lookup(const rs_oracle_ctx* c, uint64_t id, double* E, int32_t* mat, double M[4],
                      int32_t* v);
/* Lookups [first, first+count) on nthreads threads; returns sum of v.
 * Per-lookup arrays (E[count], mat[count], M[count][4], v[count]) may be NULL. */
uint64_t rs_oracle_run(const rs_oracle_ctx* c, uint64_t first, uint64_t count, int nthreads,
                       double* E, int32_t* mat, double* M, int32_t* v);

#ifdef __cplusplus
}
#endif
#endif
