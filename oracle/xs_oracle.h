/*
 * xs_oracle.h — CPU ORACLE for the XSBench event-based macroscopic
 * cross-section lookup.  TEST INFRASTRUCTURE ONLY: only tests/,
 * __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference leg
 * may load or call this.  The product path (paper_conf_sc_tianscd23_b200/)
 * never links or imports it and shares no code with it; the only shared
 * module is the seeded input generator gen/xs_gen.h.
 *
 * Plain, serial-per-lookup, fp64 (plus the fp32 variant of R18, selected
 * by ORACLE_F32), compiled with -O2 -ffp-contract=off (no
 * FMA contraction, no fast-math), one function per step of the method, each
 * citing the passage it follows.  PAPER.md states only what is computed
 * ("continuous energy macroscopic neutron cross-section lookup",
 * PAPER.md:911-915, XSBench "-m event", self-verified by a
 * checksum); the step definitions follow BASELINE.json
 * north_star and the readings R1..R17 listed in DESIGN.md.
 *
 * Parity pins: every function here is pinned by a `-m "not gpu"` test in
 * tests/test_oracle_*.py.  None is unpinned.
 */
#ifndef XS_ORACLE_H
#define XS_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

enum { ORACLE_UNIONIZED = 0, ORACLE_NUCLIDE = 1, ORACLE_HASH = 2 };
/* OR'ed into `mode` of oracle_lookup / oracle_run*: the fp32 variant (R18) */
enum { ORACLE_F32 = 0x10 };
/* run modes that return an error scale in M instead of M (oracle_macro_scales) */
enum { ORACLE_SCALE_A = 0x20, ORACLE_SCALE_S = 0x40 };

typedef struct oracle_ctx oracle_ctx;

/* ---- RNG and sampling (north_star "samples an energy E and a material m";
 *      DESIGN.md R2/R3) ---- */
uint64_t oracle_lcg_step(uint64_t s);                  /* (a s + c) mod 2^63 */
double   oracle_lcg_to_double(uint64_t s);             /* s / 2^63 */
uint64_t oracle_fast_forward(uint64_t s, uint64_t n);  /* LCG^n(s) in O(log n) */
void     oracle_thresholds(double T[12]);              /* T[m], m=1..11; T[0]=0 */
int32_t  oracle_pick_mat(double roll);
void     oracle_sample(uint64_t lookup_seed, uint64_t id, double* p, int32_t* mat);

/* ---- Search (north_star "binary-searches the unionized (or hash) grid";
 *      DESIGN.md R5-R9) ---- */
int64_t oracle_grid_search(const double* A, int64_t lo, int64_t hi, double q);
int64_t oracle_upper_bound(const double* A, int64_t n, double q);   /* #{x <= q} */

/* ---- Context: the problem data plus the oracle's own acceleration tables */
oracle_ctx* oracle_create_spec(int32_t n_isotopes, int64_t n_gridpoints, uint64_t grid_seed,
                               uint64_t conc_seed, int32_t material_rule, uint64_t lookup_seed,
                               int32_t hash_bins, int nthreads, int* err);
oracle_ctx* oracle_create_arrays(int32_t n_isotopes, int64_t n_gridpoints, const double* grid,
                                 int32_t n_mats, int32_t max_num_nucs, const int32_t* num_nucs,
                                 const int32_t* mats, const double* concs, uint64_t lookup_seed,
                                 int32_t hash_bins, int* err);
void oracle_free(oracle_ctx* c);

int32_t oracle_n_isotopes(const oracle_ctx* c);
int64_t oracle_n_gridpoints(const oracle_ctx* c);
int32_t oracle_n_mats(const oracle_ctx* c);
int32_t oracle_max_num_nucs(const oracle_ctx* c);
int64_t oracle_union_len(const oracle_ctx* c);
const double*  oracle_grid(const oracle_ctx* c);        /* [I][N][6] */
const double*  oracle_union(const oracle_ctx* c);       /* [NU] */
const int32_t* oracle_num_nucs(const oracle_ctx* c);
const int32_t* oracle_mats(const oracle_ctx* c);
const double*  oracle_concs(const oracle_ctx* c);

/* k_n(p) = clamp(ub(E_n, p) - 1, 0, N-2): the plain definition (R5). */
int64_t oracle_nuclide_bracket(const oracle_ctx* c, int32_t n, double p);
/* u = clamp(ub(U, p) - 1, 0, NU-2) (R6). */
int64_t oracle_union_index(const oracle_ctx* c, double p);
/* IG[e][n] = clamp(ub(E_n, U[e]) - 1, 0, N-2) (R6). */
int32_t oracle_index_grid_entry(const oracle_ctx* c, int64_t e, int32_t n);
/* XSBench's incremental construction of the whole IG (R6, pin P5). */
int     oracle_index_grid_sweep(const oracle_ctx* c, int32_t* out /* [NU][I] */);
/* b = min(trunc(p / du), B-1), du = 1/B (R8, R9). */
int64_t oracle_hash_bin(const oracle_ctx* c, double p);
/* HG[b][n] = clamp(ub(E_n, b du) - 1, 0, N-2) (R7). */
int32_t oracle_hash_entry(const oracle_ctx* c, int64_t b, int32_t n);
/* XSBench's bracketed hash search (R7): result equals k_n(p). */
int64_t oracle_hash_bracket(const oracle_ctx* c, int64_t b, int32_t n, double p);

/* ---- Interpolate / accumulate / verify (north_star "linearly interpolates
 *      the five XS channels ... accumulates the concentration-weighted
 *      macroscopic XS"; checksum PAPER.md:923-927; R10-R12) ---- */
void oracle_micro_xs(const oracle_ctx* c, int32_t n, int64_t k, double p, double xs[5]);
void oracle_macro_xs(const oracle_ctx* c, double p, int32_t mat, int mode, double M[5],
                     int64_t* grid_index);
int  oracle_verify(const double M[5]);
/* R18: the fp32 variant (binary64 search and f, binary32 channels,
 * concentrations and accumulation); M is the binary32 result widened. */
void oracle_micro_xs_f32(const oracle_ctx* c, int32_t n, int64_t k, double p, float xs[5]);
void oracle_macro_xs_f32(const oracle_ctx* c, double p, int32_t mat, int mode, double M[5],
                         int64_t* grid_index);

/* One lookup id end to end; any output pointer may be NULL. */
void oracle_lookup(const oracle_ctx* c, uint64_t id, int mode, double* p, int32_t* mat,
                   int64_t* grid_index, double M[5], int32_t* v);

/* Lookups [first, first+count) on nthreads host threads over contiguous
 * ranges (R14).  Returns S = sum of v.  Per-lookup arrays may be NULL. */
uint64_t oracle_run(const oracle_ctx* c, uint64_t first, uint64_t count, int mode, int nthreads,
                    double* p, int32_t* mat, int64_t* grid_index, double* M, int32_t* v);

/* Explicit (energy, material) lookups (same per-lookup function, no sampling). */
uint64_t oracle_run_explicit(const oracle_ctx* c, const double* p, const int32_t* mat,
                             uint64_t count, int mode, int nthreads, double* M, int32_t* v);

/* History mode (R19): particles
 * [first_particle, first_particle + n_particles), each `lookups` chained
 * lookups; returns S = sum of v.  Per-lookup arrays (NULL allowed) are
 * indexed [q * lookups + i], q relative to first_particle. */
uint64_t oracle_run_history(const oracle_ctx* c, uint64_t first_particle, uint64_t n_particles,
                            int32_t lookups, int mode, int nthreads, double* p, int32_t* mat,
                            double* M, int32_t* v);

/* hash = S mod 999983, once, after the global sum (R13). */
uint64_t oracle_hash_finalize(uint64_t S);
/* error scales of the binary64 result (Q12's A_c, R18's S_c) */
void oracle_macro_scales(const oracle_ctx* c, double p, int32_t mat, double A[5], double S[5]);
/* IG rows [e0, e1) by definition (R6), [e1 - e0][I] */
void oracle_index_grid_rows(const oracle_ctx* c, int64_t e0, int64_t e1, int32_t* out);
/* the hash grid HG[b][n] (R7), [B][I] */
void oracle_hash_grid(const oracle_ctx* c, int32_t* out);

#ifdef __cplusplus
}
#endif
#endif
