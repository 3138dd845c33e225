/*
 * xs_gen.h — seeded synthetic INPUT generator (the XSBench problem data).
 *
 * This module is the one piece of code that both the CUDA product path
 * (paper_conf_sc_tianscd23_b200/csrc, via xs_init_grid) and the CPU oracle
 * (oracle/) call.  It produces only the *inputs* of the method: the
 * per-nuclide energy/XS tables, the material composition lists and the
 * nuclide concentrations.  It holds none of the method's arithmetic — no
 * energy/material sampling, no unionized/hash grid, no search, no
 * interpolation, no accumulation, no verification.  Each side implements
 * those on its own.
 *
 * What is generated (the paper only names the workload,
 * PAPER.md:835 "XSBench ... -m event", "continuous energy
 * macroscopic neutron cross-section lookup"; the data recipe follows the
 * public XSBench v20 conventions):
 *
 *   RNG      s <- (a*s + c) mod 2^63, a = 2806196910506780709, c = 1;
 *            a draw is (double)s / 2^63 (round to nearest).
 *   grid     for g = 0 .. I*N-1 (nuclide-major) draw E, σt, σs, σa, σf, νσf
 *            from grid_seed, then sort each nuclide's N records by E.
 *            Energies must be strictly increasing per nuclide; a duplicate
 *            makes the call fail with XSGEN_ERR_DUP_ENERGY.
 *   mats     rule 0: XSBench Hoogenboom-Martin tables (I must be 68 or 355);
 *            rule 1: the large tables' ids taken mod I, duplicates dropped
 *            keeping the first occurrence (used by "tiny").
 *   concs    concs[m][j] = consecutive draws from conc_seed, m = 0..11,
 *            j = 0..num_nucs[m]-1 (row stride max_num_nucs, padding 0.0).
 *
 * Layout (all host memory owned by the caller):
 *   grid   double[I][N][6]  (E, total, elastic, absorption, fission, nu-fission)
 *   mats   int32[12][max_num_nucs], concs double[12][max_num_nucs]
 */
#ifndef XS_GEN_H
#define XS_GEN_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define XSGEN_N_MATS 12

enum {
  XSGEN_OK = 0,
  XSGEN_ERR_INVALID_ARG = 1,   /* I < 1, N < 2, unknown rule, rule 0 with I not in {68,355} */
  XSGEN_ERR_DUP_ENERGY = 2     /* two equal energies inside one nuclide's grid */
};

/* num_nucs[12] for (I, rule). */
int xsgen_num_nucs(int32_t n_isotopes, int32_t material_rule, int32_t num_nucs[XSGEN_N_MATS]);

/* max over num_nucs (the row stride of mats/concs), or -1 on bad args. */
int32_t xsgen_max_num_nucs(int32_t n_isotopes, int32_t material_rule);

/* mats[12][max_num_nucs]; unused slots are set to -1. */
int xsgen_mats(int32_t n_isotopes, int32_t material_rule, int32_t max_num_nucs, int32_t* mats);

/* concs[12][max_num_nucs]; unused slots are set to 0.0. */
int xsgen_concs(uint64_t conc_seed, const int32_t num_nucs[XSGEN_N_MATS], int32_t max_num_nucs,
                double* concs);

/* grid[I][N][6]; nthreads <= 0 means hardware concurrency.  Deterministic
 * (independent of nthreads). */
int xsgen_nuclide_grid(int32_t n_isotopes, int64_t n_gridpoints, uint64_t grid_seed,
                       double* grid, int nthreads);

#ifdef __cplusplus
}
#endif
#endif
