/*
 * rs_gen.h — seeded synthetic INPUT generator for the RSBench problem
 * ("RSBench ... also a proxy
 * application for the OpenMC project ... a compute-bound implementation").
 *
 * Like gen/xs_gen.h this is the one module both the CUDA product path
 * (rs_init, include/rs.h) and the CPU oracle (oracle/rs_oracle.c) call.  It
 * produces only the *inputs* of the multipole lookup: the material lists and
 * concentrations, the number of poles and windows per nuclide, the pole
 * parameters, the window parameters (background coefficients and the
 * contiguous pole range of each window) and the pseudo K0RS values.  It holds
 * none of the method's arithmetic (no sampling, window selection, phase
 * factors, Faddeeva evaluation, accumulation or verification).
 *
 * Recipe (PAPER.md names RSBench only; the recipe follows the public RSBench
 * v13 conventions as recalled — DESIGN.md reading R20):
 *   RNG      the 63-bit LCG of xs_gen.h; one stream from `seed` (42) feeds,
 *            in this order:
 *   concs    concs[m][j], m = 0..11, j < num_nucs[m] (H-M material tables of
 *            xs_gen.h: rule 0 needs I in {68, 355}, rule 1 = ids mod I);
 *   n_poles  every nuclide starts at 1, then avg_n_poles*I - I times
 *            n_poles[r mod I]++ with r the raw 63-bit LCG state;
 *   n_windows the same with avg_n_windows;
 *   poles    for n, for j < n_poles[n]: EA.re, EA.im, RT.re, RT.im, RA.re,
 *            RA.im, RF.re, RF.im (draws), then l = r mod numL (raw state);
 *   windows  for n: space = n_poles/n_windows, rem = n_poles - space*n_windows;
 *            for w < n_windows[n]: T, A, F (draws); start = ctr,
 *            end = ctr + space - 1, ctr += space; if w < rem: ctr++, end++;
 *   K0RS     for n, for l < numL: one draw.
 *
 * Layout (host memory owned by the caller; P = max n_poles, W = max n_windows):
 *   poles    double[I][P][8]  (EA.re, EA.im, RT.re, RT.im, RA.re, RA.im,
 *                              RF.re, RF.im), unused slots 0
 *   l_value  int32[I][P]
 *   windows  double[I][W][3]  (T, A, F), unused slots 0
 *   wrange   int32[I][W][2]   (start, end)
 *   k0rs     double[I][numL]
 */
#ifndef RS_GEN_H
#define RS_GEN_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

enum { RSGEN_OK = 0, RSGEN_ERR_INVALID_ARG = 1 };

typedef struct {
  int32_t n_nuclides;     /* I */
  int32_t avg_n_poles;    /* RSBench default 1000 */
  int32_t avg_n_windows;  /* RSBench default 100 */
  int32_t numL;           /* RSBench default 4 */
  int32_t material_rule;  /* 0 = H-M tables (I in {68, 355}), 1 = ids mod I */
  uint64_t seed;          /* RSBench INITIALIZATION_SEED 42 */
} rsgen_spec;

/* Pass 1: counts.  Fills n_poles[I], n_windows[I] (caller arrays) and the
 * maxima; needs no other memory.  Deterministic. */
int rsgen_counts(const rsgen_spec* spec, int32_t* n_poles, int32_t* n_windows,
                 int32_t* max_poles, int32_t* max_windows);

/* Pass 2: everything (re-derives the counts).  concs has stride max_num_nucs
 * (xsgen_max_num_nucs(I, rule)); every pointer must be non-NULL. */
int rsgen_data(const rsgen_spec* spec, int32_t max_num_nucs, int32_t max_poles,
               int32_t max_windows, double* concs, int32_t* n_poles, int32_t* n_windows,
               double* poles, int32_t* l_value, double* windows, int32_t* wrange,
               double* k0rs);

#ifdef __cplusplus
}
#endif
#endif
