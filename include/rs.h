/*
 * rs.h — C-ABI of the RSBench event-based multipole macroscopic cross-section
 * lookup in libxs.so ("RSBench event mode (multipole
 * XS, compute-bound)"; RSBench "is also a proxy
 * application for the OpenMC project ... offering a compute-bound
 * implementation").  The arithmetic follows DESIGN.md readings R20-R27
 * (the public RSBench v13 event kernel, recalled; PAPER.md gives none of it).
 *
 * One lookup:
 *   R1  sample energy E and material m exactly as XSBench does (xs.h A1)
 *   R2  (RS_FLAG_SORT) order the batch by (material, energy bin)
 *   R3  per nuclide n of m: window w = (int)(E / (1/n_windows[n]))
 *   R4  phase factors f_l = exp(-2i phi_l), phi_l the hard-sphere phase of
 *       K0RS[n][l] sqrt(E), l = 0..3
 *   R5  sigma = E * (T, A, F)_w, then over the window's poles
 *       start <= i < end: W = fast_nuclear_W((E - EA_i)/2) (the Abrarov
 *       Faddeeva approximation), sigT += Re(RT W f_l), sigA += Re(RA W),
 *       sigF += Re(RF W); sigE = sigT - sigA
 *   R6  M_c += micro_c * conc_j over the material's nuclides (list order)
 *   R7  v = 1 + argmax_c M_c (max from -DBL_MAX, strict >); vsum += {v, 1};
 *       the caller all-reduces vsum; hash = sum mod 999983 (xs_hash_finalize)
 *
 * Conventions: those of xs.h (status codes xs_status, thread-local message
 * from xs_last_error(), device pointers owned by the caller and kept alive
 * until the stream work completes, asynchronous on `cuda_stream`, results
 * depend only on (data, global lookup id), no CPU fallback).  Precision:
 * binary64 throughout; the Abrarov series keeps the oracle's operation
 * order with products and sums contracted into FMAs and divisions within
 * ~1 ulp, sqrt is IEEE,
 * e^{12iZ} and the phase factors use algebraically equal forms (angle
 * addition with init-time pole factors, R29; no atan, R30) and
 * sin/cos are CUDA's, so macro XS agree with the CPU oracle to ~1e-13
 * relative rather than bit for bit (R28; the tests require <= 1e-11 of
 * 1 + |M|); energies, materials and the verification sum are exact.
 */
#ifndef RS_H
#define RS_H
#include <stddef.h>
#include <stdint.h>

#include "xs.h"

#ifdef __cplusplus
extern "C" {
#endif

#define RS_ABI_VERSION 1u

/* Synthetic RSBench problem, regenerated on the host from seeds by the
 * shared input generator (gen/rs_gen.h; R20).  RSBench defaults:
 * 355 nuclides (large; 68 = small), 1000 poles and 100 windows per nuclide
 * on average, numL 4, doppler 1, seed 42, lookup seed 1070. */
typedef struct {
  uint32_t abi_version;  /* = RS_ABI_VERSION                                    */
  int32_t n_nuclides;    /* I >= 1 (material_rule 0 requires 68 or 355)         */
  int32_t avg_n_poles;   /* >= 1                                                */
  int32_t avg_n_windows; /* >= 1                                                */
  int32_t numL;          /* must be 4 (R4 defines four phase factors)           */
  int32_t material_rule; /* 0 = XSBench/RSBench H-M tables, 1 = ids mod I       */
  int32_t doppler;       /* 1 = Faddeeva (default), 0 = the non-doppler kernel   */
  uint64_t seed;         /* input draws (42)                                    */
  uint64_t lookup_seed;  /* lookup stream (1070)                                */
} rs_spec;

typedef struct rs_data rs_data; /* opaque: one replica on one device */

/* Outputs of a batch; DEVICE pointers owned by the caller, each NULL or
 * sized [count] (macro_xs [count][4] = sigT, sigA, sigF, sigE), indexed by
 * the lookup's position id - first_id.  vsum (uint64[2], {sum v, count}) is
 * required and ACCUMULATED (+=). */
typedef struct {
  double* macro_xs;
  int32_t* mat;
  double* energy;
  uint64_t* vsum;
} rs_outputs;

#define RS_FLAG_SORT 0x1u     /* R2: bucket by material and energy before R3-R7 */
#define RS_FLAG_HOST_IO 0x2u  /* rs_lookup_explicit: energy, mat and the outputs
                                 are HOST pointers (pinned for speed); inputs
                                 are staged in the workspace and the call
                                 synchronizes the stream before returning */
#define RS_FLAG_BASELINE 0x4u /* one thread per lookup in id order, no bucketing
                                 (RSBench's CUDA kernel shape; comparison only) */

/* Generates the problem (host, gen/rs_gen.h), uploads it to `device` on
 * `cuda_stream` and synchronizes.  Errors: XS_ERR_INVALID_ARG (bad spec or
 * abi_version), XS_ERR_UNSUPPORTED (device not sm_100, numL != 4),
 * XS_ERR_OUT_OF_MEMORY, XS_ERR_CUDA.  *out is set only on success. */
xs_status rs_init(const rs_spec* spec, int device, void* cuda_stream, rs_data** out);

/* Bytes of device workspace rs_lookup_batch needs for `count` lookups with
 * `flags` (0 when no workspace is needed). */
xs_status rs_workspace_size(const rs_data* d, uint64_t count, uint32_t flags, size_t* bytes);

/* Lookups with global ids [first_id, first_id + count), count < 2^31, on
 * `cuda_stream` (asynchronous).  `workspace` is a device buffer of at least
 * rs_workspace_size() bytes (may be NULL if that is 0).  count == 0 is a
 * no-op.  Errors: XS_ERR_INVALID_ARG (NULL data/outputs/vsum, count too
 * large, workspace too small, unknown flags), XS_ERR_CUDA (launch). */
xs_status rs_lookup_batch(rs_data* d, uint64_t first_id, uint64_t count, uint32_t flags,
                          const rs_outputs* out, void* workspace, size_t workspace_bytes,
                          void* cuda_stream);

/* R2-R7 for caller-given lookups: energy[count] (binary64) and mat[count]
 * (material ids as bytes), DEVICE pointers, or HOST pointers with
 * RS_FLAG_HOST_IO (then `out` holds host pointers too and only vsum and
 * macro_xs may be requested: XS_ERR_UNSUPPORTED otherwise).  A lookup with
 * mat >= 12 or an energy outside [0, 1] (R22's window rule is defined there)
 * is skipped: not counted in vsum, macro_xs = NaN.  Results of valid lookups
 * equal those of the sampled lookup with the same (energy, material).
 * flags: RS_FLAG_SORT, RS_FLAG_BASELINE, RS_FLAG_HOST_IO; workspace as
 * rs_workspace_size(count, flags).  Errors as rs_lookup_batch. */
xs_status rs_lookup_explicit(rs_data* d, const double* energy, const uint8_t* mat, uint64_t count,
                             uint32_t flags, const rs_outputs* out, void* workspace,
                             size_t workspace_bytes, void* cuda_stream);

/* Instrumentation (not part of a lookup): work[0] += the number of
 * (lookup, nuclide) evaluations and work[1] += the number of pole terms R5
 * evaluates for lookup ids [first_id, first_id + count) — the units of the
 * roofline count.  `work` is a DEVICE uint64[2]; async. */
xs_status rs_work_count(const rs_data* d, uint64_t first_id, uint64_t count, uint64_t* work,
                        void* cuda_stream);

/* Tuning knob: "variant" selects the lookup kernel's launch configuration
 * (0 = 256 threads x 2 blocks/SM, default; 1 = 256 x 3; 2 = 128 x 5;
 * 3 = 128 x 4; 4 = 256 x 1; 5 = 192 x 2).  Results do not depend on it.  XS_ERR_INVALID_ARG for an
 * unknown name or value. */
xs_status rs_set_param(rs_data* d, const char* name, int64_t value);

/* Kernels launched by rs_lookup_batch so far (instrumentation). */
uint64_t rs_launch_count(const rs_data* d);

/* Bytes of device memory the problem tables occupy. */
uint64_t rs_device_bytes(const rs_data* d);

/* Frees the device tables (synchronizes the device first).  NULL is a no-op. */
void rs_free(rs_data* d);

#ifdef __cplusplus
}
#endif
#endif
