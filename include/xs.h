/*
 * xs.h — C-ABI of libxs.so, the B200-native XSBench event-based macroscopic
 * neutron cross-section (XS) lookup (the data-parallel hot path of Tian et
 * al., "OpenMP Kernel Language Extensions for Performance Portable GPU
 * Codes", SC-W 2023: XSBench "-m event"; "computing the
 * continuous energy macroscopic neutron cross-section lookup",
 * PAPER.md:911-915; self-verified by a checksum).
 *
 * One lookup (BASELINE.json north_star; DESIGN.md §1 and readings R1-R17):
 *   A1  sample energy p and material m from a counter-based LCG stream
 *   A2  (optional) sort the batch by (material, energy) — XS_FLAG_SORT
 *   A3  find p on the unionized energy grid (binary search) or hash grid
 *   A4  gather the bracket index k_n of every nuclide n in material m
 *   A5  gather the record pair (k_n, k_n+1) of each nuclide
 *   A6  interpolate the five channels (total, elastic, absorption, fission,
 *       nu-fission) linearly in energy
 *   A7  accumulate M_c += x_c * conc_j over the material's nuclides
 *   A8  verification value v = 1 + argmax_c M_c; vsum += {v, 1}
 *   A9  (caller) all-reduce vsum across ranks; hash = sum mod 999983
 *
 * Conventions (all entry points):
 *   - extern "C", plain pointers and sizes; no C++ types cross the ABI.
 *   - Every call returns xs_status; on failure xs_last_error() returns a
 *     thread-local message.  No exceptions, no abort().
 *   - "device pointer" = memory on the grid's device (e.g. a torch tensor's
 *     data_ptr()); the caller owns it and must keep it alive until the work
 *     enqueued on `cuda_stream` completes.  `cuda_stream` is a cudaStream_t
 *     (NULL = legacy default stream), e.g. torch.cuda.current_stream().
 *   - Work is enqueued asynchronously on the stream; device faults surface
 *     as XS_ERR_CUDA at the next call that synchronizes.
 *   - Results depend only on (grid, global lookup id), never on batching,
 *     sharding, sorting or launch configuration (shard = [first, first+count)).
 *   - The library owns the grid tables (freed by xs_free_grid).  One grid
 *     lives on one device; calls on one grid are ordered by the caller.
 *   - There is no CPU fallback: without a usable sm_100 device every
 *     compute entry point fails with XS_ERR_CUDA / XS_ERR_UNSUPPORTED.
 */
#ifndef XS_H
#define XS_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define XS_ABI_VERSION 1u

typedef enum {
  XS_OK = 0,
  XS_ERR_INVALID_ARG = 1,   /* NULL/inconsistent argument, bad spec, range error */
  XS_ERR_OUT_OF_MEMORY = 2, /* device or host allocation failed                 */
  XS_ERR_CUDA = 3,          /* CUDA runtime/launch error (message has details)  */
  XS_ERR_UNSUPPORTED = 4,   /* feature not available for this grid/device       */
  XS_ERR_STATE = 5,         /* call made in the wrong state (e.g. wrong device) */
  XS_ERR_DATA = 6           /* input data invalid (e.g. duplicate energies)     */
} xs_status;

/* Energy-search acceleration (north_star: "binary-searches the unionized (or
 * hash-accelerated) energy grid"; R6-R9). */
typedef enum {
  XS_GRID_UNIONIZED = 0, /* U = sorted union of all energies + index grid IG[NU][I] */
  XS_GRID_NUCLIDE = 1,   /* no acceleration: binary search per nuclide            */
  XS_GRID_HASH = 2       /* hash grid HG[B][I] over equal-width energy bins        */
} xs_grid_type;

/* Synthetic XSBench problem, regenerated from seeds by the shared input
 * generator (gen/xs_gen.h; R1).  Presets: tiny (12, 1000, rule 1),
 * small (68, 11303), large (355, 11303), XL (355, 238847); grid_seed 42,
 * conc_seed 1070^2, lookup_seed 1070. */
typedef struct {
  uint32_t abi_version;   /* = XS_ABI_VERSION                                   */
  int32_t n_isotopes;     /* I >= 1 (rule 0 requires 68 or 355)                */
  int64_t n_gridpoints;   /* N >= 2 points per nuclide                          */
  int32_t grid_type;      /* xs_grid_type                                       */
  int32_t hash_bins;      /* B >= 1, used iff grid_type == XS_GRID_HASH         */
  uint64_t grid_seed;     /* nuclide grid draws                                 */
  uint64_t conc_seed;     /* concentration draws                                */
  uint64_t lookup_seed;   /* lookup stream seed (A1)                            */
  int32_t material_rule;  /* 0 = XSBench H-M tables, 1 = ids mod I (tiny)       */
  int32_t index_layout;   /* XS_INDEX_*: unionized index-grid layout(s), 0 = auto */
} xs_grid_spec;

/* Unionized index grid layouts (same values, different memory order):
 *   ROW  IG[u][n]  (u-major, row of I ints per unionized energy): one lookup
 *        reads a contiguous row — best for unsorted batches;
 *   COL  IGT[n][u] (nuclide-major): the lookups of an energy-sorted batch
 *        read neighbouring entries of one column — best with XS_FLAG_SORT.
 * AUTO builds both when they fit comfortably in device memory (large: 2 x
 * 5.7 GB), else COL only (XL: 120 GB). */
#define XS_INDEX_AUTO 0
#define XS_INDEX_ROW 1
#define XS_INDEX_COL 2
#define XS_INDEX_BOTH 3

/* Caller-supplied nuclear data (HOST pointers, copied during init).  The
 * nuclide grid is [I][N][6] doubles (E, total, elastic, absorption, fission,
 * nu-fission) with E strictly increasing per nuclide; mats/concs are
 * [n_mats][max_num_nucs] row-major, only the first num_nucs[m] entries of
 * row m are read.  Sampled batches (xs_lookup_batch) need n_mats == 12 (the
 * XSBench material distribution); explicit lookups accept any n_mats >= 1. */
typedef struct {
  uint32_t abi_version;
  int32_t n_isotopes;
  int64_t n_gridpoints;
  const double* nuclide_grid;
  int32_t n_mats;
  int32_t max_num_nucs;
  const int32_t* num_nucs;
  const int32_t* mats;
  const double* concs;
  int32_t grid_type;
  int32_t hash_bins;
  uint64_t lookup_seed;
  int32_t index_layout;   /* XS_INDEX_* (unionized only), 0 = auto */
  int32_t reserved0;      /* must be 0 */
} xs_grid_data;

typedef struct xs_grid xs_grid; /* opaque: one replica of the tables on one device */

typedef struct {
  int32_t n_isotopes, n_mats, max_num_nucs, grid_type, hash_bins, device;
  int64_t n_gridpoints;
  int64_t n_union;        /* NU = I*N for UNIONIZED, else 0                     */
  int64_t index_grid_len; /* NU*I (UNIONIZED), B*I (HASH), 0 (NUCLIDE)          */
  uint64_t device_bytes;  /* bytes of device memory the grid holds              */
  uint64_t lookup_seed;
  int32_t index_layout;   /* layouts actually built (XS_INDEX_ROW | XS_INDEX_COL) */
  int32_t reserved0;
} xs_grid_info;

/* Per-lookup outputs, indexed by position i in the batch (lookup id
 * first_id + i).  Every pointer may be NULL except vsum.  DEVICE pointers
 * unless XS_FLAG_HOST_IO is set, in which case they are HOST pointers
 * (pageable or pinned) and the library stages them through the workspace. */
typedef struct {
  double* macro_xs;      /* [count][5]  M_c, channel order as above          */
  double* energy;        /* [count]     sampled p                            */
  int32_t* mat;          /* [count]     sampled material                     */
  int64_t* grid_index;   /* [count]     u (UNIONIZED), b (HASH), -1 (NUCLIDE) */
  int32_t* verification; /* [count]     v in 1..5 (0 for an invalid lookup)   */
  uint64_t* vsum;        /* [2]         ACCUMULATED: += {sum v, #valid}       */
} xs_outputs;

/* flags */
#define XS_FLAG_SORT 0x1u     /* A2: order the batch by (material, energy bin):
                                 one in-house counting-sort radix pass       */
#define XS_FLAG_HOST_IO 0x2u  /* inputs/outputs are host pointers               */
#define XS_FLAG_BASELINE 0x4u /* thread-per-lookup, unbucketed kernel (XSBench's
                                 CUDA baseline shape; for comparison only)     */
#define XS_FLAG_F32 0x8u      /* the fp32 variant (R18; north_star "1e-5
                                 if an fp32 variant is offered"): energies, the
                                 search and f stay binary64; channel values,
                                 concentrations and the accumulation are
                                 binary32 with fused multiply-adds.  macro_xs
                                 receives the binary32 results widened.  Not
                                 combinable with XS_FLAG_BASELINE.             */
#define XS_FLAG_MAT_U8 0x10u  /* xs_lookup_explicit: `mat` points to uint8_t[count]
                                 (a material id per byte) instead of int32_t —
                                 a quarter of the material bytes to upload    */
#define XS_FLAG_HOST_ASYNC 0x20u /* like XS_FLAG_HOST_IO (host pointers in and out),
                                 but the call does not wait: the inputs are
                                 uploaded on the library's copy stream and the
                                 outputs (vsum included) are copied back on
                                 `cuda_stream`; the caller keeps the host
                                 buffers and the workspace alive and
                                 unmodified, and synchronizes `cuda_stream`
                                 before reading outputs.  The upload of one
                                 call overlaps the lookups of the previous
                                 call when the two use different workspaces
                                 (a workspace's staging area is reused only
                                 after the call that last used it is done).
                                 Not combinable with XS_FLAG_HOST_IO.        */

/* tables for xs_get_table (element type in brackets) */
#define XS_TABLE_NUCLIDE_GRID 0 /* [double] I*N*6                               */
#define XS_TABLE_UNION_ENERGY 1 /* [double] NU                                  */
#define XS_TABLE_INDEX_GRID 2   /* [int32]  IG (NU*I) or HG (B*I), row-major     */
#define XS_TABLE_NUM_NUCS 3     /* [int32]  n_mats                              */
#define XS_TABLE_MATS 4         /* [int32]  n_mats*max_num_nucs                 */
#define XS_TABLE_CONCS 5        /* [double] n_mats*max_num_nucs                 */
#define XS_TABLE_INDEX_GRID_T 6 /* [int32]  IGT (I*NU), nuclide-major            */
#define XS_TABLE_INTERVALS 7    /* [double] I*N*14: interval table (DESIGN.md §4 K0d):
                                   entry (n, k) = {E[k+1], E[k+1] - E[k], ~1/gap, 0,
                                   (hi.c, hi.c - lo.c) x 5}; entry N-1 is zero     */
#define XS_TABLE_INTERVALS32 8  /* [double] I*N*10: fp32-variant table (K0e): {E[k+1],
                                   gap, ~1/gap, 0} then 12 floats (h_c, d_c) x 5, 0, 0 */
#define XS_TABLE_INTERVALS_U 9  /* [double] I*N*12: the unsorted gather's 96-B,
                                   32-B aligned entries (K0u): {E[k+1], gap,
                                   (hi.c, hi.c - lo.c) x 5}; entry N-1 is zero;
                                   UNSUPPORTED when the grid did not build it
                                   (built only with ample free device memory,
                                   and never for a unionized grid without the
                                   row layout, whose unsorted batches take the
                                   staged gather) */

uint32_t xs_abi_version(void);

/* Generate the problem from `spec` on the host (gen/xs_gen.h), upload it to
 * `device` and build the acceleration tables there (unionized energy sort,
 * index grid or hash grid).  Synchronizes `cuda_stream` before returning.
 * Errors: INVALID_ARG (bad spec), DATA (duplicate energy in a nuclide),
 * OUT_OF_MEMORY, CUDA.  On success *out owns all device tables. */
xs_status xs_init_grid(const xs_grid_spec* spec, int device, void* cuda_stream, xs_grid** out);

/* Same with caller-supplied nuclear data (host arrays, copied). */
xs_status xs_init_grid_data(const xs_grid_data* data, int device, void* cuda_stream,
                            xs_grid** out);

xs_status xs_grid_get_info(const xs_grid* g, xs_grid_info* info);

/* Bytes of device workspace xs_lookup_batch / xs_lookup_explicit need for a
 * batch of `count` lookups with `flags`.  Workspace must be 256-B aligned. */
xs_status xs_workspace_size(const xs_grid* g, uint64_t count, uint32_t flags, size_t* bytes);

/* A1-A8 for lookup ids [first_id, first_id + count), enqueued on the stream.
 * 0 <= count < 2^32.  vsum is accumulated (+=), so shards can share it.
 * Requires n_mats == 12 (sampling distribution).  count == 0 is a no-op. */
xs_status xs_lookup_batch(xs_grid* g, uint64_t first_id, uint64_t count, uint32_t flags,
                          const xs_outputs* out, void* workspace, size_t workspace_bytes,
                          void* cuda_stream);

/* Energy-range shard of a sampled batch (multi-GPU strong scaling; DESIGN.md
 * §6): A1 for lookup ids [first_id, first_id + count), then A2-A8 only for the
 * lookups whose energy p lies in shard `shard` of `n_shards`:
 *   b_s <= p < b_{s+1},  b_s = RN(s / n_shards) (binary64 quotient) for
 *   0 < s < n_shards, b_0 = -inf, b_{n_shards} = +inf,
 * so the shards of one batch partition it (every lookup is looked up by
 * exactly one shard) and the vsum of all shards equals xs_lookup_batch's.
 * Each shard keeps the full batch's density in energy (a rank's lookups are
 * as close together as in one big batch, unlike a contiguous id range).
 * vsum += {sum v, #lookups in the shard}; per-lookup outputs (device
 * pointers indexed by batch position) are written only for the shard's
 * lookups, the other positions are left untouched.  Requires XS_FLAG_SORT
 * (the partitioned A2), optionally XS_FLAG_F32; XS_FLAG_BASELINE and
 * XS_FLAG_HOST_IO are INVALID_ARG; a batch or variant the partitioned A2
 * cannot serve is UNSUPPORTED.  Workspace as xs_workspace_size(count, flags). */
xs_status xs_lookup_batch_shard(xs_grid* g, uint64_t first_id, uint64_t count, int32_t shard,
                                int32_t n_shards, uint32_t flags, const xs_outputs* out,
                                void* workspace, size_t workspace_bytes, void* cuda_stream);

/* A2-A8 for caller-given lookups: energy[i] (any double; outside the grid the
 * XS are extrapolated) and mat[i] (0 <= mat < n_mats; an out-of-range mat
 * gives v = 0, NaN macro_xs and is not counted in vsum[1]).  energy/mat are
 * device pointers, or host pointers with XS_FLAG_HOST_IO (then the outputs
 * are host pointers too and the call synchronizes the stream on return). */
xs_status xs_lookup_explicit(xs_grid* g, const double* energy, const int32_t* mat,
                             uint64_t count, uint32_t flags, const xs_outputs* out,
                             void* workspace, size_t workspace_bytes, void* cuda_stream);

/* History mode (XSBench "-m history"; R19; SURVEY.md §8(f)
 * NEXT-3 — the paper runs the event driver).  Particles
 * q in [first_particle, first_particle + n_particles) each carry one stream
 * of the lookup LCG through `lookups` chained lookups: s = LCG^(10 lookups q)
 * (lookup_seed), draw (p, mat); per lookup: M = A3-A8 at (p, mat), v =
 * 1 + argmax M, skip n_forward = #{c : M_c > 1.0} draws, draw the next
 * (p, mat).  Outputs (DEVICE pointers, any NULL except vsum): macro_xs
 * [n][lookups][5], energy / mat / verification [n][lookups] (lookup i of
 * particle q at q * lookups + i); grid_index must be NULL (XS_ERR_UNSUPPORTED).
 * vsum += {sum v, n_particles * lookups}.  flags: 0 or XS_FLAG_SORT (each
 * round's batch through A2).  Requires n_mats == 12, 1 <= lookups,
 * n_particles < 2^32; workspace from xs_history_workspace_size (256-B
 * aligned, caller-owned, alive until the stream passes the call).  Enqueued
 * on the stream: lookups rounds of the event pipeline plus one state-update
 * kernel each. */
xs_status xs_history_workspace_size(const xs_grid* g, uint64_t n_particles, uint32_t flags,
                                    size_t* bytes);
xs_status xs_lookup_history(xs_grid* g, uint64_t first_particle, uint64_t n_particles,
                            int32_t lookups, uint32_t flags, const xs_outputs* out,
                            void* workspace, size_t workspace_bytes, void* cuda_stream);

/* A8 alone on stored results: vsum += {sum_i (1 + argmax_c macro_xs[i][c]), count}
 * (device pointers). */
xs_status xs_verify(const xs_grid* g, const double* macro_xs, uint64_t count, uint64_t* vsum,
                    void* cuda_stream);

/* Diagnostic for A3/A4 parity: k_out[i] = bracket of nuclide nuclide[i] at
 * energy[i] found through the grid's own acceleration structure (device
 * pointers; 0 <= nuclide < I). */
xs_status xs_nuclide_index(const xs_grid* g, const double* energy, const int32_t* nuclide,
                           uint64_t count, int32_t* k_out, void* cuda_stream);

/* Synchronous copy of elements [offset, offset+count) of a device table to
 * host memory (parity checks of the device-built tables). */
xs_status xs_get_table(const xs_grid* g, int32_t table, uint64_t offset, uint64_t count,
                       void* host_dst);

/* Tuning knobs: "variant" (gather kernel: 0 = the default, chosen by batch
 * density for sorted batches and k_gather_u for unsorted ones; 1-4, 9-12,
 * 17-28, 31-36, 40-58 = the kernel shapes listed in DESIGN.md §4 and
 * lookup.cu), "blocks_per_sm"
 * (0 = occupancy calculator), "legacy_sort" (1: XS_FLAG_SORT through the
 * global-atomic bins and a permutation instead of the partitioned counting
 * sort; comparison only), "part_cbits" (coarse energy bits of the partitioned
 * sort, 6-9; 0 = the default, 7, or 8 for an energy-range shard whose coarse
 * segments would average more than two fine-pass windows; a value whose
 * tables do not fit the batch or the workspace falls back to the widest that
 * does), "shard_tiles" (energy-range shards: cap on the factor by which the
 * sort's tiles are lengthened, 1-16; 0 = the default, n/2 for a 1/n shard),
 * "fine_direct" (the sort's fine pass scatters a coarse
 * key's segment in one pass when it exceeds this many shared-memory windows,
 * else sorts it window by window; default 2), "fine_cap" (that window in
 * energies, 2048-24576; 0 = the default 24576) and "host_chunk" (XS_FLAG_HOST_IO explicit lookups upload their inputs in
 * chunks of this many lookups, overlapped with the lookups of the previous
 * chunk; default 10^7, split evenly).  INVALID_ARG for an
 * unknown name or value.  Never changes results. */
xs_status xs_set_param(xs_grid* g, const char* name, int64_t value);

/* Per-phase device timing of lookup calls, measured with CUDA events
 * recorded on the caller's stream around each phase (enable costs four
 * event records per call).  kernel_launches counts the library's own kernel
 * launches (always on). */
typedef struct {
  uint64_t calls;           /* lookup calls since the last read              */
  uint64_t kernel_launches; /* kernels those calls launched                  */
  double ms_count;          /* A1: material (and energy-bin) histogram       */
  double ms_bucket;         /* A1+A3 (+A2): sample, search, scatter to bins  */
  double ms_gather;         /* A4-A8: the gather/interpolate/verify kernel   */
  double ms_total;          /* sum of the above                              */
} xs_timing;

xs_status xs_timing_enable(xs_grid* g, int enable);
/* Waits for the recorded events, returns the sums since the previous read
 * (or enable) and resets them. */
xs_status xs_timing_read(xs_grid* g, xs_timing* out);

/* A9 epilogue: hash = global sum mod 999983 (R13). */
uint64_t xs_hash_finalize(uint64_t global_sum);

void xs_free_grid(xs_grid* g);

const char* xs_last_error(void);

#ifdef __cplusplus
}
#endif
#endif
