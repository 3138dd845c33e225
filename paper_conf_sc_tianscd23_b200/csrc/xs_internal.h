// xs_internal.h — internal (C++) interface between the C-ABI layer
// (xs_api.cu) and the kernels (grid_build.cu, lookup.cu).  Not installed.
#pragma once
#include <cuda_runtime.h>
#include <stddef.h>
#include <stdint.h>

#include "../../include/xs.h"

namespace xs {

// one lookup after A1/A3: energy, position in the batch, grid index (u or b)
struct alignas(16) LookupRec {
  double p;
  uint32_t idx;
  int32_t gidx;
};

constexpr int kMaxMats = 64;  // materials supported by the bucketed kernels
constexpr uint32_t kEnergyBins = 1u << 18;  // A2: energy bins per material
constexpr int kIvDoubles = 14;  // interval-table entry (112 B; grid_build.cu K0d)
constexpr int kIv32Doubles = 10;  // fp32-variant entry (80 B; grid_build.cu K0e)

struct DeviceGrid {
  int device = 0;
  int sm_count = 0;
  int32_t I = 0;
  int64_t N = 0;
  int32_t n_mats = 0, max_nucs = 0;
  int32_t tab_total = 0;     // sum of num_nucs (packed material table entries)
  int32_t grid_type = 0, B = 0;
  double du = 0.0;
  uint64_t lookup_seed = 0;
  int64_t NU = 0, index_len = 0;
  double* grid = nullptr;    // [I][N][6]
  double* iv = nullptr;      // [I][N][kIvDoubles] interval table (K0d), or null
  double* iv32 = nullptr;    // [I][N][kIv32Doubles] fp32-variant interval table (K0e)
  double* ivu = nullptr;     // [I][N][16] 128-B line-aligned interval table (K0u), or null
  double* U = nullptr;       // [NU]
  int32_t* UB = nullptr;     // [UBn + 1]: UB[b] = ub(U, b / UBn)  (A3 search table)
  int32_t UBn = 0;           // power of two
  int32_t* index = nullptr;  // IG [NU][I] (row layout) or HG [B][I]; null if no row IG
  int32_t* index_t = nullptr;  // IGT [I][NU] (column layout), unionized only
  int32_t index_layout = 0;    // XS_INDEX_ROW | XS_INDEX_COL actually built
  int32_t* num_nucs = nullptr;
  int32_t* mats = nullptr;   // [n_mats][max_nucs]
  double* concs = nullptr;   // [n_mats][max_nucs]
  uint64_t device_bytes = 0;
  bool dyadic63 = false;     // every grid energy is k * 2^-63 in [0, 1]
  // tuning
  int unroll = 0;          // gather variant (0 = default; see launch_gather_u)
  int blocks_per_sm = 0;   // 0 = occupancy calculator
  int legacy_sort = 0;     // 1: A2 through the global-atomic bins + permutation (comparison)
  int part_cbits = 0;      // partitioned A2 coarse energy bits (0 = default)
  int fine_direct = 2;     // k_part_fine: direct scatter above this many windows
  int fine_cap = 0;        // k_part_fine window in energies (0 = default 24576)
  int shard_tiles = 0;     // energy-range shards: A2 tile-length multiplier cap (0 = default)
  // instrumentation (host side)
  uint64_t launches = 0;   // kernels launched by lookup calls
};

// Per-call parameters of the lookup pipeline.
struct LookupArgs {
  uint64_t first_id = 0;
  uint32_t count = 0;
  uint32_t flags = 0;
  const double* in_energy = nullptr;  // explicit mode (device)
  bool energy_sampled = false;        // in_energy holds the library's own draws
                                      // (history mode): no range check needed
  const int32_t* in_mat = nullptr;
  const uint8_t* in_mat8 = nullptr;   // XS_FLAG_MAT_U8 (explicit mode, device)
  xs_outputs out{};                    // device pointers
  cudaEvent_t* ev = nullptr;           // [4] phase events (optional)
  uint64_t* launches = nullptr;        // incremented per kernel launch
  // energy-range shard (xs_lookup_batch_shard): only lookups with
  // e_lo <= p < e_hi are looked up (partitioned A2 only)
  bool shard = false;
  double e_lo = 0.0, e_hi = 0.0;
};

// workspace layout for a batch
struct Workspace {
  uint32_t* counts;   // [kMaxMats + 1]
  uint32_t* cursor;   // [kMaxMats + 1]
  LookupRec* recs;    // [count]
  uint32_t* bins;     // A2: [(n_mats + 1) * kEnergyBins]
  LookupRec* tmp;     // [count] records in batch order
  uint8_t* mat8;      // [count]
  uint32_t* partials; // A2 scan: [(n_mats + 1) * kEnergyBins / 4096]
  uint32_t* perm;     // A2: [count]
  uint32_t* gate;     // [1] k_check_energies flag (explicit energies)
  size_t bins_bytes;  // capacity of the bin area (the partitioned A2's tile
                      // histograms must fit it: coarse keys are narrowed if not)
  size_t total;
};
size_t workspace_layout(uint64_t count, uint32_t flags, int32_t n_mats, void* base,
                        Workspace* ws);

// xs_api.cu: sets the thread-local message of xs_last_error() and returns code
xs_status report_error(xs_status code, const char* msg, cudaError_t ce);

// grid_build.cu
cudaError_t build_union_grid(const DeviceGrid& g, double* U, cudaStream_t st);
cudaError_t build_index_grid(const DeviceGrid& g, cudaStream_t st);
cudaError_t build_index_grid_t(const DeviceGrid& g, cudaStream_t st);
cudaError_t build_hash_grid(const DeviceGrid& g, cudaStream_t st);
cudaError_t build_union_table(const DeviceGrid& g, cudaStream_t st);
cudaError_t build_intervals(const DeviceGrid& g, cudaStream_t st);
cudaError_t build_intervals32(const DeviceGrid& g, cudaStream_t st);
cudaError_t build_intervals_u(const DeviceGrid& g, cudaStream_t st);
cudaError_t init_constants();

// lookup.cu
size_t part_bins_bytes(uint64_t count, int32_t n_mats);  // partitioned A2's bin-area need
uint32_t energy_bin_host(double p);  // A2's energy bin of p (same arithmetic as the device)
bool part_cbits_fit(uint64_t count, int32_t n_mats, int cbits);  // shared memory / key-width limits
cudaError_t run_lookup(const DeviceGrid& g, const LookupArgs& a, const Workspace& ws,
                       cudaStream_t st);
// history mode (R19): `lookups` rounds of explicit lookups over
// the particle population, the per-particle stream state in hist_* arrays
struct HistoryArgs {
  uint64_t first_particle = 0;
  uint32_t n_particles = 0;
  int32_t lookups = 0;
  uint32_t flags = 0;                  // XS_FLAG_SORT only
  xs_outputs out{};                    // per-lookup arrays [n][lookups], vsum
  uint64_t* hist_state = nullptr;      // [n] LCG state after the last draw
  double* hist_energy = nullptr;       // [n] energy of the particle's next lookup
  int32_t* hist_mat = nullptr;         // [n] its material
  double* hist_M = nullptr;            // [n][5] macroscopic XS of the current round
  uint64_t* launches = nullptr;
};
cudaError_t run_history(const DeviceGrid& g, const HistoryArgs& h, const Workspace& ws,
                        cudaStream_t st);
cudaError_t run_verify(const DeviceGrid& g, const double* M, uint64_t count, uint64_t* vsum,
                       cudaStream_t st);
cudaError_t run_nuclide_index(const DeviceGrid& g, const double* energy, const int32_t* nuc,
                              uint64_t count, int32_t* k_out, cudaStream_t st);

}  // namespace xs
