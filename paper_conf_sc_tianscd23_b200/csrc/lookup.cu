// lookup.cu — the timed hot path: A1 sample, A2 (optional) sort, A3 search,
// A4 index gather, A5 record-pair gather, A6 interpolate, A7 accumulate,
// A8 verify (BASELINE.json north_star).
//
// Pipeline of one xs_lookup_batch call (all on the caller's stream):
//   sorted batches (XS_FLAG_SORT, the default of bench.py): the partitioned
//   A2 — k_part_count (A1 + per-tile coarse-key histograms; k_part_count_shard
//   for an energy-range shard), k_part_colscan / k_part_keyscan (scans),
//   k_part_place (A1 again, coarse-key order), k_part_fine (fine-key order) —
//   then the staged gather k_gather_s4 (A3 at each task's extremes, A4-A8;
//   variant table in launch_gather_tv).
//   unsorted batches:
//   k_sample    A1 + A3: sample (p, m) from the counter-based stream (or read
//               the caller's energies), search u (unionized) / bin b (hash),
//               write a 16-B LookupRec in batch order, count lookups per
//               material;
//   k_scatter   records into their material buckets;
//   k_gather_u  A4-A8 (k_gather without the K0u table).
//   Every gather fuses the verification v = 1 + argmax and adds one atomic
//   pair per block into vsum.  (k_sample / k_scan_* / k_scatter with binned
//   counts are the global-atomic A2, kept for comparison: "legacy_sort".)
#include <cfloat>
#include <type_traits>

#include "common.cuh"
#include "radix_sort.cuh"
#include "search.cuh"
#include "xs_internal.h"

namespace xs {

__constant__ JumpTable c_jump;
__device__ uint4 g_pick_tab[256];  // pick_material per 2^51-state bucket (below), 4096 B

// pick_material(RN(s) * 2^-63) from the raw state (integer thresholds in
// constant memory, common.cuh fill_pick_thresholds): 1 + #{k : s >= c_k},
// 12 -> 0 (fuel)
__device__ __forceinline__ int pick_material_state(uint64_t s) {
  int c = 0;
#pragma unroll
  for (int k = 0; k < 11; ++k) c += s >= c_jump.pick[k] ? 1 : 0;
  return c == 11 ? 0 : c + 1;
}

// The same through a 4096-bucket table of the top 12 state bits (built at
// init by make_pick_table, staged in shared memory per block): a bucket
// whose first and last state pick the same material picks it everywhere
// (the count above is monotone in s); the 11 buckets holding a threshold
// say kPickExact and take the compares.
constexpr int kPickBuckets = 4096;
constexpr uint8_t kPickExact = 0xff;
__device__ __forceinline__ void pick_table_fill(uint8_t* t) {
  for (int b = threadIdx.x; b < kPickBuckets / 16; b += blockDim.x)
    reinterpret_cast<uint4*>(t)[b] = g_pick_tab[b];
}
__device__ __forceinline__ int pick_material_tab(const uint8_t* t, uint64_t s) {
  const int m = t[s >> 51];
  return m != kPickExact ? m : pick_material_state(s);
}

// host: the bucket table of pick_material_tab (same integer decision)
static void make_pick_table(const JumpTable& t, uint8_t* out) {
  auto pick = [&](uint64_t s) {
    int c = 0;
    for (int k = 0; k < 11; ++k) c += s >= t.pick[k] ? 1 : 0;
    return c == 11 ? 0 : c + 1;
  };
  for (int b = 0; b < 4096; ++b) {
    const uint64_t lo = static_cast<uint64_t>(b) << 51, hi = lo + ((1ull << 51) - 1);
    const int a = pick(lo), z = pick(hi);
    out[b] = a == z ? static_cast<uint8_t>(a) : 0xff;
  }
}

cudaError_t init_constants() {
  JumpTable t = make_jump_table();
  cudaError_t e = cudaMemcpyToSymbol(c_jump, &t, sizeof(t));
  if (e != cudaSuccess) return e;
  alignas(16) uint8_t tab[4096];
  make_pick_table(t, tab);
  return cudaMemcpyToSymbol(g_pick_tab, tab, sizeof(tab));
}

// ------------------------------------------------------------------ A1 ----
// LCG^n(s) through the constant-memory jump table (powers of one affine map
// commute, so the bits can be applied in any order).
__device__ __forceinline__ uint64_t fast_forward(uint64_t s, uint64_t n) {
  s &= kMask63;
  int b = 0;
  while (n) {
    if (n & 1ULL) s = (c_jump.A[b] * s + c_jump.C[b]) & kMask63;
    n >>= 1;
    ++b;
  }
  return s;
}

struct Sample {
  double p;
  int32_t mat;
};

// lookup id -> (p, mat): s = FF(seed, 2 id); p = draw; roll = draw (R4)
__device__ __forceinline__ Sample sample_lookup(uint64_t seed, uint64_t id) {
  uint64_t s = fast_forward(seed, 2 * id);
  s = lcg_next(s);
  const double p = lcg_double(s);
  s = lcg_next(s);
  return Sample{p, pick_material_state(s)};
}

struct Params {
  // grid
  const double* grid;
  const double* iv;         // interval table [I][N][kIvDoubles] (K0d)
  const double* iv32;       // fp32-variant interval table [I][N][kIv32Doubles] (K0e)
  const double* ivu;        // 32-B aligned interval table [I][N][12] (K0u), or null
  int32_t I;
  int64_t N;
  const double* U;
  int64_t NU;
  const int32_t* UB;
  int32_t UBn;
  const int32_t* index;     // IG (row layout) / HG, or null
  const int32_t* index_t;   // IGT (column layout), or null
  int32_t B;
  double du;
  const int32_t* num_nucs;
  const int32_t* mats;
  const double* concs;
  int32_t n_mats, max_nucs;
  // batch
  uint64_t seed, first_id;
  uint32_t count;
  const double* in_energy;
  const int32_t* in_mat;
  const uint8_t* in_mat8;   // XS_FLAG_MAT_U8 (else null)
  // workspace
  uint32_t* counts;
  uint32_t* cursor;
  uint32_t* task_next;  // dynamic task counter of the staged gather (zeroed per call)
  // explicit energies: the gather is launched twice, with and without the
  // division range checks; each copy runs only if *gate == gate_want
  // (k_check_energies: 1 = some energy outside the exact fast-division range)
  const uint32_t* gate;
  uint32_t gate_want;
  LookupRec* recs;
  uint32_t* bins;   // [(n_mats + 1) * kEnergyBins] histogram -> cursors (A2)
  LookupRec* tmp;   // [count] records in batch order
  uint8_t* mat8;    // [count] material (n_mats = invalid)
  uint32_t* partials;  // A2 scan: per-chunk sums -> offsets
  uint32_t* perm;      // A2: batch positions in (material, energy) order (else null)
  int need_gidx;       // k_sample must search u per lookup (else the staged gather
                       // searches only each task's extreme energies)
  // partitioned A2 (k_part_*): H[block][key] lives in bins
  int cbits;            // coarse energy bits per material
  int nkr;              // coarse keys per material: (energy_bin >> (18 - cbits)) in
                        // [kc_lo, kc_lo + nkr) (all 2^cbits of them unless sharded)
  int kc_lo;
  int shard;            // 1: only lookups with e_lo <= p < e_hi are looked up
  double e_lo, e_hi;    //    (energy-range shard, xs_lookup_batch_shard)
  uint64_t s_lo, s_hi;  // the same range on the raw LCG state of the energy draw:
                        // e_lo <= RN(s) 2^-63 < e_hi <=> s_lo <= s < s_hi
  uint32_t tchunks;     // chunks per A2 tile (part_tile_chunks, times the shard
                        // multiplier for energy-range shards)
  uint32_t place_cap;   // k_part_place: tile lookups staged in shared memory (rank >= cap:
                        // stored straight to global memory; = tile length unless sharded)
  double* slab_p;       // shard mode: k_part_count keeps the tile's lookups of the
  uint64_t* slab_k;     // shard (energy; position << 16 | key) for k_part_place
  int fine_direct;      // k_part_fine scatters directly above this many windows
  int fine_cap;         // k_part_fine window (lookups)
  uint32_t* key_tot;    // [nkeys] lookups per coarse key
  uint32_t* key_start;  // [nkeys] first position of the key
  double* sp_tmp;       // [count] energies in coarse-key order
  uint32_t* sidx_tmp;   // [count] their batch positions (null: no per-lookup outputs)
  double* sp;           // [count] energies in (material, energy bin) order
  uint32_t* sidx;       // [count] their batch positions, or null
  // outputs
  double* out_M;
  double* out_E;
  int32_t* out_mat;
  int64_t* out_gidx;
  int32_t* out_v;
  unsigned long long* vsum;
};

__device__ __forceinline__ Sample get_lookup(const Params& P, uint32_t i) {
  if (P.in_energy) {
    int32_t m = P.in_mat8 ? static_cast<int32_t>(P.in_mat8[i]) : P.in_mat[i];
    if (m < 0 || m >= P.n_mats) m = P.n_mats;  // invalid bucket
    return Sample{P.in_energy[i], m};
  }
  return sample_lookup(P.seed, P.first_id + i);
}

template <int GT>
__device__ __forceinline__ int32_t grid_index_of(const Params& P, double p) {
  if (GT == XS_GRID_UNIONIZED) return static_cast<int32_t>(union_search(P.U, P.NU, p));
  if (GT == XS_GRID_HASH) return hash_bin(p, P.du, P.B);
  return -1;
}

// true when this launch of a gated gather pair is the inactive one
__device__ __forceinline__ bool gated_off(const Params& P) {
  return P.gate != nullptr && ((*P.gate != 0u) != (P.gate_want != 0u));
}

// Explicit energies p keep the fast correctly rounded division of A6 exact
// (no CHECK) when the grid is dyadic63 and every p is 0 or in [2^-440, 2^400]:
// then an = E[k+1] - p is 0 or a nonzero multiple of ulp >= 2^-492 and at most
// 2^401, inside div_in_range.  Sets *flag = 1 if any p is outside.
__global__ void k_check_energies(const double* __restrict__ p, uint32_t n, uint32_t* flag) {
  bool bad = false;
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const double v = p[i];
    bad |= !(v == 0.0 || (v >= 0x1p-440 && v <= 0x1p400));
  }
  if (__syncthreads_or(bad) && threadIdx.x == 0) atomicOr(flag, 1u);
}

__host__ __device__ __forceinline__ uint32_t energy_bin(double p) {
  const double q = p * static_cast<double>(kEnergyBins);
  if (!(q > 0.0)) return 0u;
  return q < static_cast<double>(kEnergyBins - 1) ? static_cast<uint32_t>(q) : kEnergyBins - 1u;
}

constexpr int kPrepThreads = 256;
constexpr int kPrepItems = 4;  // lookups per thread, searched in lockstep

__device__ __forceinline__ void write_invalid(const Params& P, uint32_t i) {
  if (P.out_M)
    for (int c = 0; c < 5; ++c)
      P.out_M[static_cast<uint64_t>(i) * 5 + c] = __longlong_as_double(0x7ff8000000000000LL);
  if (P.out_v) P.out_v[i] = 0;
}

// u = clamp(ub(U, p) - 1, 0, NU-2): the XSBench bisection loop started from
// the equal-width table's range [UB[b] - 1, UB[b+1]] (the loop invariant
// U[lo] <= p < U[hi] holds there, so the result is the full search's).
__device__ __forceinline__ int32_t union_index_tab(const Params& P, double p) {
  const double q = p * static_cast<double>(P.UBn);
  const int32_t b = q > 0.0 ? (q < static_cast<double>(P.UBn) ? static_cast<int32_t>(q) : P.UBn - 1) : 0;
  const int64_t l = q > 0.0 ? static_cast<int64_t>(__ldg(P.UB + b)) - 1 : 0;  // p <= 0: from 0
  int64_t lo = l < 0 ? 0 : (l > P.NU - 2 ? P.NU - 2 : l);
  int64_t hi = P.NU - 1;
  if (q < static_cast<double>(P.UBn)) {
    const int64_t h = __ldg(P.UB + b + 1);
    hi = h < P.NU - 1 ? h : P.NU - 1;
  }
  int64_t len = hi - lo;
  while (len > 1) {
    const int64_t mid = lo + (len >> 1);
    if (__ldg(P.U + mid) > p)
      hi = mid;
    else
      lo = mid;
    len = hi - lo;
  }
  return static_cast<int32_t>(lo);
}

// Conservative A3 bounds from the equal-width table alone (no bisection):
// ulo <= u(p) for p >= plo and uhi >= u(p) for p <= phi.  UB[b] = ub(U, b/UBn)
// and b/UBn <= p < (b+1)/UBn give ub(U, p) in [UB[b], UB[b+1]].  IGT is
// monotone in u, so the brackets read at ulo / uhi bound every bracket of the
// energies in [plo, phi]; the exact bracket is then found inside the window.
__device__ __forceinline__ int32_t union_lower_tab(const Params& P, double p) {
  const double q = p * static_cast<double>(P.UBn);
  if (!(q > 0.0)) return 0;
  const int32_t b = q < static_cast<double>(P.UBn) ? static_cast<int32_t>(q) : P.UBn;
  const int32_t l = __ldg(P.UB + b) - 1;
  return l < 0 ? 0 : (l > P.NU - 2 ? static_cast<int32_t>(P.NU - 2) : l);
}
__device__ __forceinline__ int32_t union_upper_tab(const Params& P, double p) {
  const double q = p * static_cast<double>(P.UBn);
  const int32_t b = q > 0.0 ? (q < static_cast<double>(P.UBn) ? static_cast<int32_t>(q) : P.UBn) : 0;
  if (b >= P.UBn) return static_cast<int32_t>(P.NU - 2);
  const int32_t h = __ldg(P.UB + b + 1) - 1;
  return h < 0 ? 0 : (h > P.NU - 2 ? static_cast<int32_t>(P.NU - 2) : h);
}

// k_sample: A1 + A3 in batch order.  Thread t of a block handles lookups
// c0 + kPrepItems*t + it, it < kPrepItems; their unionized searches run in
// lockstep (kPrepItems independent probes in flight per thread).  Writes
// the 16-B record tmp[i] = {p, i, u|b}, the material mat8[i] and the
// histogram: per material (plain) or per (material, energy bin) (A2).
template <int GT, bool BINNED>
__global__ void __launch_bounds__(kPrepThreads) k_sample(Params P) {
  __shared__ uint32_t s_h[kMaxMats + 1];
  if (!BINNED) {
    for (int t = threadIdx.x; t <= P.n_mats; t += blockDim.x) s_h[t] = 0;
    __syncthreads();
  }
  const uint32_t chunk = kPrepThreads * kPrepItems;
  for (uint64_t c0 = static_cast<uint64_t>(blockIdx.x) * chunk; c0 < P.count;
       c0 += static_cast<uint64_t>(gridDim.x) * chunk) {
    // A1: stream state at this chunk's first lookup, then short jumps
    __shared__ uint64_t s_state;
    if (!P.in_energy) {
      if (threadIdx.x == 0) s_state = fast_forward(P.seed, 2 * (P.first_id + c0));
      __syncthreads();
    }
    Sample smp[kPrepItems];
    bool ok[kPrepItems];
    int64_t lo[kPrepItems], hi[kPrepItems];
    // thread t owns the kPrepItems consecutive lookups c0 + kPrepItems*t + it:
    // one jump to the first, then two LCG steps per lookup (R4: lookup i+1's
    // stream starts where lookup i's two draws end)
    uint64_t st = 0;
    if (!P.in_energy) st = fast_forward(s_state, 2ull * kPrepItems * threadIdx.x);
#pragma unroll
    for (int it = 0; it < kPrepItems; ++it) {
      const uint64_t k = static_cast<uint64_t>(kPrepItems) * threadIdx.x + it;
      const uint64_t i = c0 + k;
      ok[it] = i < P.count;
      if (P.in_energy) {
        smp[it] = ok[it] ? get_lookup(P, static_cast<uint32_t>(i)) : Sample{0.0, 0};
      } else {
        st = lcg_next(st);
        const double pe = lcg_double(st);
        st = lcg_next(st);
        smp[it] = Sample{pe, pick_material_state(st)};
      }
      lo[it] = 0;
      hi[it] = P.NU - 1;
      if (GT == XS_GRID_UNIONIZED && P.need_gidx) {
        // A3 search range from the equal-width table: u in [UB[b]-1, UB[b+1]]
        const double q = smp[it].p * static_cast<double>(P.UBn);
        const int32_t b = q > 0.0 ? (q < static_cast<double>(P.UBn) ? static_cast<int32_t>(q)
                                                                    : P.UBn - 1)
                                  : 0;
        const int64_t l = q > 0.0 ? static_cast<int64_t>(__ldg(P.UB + b)) - 1 : 0;
        lo[it] = l < 0 ? 0 : (l > P.NU - 2 ? P.NU - 2 : l);
        if (q < static_cast<double>(P.UBn)) {  // p < 1: U[UB[b+1]] > p
          const int64_t h = __ldg(P.UB + b + 1);
          hi[it] = h < P.NU - 1 ? h : P.NU - 1;
        }
      }
    }
    if (!P.in_energy) __syncthreads();  // s_state is rewritten next chunk
    if (GT == XS_GRID_UNIONIZED && P.need_gidx) {
      // XSBench grid_search loop on [lo, hi] (invariant U[lo] <= p < U[hi]),
      // the kPrepItems searches interleaved
      bool busy = true;
      while (busy) {
        busy = false;
#pragma unroll
        for (int it = 0; it < kPrepItems; ++it) {
          const int64_t len = hi[it] - lo[it];
          if (len > 1) {
            const int64_t mid = lo[it] + (len >> 1);
            if (__ldg(P.U + mid) > smp[it].p)
              hi[it] = mid;
            else
              lo[it] = mid;
            busy |= (hi[it] - lo[it]) > 1;
          }
        }
      }
    }
    if (!BINNED) {
#pragma unroll
      for (int it = 0; it < kPrepItems; ++it) {
        const int key = ok[it] ? smp[it].mat : kMaxMats + 7;
        const uint32_t peers = __match_any_sync(0xffffffffu, key);
        if (ok[it] && (threadIdx.x & 31) == __ffs(peers) - 1) atomicAdd(&s_h[key], __popc(peers));
      }
    }
#pragma unroll
    for (int it = 0; it < kPrepItems; ++it) {
      if (!ok[it]) continue;
      const uint32_t i = static_cast<uint32_t>(c0 + static_cast<uint64_t>(kPrepItems) * threadIdx.x +
                                               it);
      const int32_t m = smp[it].mat;
      const double p = smp[it].p;
      const bool valid = m < P.n_mats;
      int32_t gi = -1;
      if (GT == XS_GRID_UNIONIZED) gi = static_cast<int32_t>(lo[it]);
      if (GT == XS_GRID_HASH) gi = hash_bin(p, P.du, P.B);
      LookupRec r;
      r.p = p;
      r.idx = i;  // BINNED: the rank within the (material, energy) bin instead
      r.gidx = valid ? gi : 0;
      if (BINNED)
        r.idx = atomicAdd(&P.bins[static_cast<uint32_t>(m) * kEnergyBins + energy_bin(p)], 1u);
      P.tmp[i] = r;
      P.mat8[i] = static_cast<uint8_t>(m);
      if (P.out_E) P.out_E[i] = p;
      if (P.out_mat)
        P.out_mat[i] = valid ? m : (P.in_mat8 ? static_cast<int32_t>(P.in_mat8[i])
                                    : (P.in_mat ? P.in_mat[i] : -1));
      if (P.out_gidx) P.out_gidx[i] = valid ? gi : -1;
      if (!valid) write_invalid(P, i);
    }
  }
  if (!BINNED) {
    __syncthreads();
    for (int t = threadIdx.x; t <= P.n_mats; t += blockDim.x)
      if (s_h[t]) atomicAdd(&P.counts[t], s_h[t]);
  }
}

// A2 scan of the (material, energy bin) histogram: exclusive prefix sums in
// place (they become the scatter cursors) and the per-material totals.
// Three kernels over chunks of kScanChunk bins (kEnergyBins is a multiple).
constexpr int kScanChunk = 4096;

// block-wide exclusive scan of v (1024 threads); returns the block total
__device__ __forceinline__ uint32_t block_excl_scan(uint32_t v, uint32_t* excl) {
  __shared__ uint32_t s_w[32];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  uint32_t x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) s_w[w] = x;
  __syncthreads();
  if (w == 0) {
    uint32_t t = s_w[lane];
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, t, o);
      if (lane >= o) t += y;
    }
    s_w[lane] = t;
  }
  __syncthreads();
  *excl = (w ? s_w[w - 1] : 0u) + x - v;
  const uint32_t total = s_w[31];
  __syncthreads();
  return total;
}

// the same for NT threads (a multiple of 32, at most 1024)
template <int NT>
__device__ __forceinline__ uint32_t block_excl_scan_n(uint32_t v, uint32_t* excl) {
  constexpr int kW = NT / 32;
  __shared__ uint32_t s_w[kW];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  uint32_t x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) s_w[w] = x;
  __syncthreads();
  if (w == 0) {
    uint32_t t = lane < kW ? s_w[lane] : 0u;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, t, o);
      if (lane >= o) t += y;
    }
    if (lane < kW) s_w[lane] = t;
  }
  __syncthreads();
  *excl = (w ? s_w[w - 1] : 0u) + x - v;
  const uint32_t total = s_w[kW - 1];
  __syncthreads();
  return total;
}

__global__ void __launch_bounds__(1024) k_scan_partial(Params P) {
  const uint32_t* c = P.bins + static_cast<uint64_t>(blockIdx.x) * kScanChunk;
  uint32_t v = 0;
  for (int t = threadIdx.x; t < kScanChunk; t += blockDim.x) v += c[t];
  uint32_t ex;
  const uint32_t tot = block_excl_scan(v, &ex);
  if (threadIdx.x == 0) P.partials[blockIdx.x] = tot;
}

__global__ void __launch_bounds__(1024) k_scan_top(Params P, uint32_t nchunks) {
  constexpr uint32_t kPer = kEnergyBins / kScanChunk;
  constexpr int kMaxPer = 8;  // nchunks <= 8192 (65 materials x 64 chunks)
  const uint32_t per = (nchunks + 1023) / 1024;
  uint32_t v[kMaxPer];
  uint32_t sum = 0;
#pragma unroll
  for (int q = 0; q < kMaxPer; ++q) {
    const uint32_t i = threadIdx.x * per + q;
    v[q] = (q < static_cast<int>(per) && i < nchunks) ? P.partials[i] : 0u;
    sum += v[q];
  }
  uint32_t ex;
  block_excl_scan(sum, &ex);
#pragma unroll
  for (int q = 0; q < kMaxPer; ++q) {
    const uint32_t i = threadIdx.x * per + q;
    if (q < static_cast<int>(per) && i < nchunks) {
      P.partials[i] = ex;
      if (v[q]) atomicAdd(&P.counts[i / kPer], v[q]);
      ex += v[q];
    }
  }
}

__global__ void __launch_bounds__(1024) k_scan_apply(Params P) {
  uint32_t* c = P.bins + static_cast<uint64_t>(blockIdx.x) * kScanChunk;
  constexpr int kPerThread = kScanChunk / 1024;
  uint32_t v[kPerThread];
  uint32_t sum = 0;
#pragma unroll
  for (int q = 0; q < kPerThread; ++q) {
    v[q] = c[threadIdx.x * kPerThread + q];
    sum += v[q];
  }
  uint32_t ex;
  block_excl_scan(sum, &ex);
  ex += P.partials[blockIdx.x];
#pragma unroll
  for (int q = 0; q < kPerThread; ++q) {
    c[threadIdx.x * kPerThread + q] = ex;
    ex += v[q];
  }
}

// k_scatter: place each record in its material bucket (plain: block-
// aggregated per-material cursors) or (material, energy bin) slot (A2: the
// scanned histogram gives the bin start, k_sample's atomic the rank within
// the bin).  Order inside a bucket or bin is arbitrary: results never
// depend on it.
template <bool BINNED>
__global__ void __launch_bounds__(kPrepThreads) k_scatter(Params P) {
  __shared__ uint32_t s_off[kMaxMats + 2];
  __shared__ uint32_t s_cnt[kMaxMats + 1];
  __shared__ uint32_t s_base[kMaxMats + 1];
  const int nm1 = P.n_mats + 1;
  if (!BINNED && threadIdx.x == 0) {
    uint32_t run = 0;
    for (int m = 0; m < nm1; ++m) {
      s_off[m] = run;
      run += P.counts[m];
    }
    s_off[nm1] = run;
  }
  __syncthreads();
  const int lane = threadIdx.x & 31;
  const uint32_t chunk = kPrepThreads * kPrepItems;
  for (uint64_t c0 = static_cast<uint64_t>(blockIdx.x) * chunk; c0 < P.count;
       c0 += static_cast<uint64_t>(gridDim.x) * chunk) {
    if (!BINNED) {
      for (int t = threadIdx.x; t < nm1; t += blockDim.x) s_cnt[t] = 0;
      __syncthreads();
    }
    LookupRec rec[kPrepItems];
    int32_t mm[kPrepItems];
    uint32_t rank[kPrepItems];
#pragma unroll
    for (int it = 0; it < kPrepItems; ++it) {
      const uint64_t i = c0 + static_cast<uint64_t>(it) * kPrepThreads + threadIdx.x;
      const bool ok = i < P.count;
      if (ok) {
        rec[it] = P.tmp[i];
        mm[it] = P.mat8[i];
      } else {
        mm[it] = kMaxMats + 7;
      }
      rank[it] = 0;
      if (BINNED) {
        if (ok) {
          rank[it] = __ldg(P.bins + static_cast<uint32_t>(mm[it]) * kEnergyBins +
                           energy_bin(rec[it].p)) + rec[it].idx;
          rec[it].idx = static_cast<uint32_t>(i);
        }
      } else {
        const uint32_t peers = __match_any_sync(0xffffffffu, mm[it]);
        const int leader = __ffs(peers) - 1;
        uint32_t b = 0;
        if (ok && lane == leader) b = atomicAdd(&s_cnt[mm[it]], __popc(peers));
        b = __shfl_sync(0xffffffffu, b, leader);
        rank[it] = b + __popc(peers & ((1u << lane) - 1u));
      }
    }
    if (!BINNED) {
      __syncthreads();
      for (int t = threadIdx.x; t < nm1; t += blockDim.x)
        s_base[t] = s_cnt[t] ? s_off[t] + atomicAdd(&P.cursor[t], s_cnt[t]) : 0u;
      __syncthreads();
    }
#pragma unroll
    for (int it = 0; it < kPrepItems; ++it) {
      const uint64_t i = c0 + static_cast<uint64_t>(it) * kPrepThreads + threadIdx.x;
      if (i < P.count) {
        if (BINNED) P.perm[rank[it]] = static_cast<uint32_t>(i);  // 4-B writes, L2-resident array
        else
          P.recs[s_base[mm[it]] + rank[it]] = rec[it];
      }
    }
    if (!BINNED) __syncthreads();
  }
}

// ----------------------------------------------- A2, partitioned variant ---
// The A2 of the staged gather (its default): a two-level counting sort that
// moves only the energy (8 B) and, when per-lookup outputs are requested, the
// batch position (4 B).  The key is the same (material, energy bin of width
// 2^-18) as above, split into a coarse part (material, top cbits of the bin;
// a small fan-out, so that every tile writes runs of whole sectors) and a
// fine part (the remaining 18 - cbits bits):
//   k_part_count    A1 (+ per-lookup A3 outputs) in batch order; per-tile
//                   histogram of coarse keys in shared memory -> H[tile][key]
//   k_part_colscan  per key: exclusive scan of H over tiles, key totals
//   k_part_keyscan  exclusive scan of the key totals -> key starts; material counts
//   k_part_place    A1 again, tile by tile; position = key start + tile offset +
//                   shared-memory rank (energies in coarse-key order)
//   k_part_fine     one block per coarse key: counting sort of its segment by
//                   the fine key (shared-memory histogram, segment L2-resident)
// Only shared-memory atomics.  Order inside a fine bin is arbitrary: results
// never depend on it.
constexpr int kPartItems = kPrepItems;
constexpr int kPlaceThreads = 512;  // k_part_place: 2 chunks of a tile in flight (one block per SM)
constexpr uint32_t kPartChunk = kPrepThreads * kPartItems;  // lookups per block round
// tiles of 8 chunks up to 2^15 tiles (268M lookups; H [tiles][nkeys] is
// 218 MB there, reserved by workspace_layout), longer tiles beyond
constexpr uint32_t kPartMaxTiles = 1u << 15;

__host__ __device__ __forceinline__ uint32_t part_tile_chunks(uint64_t count) {
  const uint64_t chunks = (count + kPartChunk - 1) / kPartChunk;
  const uint64_t per = (chunks + kPartMaxTiles - 1) / kPartMaxTiles;
  return static_cast<uint32_t>(per < 8 ? 8 : per);
}

// LCG^n as an affine map (A, C) from the constant-memory jump table
__device__ __forceinline__ void affine_pow(uint64_t n, uint64_t& A, uint64_t& C) {
  A = 1;
  C = 0;
  int b = 0;
  while (n) {
    if (n & 1ULL) {
      A = (A * c_jump.A[b]) & kMask63;
      C = (C * c_jump.A[b] + c_jump.C[b]) & kMask63;
    }
    n >>= 1;
    ++b;
  }
}

__device__ __forceinline__ uint32_t part_key(const Params& P, const Sample& s) {
  return static_cast<uint32_t>(s.mat) * static_cast<uint32_t>(P.nkr) +
         ((energy_bin(s.p) >> (18 - P.cbits)) - static_cast<uint32_t>(P.kc_lo));
}

// energy-range shard filter (always true outside shard mode)
__device__ __forceinline__ bool in_shard(const Params& P, double p) {
  return !P.shard || (p >= P.e_lo && p < P.e_hi);
}

// The kPartItems lookups of thread t in the chunk starting at c0 (the same
// assignment in k_part_count and k_part_place).  sc = stream state at the
// chunk's first lookup, tA, tC = LCG^(2 kPartItems t).
__device__ __forceinline__ void part_samples(const Params& P, uint64_t c0, uint64_t sc, uint64_t tA,
                                             uint64_t tC, const uint8_t* s_pick,
                                             Sample (&smp)[kPartItems], bool (&ok)[kPartItems],
                                             uint32_t tid = threadIdx.x) {
  uint64_t st = (tA * sc + tC) & kMask63;
#pragma unroll
  for (int it = 0; it < kPartItems; ++it) {
    const uint64_t i = c0 + static_cast<uint64_t>(kPartItems) * tid + it;
    ok[it] = i < P.count;
    if (P.in_energy) {
      smp[it] = ok[it] ? get_lookup(P, static_cast<uint32_t>(i)) : Sample{0.0, 0};
    } else {
      st = lcg_next(st);
      const double pe = lcg_double(st);
      st = lcg_next(st);
      smp[it] = Sample{pe, pick_material_tab(s_pick, st)};
      ok[it] = ok[it] && in_shard(P, pe);
    }
  }
}

// Stream constants of a k_part_* thread: the chunk-to-chunk jump and the
// thread's offset inside a chunk; the state at a tile's first lookup is one
// fast-forward per tile.
struct PartStream {
  uint64_t cA, cC, tA, tC;
  __device__ __forceinline__ void init(const Params& P, uint32_t tid = threadIdx.x,
                                       uint32_t chunk_stride = 1) {
    cA = tA = 1;
    cC = tC = 0;
    if (P.in_energy) return;
    affine_pow(2ull * kPartChunk * chunk_stride, cA, cC);
    affine_pow(2ull * kPartItems * tid, tA, tC);
  }
  __device__ __forceinline__ uint64_t at(const Params& P, uint64_t first) const {
    return P.in_energy ? 0 : fast_forward(P.seed, 2 * (P.first_id + first));
  }
  __device__ __forceinline__ uint64_t next(uint64_t sc) const { return (cA * sc + cC) & kMask63; }
};

template <int GT>
__global__ void __launch_bounds__(kPrepThreads) k_part_count(Params P) {
  extern __shared__ uint32_t s_h[];  // [nkeys]
  const int nkeys = (P.n_mats + 1) * P.nkr;
  const uint32_t tchunks = P.tchunks;
  const uint64_t tlen = static_cast<uint64_t>(tchunks) * kPartChunk;
  const uint32_t ntiles = static_cast<uint32_t>((P.count + tlen - 1) / tlen);
  const bool outputs = P.out_E || P.out_mat || P.out_gidx || P.out_M || P.out_v;
  PartStream ps;
  ps.init(P);
  __shared__ uint32_t s_kept;
  __shared__ __align__(16) uint8_t s_pick[kPickBuckets];
  pick_table_fill(s_pick);  // (first use after the tile loop's barrier)
  for (uint32_t tl = blockIdx.x; tl < ntiles; tl += gridDim.x) {
    for (int t = threadIdx.x; t < nkeys; t += blockDim.x) s_h[t] = 0;
    if (threadIdx.x == 0) s_kept = 0;
    __syncthreads();
    uint64_t sc = ps.at(P, tl * tlen);
    for (uint32_t c = 0; c < tchunks; ++c, sc = ps.next(sc)) {
      const uint64_t c0 = tl * tlen + static_cast<uint64_t>(c) * kPartChunk;
      if (c0 >= P.count) break;
      Sample smp[kPartItems];
      bool ok[kPartItems];
      part_samples(P, c0, sc, ps.tA, ps.tC, s_pick, smp, ok);
#pragma unroll
      for (int it = 0; it < kPartItems; ++it) {
        if (!ok[it]) continue;
        const uint32_t key = part_key(P, smp[it]);
        atomicAdd(&s_h[key], 1u);
        if (P.slab_p && smp[it].mat < P.n_mats) {  // shard: keep it for k_part_place
          const uint32_t q = atomicAdd(&s_kept, 1u);
          const uint64_t at = static_cast<uint64_t>(tl) * tlen + q;
          P.slab_p[at] = smp[it].p;
          P.slab_k[at] = ((c0 + static_cast<uint64_t>(kPartItems) * threadIdx.x + it) << 16) | key;
        }
        if (!outputs) continue;
        const uint32_t i = static_cast<uint32_t>(c0 + static_cast<uint64_t>(kPartItems) * threadIdx.x + it);
        const bool valid = smp[it].mat < P.n_mats;
        if (P.out_E) P.out_E[i] = smp[it].p;
        if (P.out_mat)
          P.out_mat[i] = valid ? smp[it].mat
                               : (P.in_mat8 ? static_cast<int32_t>(P.in_mat8[i]) : (P.in_mat ? P.in_mat[i] : -1));
        if (P.out_gidx) {
          int32_t gi = -1;
          if (GT == XS_GRID_UNIONIZED) gi = union_index_tab(P, smp[it].p);
          if (GT == XS_GRID_HASH) gi = hash_bin(smp[it].p, P.du, P.B);
          P.out_gidx[i] = valid ? gi : -1;
        }
        if (!valid) write_invalid(P, i);
      }
    }
    __syncthreads();
    uint32_t* row = P.bins + static_cast<uint64_t>(tl) * nkeys;
    for (int t = threadIdx.x; t < nkeys; t += blockDim.x) row[t] = s_h[t];
    __syncthreads();
  }
}

// k_part_count for an energy-range shard (xs_lookup_batch_shard): A1 for
// every lookup of the batch, but only ~1/n_shards of them are this shard's.
// Each thread draws its four energies (two LCG steps each), the warp
// compacts the lookups inside [e_lo, e_hi) through shared memory (ballot +
// prefix), and the material pick, coarse key, histogram and the slab entry
// for k_part_place are computed once per kept lookup with all lanes busy.
constexpr int kShardWarps = kPrepThreads / 32;
__global__ void __launch_bounds__(kPrepThreads) k_part_count_shard(Params P) {
  extern __shared__ uint32_t s_h[];  // [nkeys]
  __shared__ __align__(16) uint8_t s_pick[kPickBuckets];
  // a warp's kept lookups are processed in batches of at least 32 * kPartItems
  // (all lanes busy): room for one more chunk on top of that
  __shared__ uint64_t s_cs[kShardWarps][2 * 32 * kPartItems];
  __shared__ uint32_t s_ci[kShardWarps][2 * 32 * kPartItems];
  __shared__ uint32_t s_kept;
  const int nkeys = (P.n_mats + 1) * P.nkr;
  const uint32_t tchunks = P.tchunks;
  const uint64_t tlen = static_cast<uint64_t>(tchunks) * kPartChunk;
  const uint32_t ntiles = static_cast<uint32_t>((P.count + tlen - 1) / tlen);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  pick_table_fill(s_pick);
  PartStream ps;
  ps.init(P);
  for (uint32_t tl = blockIdx.x; tl < ntiles; tl += gridDim.x) {
    for (int t = threadIdx.x; t < nkeys; t += blockDim.x) s_h[t] = 0;
    if (threadIdx.x == 0) s_kept = 0;
    __syncthreads();
    uint64_t sc = ps.at(P, tl * tlen);
    uint32_t run = 0;  // kept lookups staged for this warp
    // the pick, key, histogram and slab entry of the staged lookups; the
    // warp's slab slots come from one shared atomic per batch
    auto flush = [&]() {
      uint32_t base = 0;
      if (lane == 0 && run) base = atomicAdd(&s_kept, run);
      base = __shfl_sync(0xffffffffu, base, 0);
      for (uint32_t q = lane; q < run; q += 32) {
        const uint64_t s1 = s_cs[warp][q];
        const Sample smp{lcg_double(s1), pick_material_tab(s_pick, lcg_next(s1))};
        const uint32_t key = part_key(P, smp);
        atomicAdd(&s_h[key], 1u);
        const uint64_t at = static_cast<uint64_t>(tl) * tlen + base + q;
        P.slab_p[at] = smp.p;
        P.slab_k[at] = (static_cast<uint64_t>(s_ci[warp][q]) << 16) | key;
      }
      __syncwarp();
      run = 0;
    };
    for (uint32_t c = 0; c < tchunks; ++c, sc = ps.next(sc)) {
      const uint64_t c0 = tl * tlen + static_cast<uint64_t>(c) * kPartChunk;
      if (c0 >= P.count) break;
      uint64_t st = (ps.tA * sc + ps.tC) & kMask63;
      const bool full = c0 + kPartChunk <= P.count;
#pragma unroll
      for (int it = 0; it < kPartItems; ++it) {
        const uint64_t i = c0 + static_cast<uint64_t>(kPartItems) * threadIdx.x + it;
        const uint64_t s1 = lcg_next(st);  // the energy draw's state
        st = lcg_next(s1);
        // range test on the state (no conversion for the ~(n-1)/n dropped)
        const bool keep = (full || i < P.count) && s1 >= P.s_lo && s1 < P.s_hi;
        const uint32_t ball = __ballot_sync(0xffffffffu, keep);
        if (keep) {
          const uint32_t q = run + __popc(ball & ((1u << lane) - 1u));
          s_cs[warp][q] = s1;
          s_ci[warp][q] = static_cast<uint32_t>(i);
        }
        run += __popc(ball);
      }
      __syncwarp();
      if (run >= 32 * kPartItems) flush();
    }
    flush();
    __syncthreads();
    uint32_t* row = P.bins + static_cast<uint64_t>(tl) * nkeys;
    for (int t = threadIdx.x; t < nkeys; t += blockDim.x) row[t] = s_h[t];
    __syncthreads();
  }
}

constexpr int kColIlp = 8;
// H[t][key] -> exclusive prefix over tiles t (per key); key totals.  Block =
// KX keys x SY slices of the tiles (KX * SY = 1024): few keys (energy-range
// shards) take more slices per key so that the latency-bound column walks
// spread over more SMs.
template <int KX, int SY>
__global__ void __launch_bounds__(1024) k_part_colscan(Params P, int nb) {
  static_assert(KX * SY == 1024, "block");
  __shared__ uint32_t s_p[SY][KX + 1];
  const int nkeys = (P.n_mats + 1) * P.nkr;
  const int key = blockIdx.x * KX + threadIdx.x;
  const int sl = threadIdx.y;
  const int per = (nb + SY - 1) / SY;
  const int b0 = sl * per, b1 = min(nb, b0 + per);
  // both passes keep kColIlp loads in flight (the rows are nkeys * 4 B apart;
  // a dependent walk is latency-bound at XL's 20k tiles)
  uint32_t sum = 0;
  if (key < nkeys)
    for (int b = b0; b < b1; b += kColIlp) {
      uint32_t v[kColIlp];
#pragma unroll
      for (int u = 0; u < kColIlp; ++u)
        v[u] = b + u < b1 ? P.bins[static_cast<uint64_t>(b + u) * nkeys + key] : 0u;
#pragma unroll
      for (int u = 0; u < kColIlp; ++u) sum += v[u];
    }
  s_p[sl][threadIdx.x] = sum;
  __syncthreads();
  if (sl == 0) {
    uint32_t run = 0;
    for (int q = 0; q < SY; ++q) {
      const uint32_t v = s_p[q][threadIdx.x];
      s_p[q][threadIdx.x] = run;
      run += v;
    }
    if (key < nkeys) P.key_tot[key] = run;
  }
  __syncthreads();
  if (key < nkeys) {
    uint32_t run = s_p[sl][threadIdx.x];
    for (int b = b0; b < b1; b += kColIlp) {
      uint32_t v[kColIlp];
#pragma unroll
      for (int u = 0; u < kColIlp; ++u)
        v[u] = b + u < b1 ? P.bins[static_cast<uint64_t>(b + u) * nkeys + key] : 0u;
#pragma unroll
      for (int u = 0; u < kColIlp; ++u) {
        if (b + u < b1) P.bins[static_cast<uint64_t>(b + u) * nkeys + key] = run;
        run += v[u];
      }
    }
  }
}

// key_start = exclusive scan of key_tot (one block); counts[m] per material
__global__ void __launch_bounds__(1024) k_part_keyscan(Params P) {
  const int nkeys = (P.n_mats + 1) * P.nkr;
  const int per = (nkeys + 1023) / 1024;
  const int k0 = threadIdx.x * per, k1 = min(nkeys, k0 + per);
  uint32_t sum = 0;
  for (int k = k0; k < k1; ++k) sum += P.key_tot[k];
  uint32_t ex;
  const uint32_t total = block_excl_scan(sum, &ex);
  for (int k = k0; k < k1; ++k) {
    P.key_start[k] = ex;
    ex += P.key_tot[k];
  }
  __syncthreads();
  for (int m = threadIdx.x; m <= P.n_mats; m += blockDim.x) {
    const uint32_t s = P.key_start[m * P.nkr];
    const uint32_t e = m < P.n_mats ? P.key_start[(m + 1) * P.nkr] : total;
    P.counts[m] = e - s;
  }
}

// k_part_place: A1 again, tile by tile.  Every lookup of the tile first goes
// to its rank inside the tile's coarse-key order in shared memory (the tile's
// per-key counts are the differences of the scanned H rows), then the tile
// leaves as runs of consecutive positions (coalesced stores).
// NT threads per block: NT / kPrepThreads chunks of the tile in flight at
// once (each kPrepThreads-thread slice samples every (NT / kPrepThreads)-th
// chunk; the tile and its order are those of k_part_count)
template <int GT, int NT>
__global__ void __launch_bounds__(NT) k_part_place(Params P) {
  constexpr uint32_t kSlices = NT / kPrepThreads;
  static_assert(NT % kPrepThreads == 0, "whole chunk slices");
  extern __shared__ __align__(16) unsigned char smem_pl[];
  const int nkeys = (P.n_mats + 1) * P.nkr;
  const int nvalid = P.n_mats * P.nkr;
  const uint32_t tchunks = P.tchunks;
  const uint64_t tlen = static_cast<uint64_t>(tchunks) * kPartChunk;
  const uint32_t ntiles = static_cast<uint32_t>((P.count + tlen - 1) / tlen);
  uint32_t* s_ls = reinterpret_cast<uint32_t*>(smem_pl);   // [nkeys + 1] local starts
  uint32_t* s_lc = s_ls + nkeys + 1;                       // [nkeys] local cursors
  uint32_t* s_gb = s_lc + nkeys;                           // [nkeys] global bases
  const uint32_t cap = P.place_cap;  // staged lookups per tile
  double* s_p = reinterpret_cast<double*>(smem_pl + ((3 * static_cast<size_t>(nkeys) + 1) * 4 + 15) / 16 * 16);
  uint16_t* s_k = reinterpret_cast<uint16_t*>(s_p + cap);
  uint32_t* s_i = reinterpret_cast<uint32_t*>(s_k + cap);
  __shared__ __align__(16) uint8_t s_pick[kPickBuckets];
  pick_table_fill(s_pick);  // (first use after the tile loop's barrier)
  const uint32_t slice = threadIdx.x / kPrepThreads, lt = threadIdx.x % kPrepThreads;
  PartStream ps;
  ps.init(P, lt, kSlices);
  uint64_t sA = 1, sC = 0;  // LCG^(2 kPartChunk slice): this slice's first chunk
  if (!P.in_energy) affine_pow(2ull * kPartChunk * slice, sA, sC);
  for (uint32_t tl = blockIdx.x; tl < ntiles; tl += gridDim.x) {
    const uint32_t* row = P.bins + static_cast<uint64_t>(tl) * nkeys;
    const uint32_t* nxt = tl + 1 < ntiles ? row + nkeys : nullptr;
    // local exclusive scan of the tile's per-key counts (keys in order; the
    // invalid material's keys come last)
    const int per = (nkeys + NT - 1) / NT;
    const int k0 = threadIdx.x * per, k1 = min(nkeys, k0 + per);
    uint32_t sum = 0;
    for (int k = k0; k < k1; ++k) sum += (nxt ? nxt[k] : P.key_tot[k]) - row[k];
    uint32_t ex;
    block_excl_scan_n<NT>(sum, &ex);
    for (int k = k0; k < k1; ++k) {
      s_ls[k] = ex;
      s_lc[k] = ex;
      s_gb[k] = P.key_start[k] + row[k];
      ex += (nxt ? nxt[k] : P.key_tot[k]) - row[k];
    }
    __syncthreads();
    const uint32_t nloc = s_ls[nvalid];  // valid lookups of the tile
    if (P.slab_p) {  // shard: the tile's lookups of the shard, kept by k_part_count
      // kSlabIlp slab entries in flight per thread (the loop is load-latency bound)
      constexpr int kSlabIlp = 4;
      for (uint32_t i0 = threadIdx.x; i0 < nloc; i0 += kSlabIlp * NT) {
        uint64_t kk[kSlabIlp];
        double pp[kSlabIlp];
#pragma unroll
        for (int u = 0; u < kSlabIlp; ++u) {
          const uint32_t i = i0 + u * NT;
          const uint64_t at = static_cast<uint64_t>(tl) * tlen + i;
          kk[u] = i < nloc ? P.slab_k[at] : 0ull;
          pp[u] = i < nloc ? P.slab_p[at] : 0.0;
        }
#pragma unroll
        for (int u = 0; u < kSlabIlp; ++u) {
          if (i0 + u * NT >= nloc) continue;
          const uint32_t key = static_cast<uint32_t>(kk[u] & 0xffffu);
          const uint32_t q = atomicAdd(&s_lc[key], 1u);
          if (q < cap) {
            s_p[q] = pp[u];
            s_k[q] = static_cast<uint16_t>(key);
            if (P.sidx_tmp) s_i[q] = static_cast<uint32_t>(kk[u] >> 16);
          } else {  // beyond the staging capacity: straight to its place
            const uint32_t d = s_gb[key] + (q - s_ls[key]);
            P.sp_tmp[d] = pp[u];
            if (P.sidx_tmp) P.sidx_tmp[d] = static_cast<uint32_t>(kk[u] >> 16);
          }
        }
      }
    }
    uint64_t sc = ps.at(P, tl * tlen);
    sc = (sA * sc + sC) & kMask63;
    for (uint32_t c = slice; c < tchunks && !P.slab_p; c += kSlices, sc = ps.next(sc)) {
      const uint64_t c0 = tl * tlen + static_cast<uint64_t>(c) * kPartChunk;
      if (c0 >= P.count) break;
      Sample smp[kPartItems];
      bool ok[kPartItems];
      part_samples(P, c0, sc, ps.tA, ps.tC, s_pick, smp, ok, lt);
#pragma unroll
      for (int it = 0; it < kPartItems; ++it) {
        if (!ok[it] || smp[it].mat >= P.n_mats) continue;  // invalid lookups are not gathered
        const uint32_t key = part_key(P, smp[it]);
        const uint32_t q = atomicAdd(&s_lc[key], 1u);
        s_p[q] = smp[it].p;
        s_k[q] = static_cast<uint16_t>(key);
        if (P.sidx_tmp)
          s_i[q] = static_cast<uint32_t>(c0 + static_cast<uint64_t>(kPartItems) * lt + it);
      }
    }
    __syncthreads();
    const uint32_t nst = nloc < cap ? nloc : cap;
    for (uint32_t i = threadIdx.x; i < nst; i += NT) {
      const uint32_t k = s_k[i];
      const uint32_t d = s_gb[k] + (i - s_ls[k]);
      P.sp_tmp[d] = s_p[i];
      if (P.sidx_tmp) P.sidx_tmp[d] = s_i[i];
    }
    __syncthreads();
  }
}

// k_part_fine: one block per coarse key of a valid material: counting sort
// of its segment by the fine key (the low 18 - cbits bits of the energy
// bin).  The histogram is scanned once; the output is then produced in
// windows of consecutive fine bins holding at most `cap` lookups (as many as
// the shared memory left after the histograms holds: 24576 energies, or 16384
// energy + position pairs when per-lookup outputs are written): each
// window re-reads the segment (L2-resident after the first pass), places its
// lookups in shared memory and stores the window as one coalesced run.
constexpr int kFineThreads = 1024, kFineBinsMax = 4096, kFineIlp = 4;
constexpr int kFineCapP = 24576, kFineCapPI = 16384;  // energies / energy + position
__host__ __device__ constexpr size_t fine_hist_bytes(uint32_t nf) { return ((2 * nf + 1) * 4 + 15) / 16 * 16; }
__global__ void __launch_bounds__(kFineThreads) k_part_fine(Params P) {
  extern __shared__ __align__(16) unsigned char smem_fine[];
  const int fb = 18 - P.cbits;
  const uint32_t nf = 1u << fb, fmask = nf - 1u;
  uint32_t* s_st = reinterpret_cast<uint32_t*>(smem_fine);            // [nf + 1] bin starts
  uint32_t* s_cu = s_st + nf + 1;                                      // [nf] cursors
  const uint32_t cap = static_cast<uint32_t>(P.fine_cap);
  double* s_p = reinterpret_cast<double*>(smem_fine + fine_hist_bytes(nf));  // [cap]
  uint32_t* s_i = reinterpret_cast<uint32_t*>(s_p + cap);              // [cap] (positions)
  __shared__ uint32_t s_win[2];
  const int key = blockIdx.x;
  const uint32_t s = P.key_start[key], n = P.key_tot[key];
  if (n == 0) return;
  const int t = threadIdx.x;
  for (uint32_t f = t; f < nf; f += kFineThreads) s_cu[f] = 0;
  __syncthreads();
  const double* src = P.sp_tmp + s;
  const uint32_t* isrc = P.sidx_tmp ? P.sidx_tmp + s : nullptr;
  // kFineIlp independent loads in flight per thread (one block per SM: the
  // segment streams are bound by memory-level parallelism, not bandwidth)
  for (uint32_t i0 = t; i0 < n; i0 += kFineIlp * kFineThreads) {
    double pv[kFineIlp];
#pragma unroll
    for (int u = 0; u < kFineIlp; ++u) {
      const uint32_t i = i0 + u * kFineThreads;
      pv[u] = i < n ? src[i] : 0.0;
    }
#pragma unroll
    for (int u = 0; u < kFineIlp; ++u)
      if (i0 + u * kFineThreads < n) atomicAdd(&s_cu[energy_bin(pv[u]) & fmask], 1u);
  }
  __syncthreads();
  // exclusive scan -> s_st (nf / kFineThreads bins per thread)
  const uint32_t per = (nf + kFineThreads - 1) / kFineThreads;
  const uint32_t f0 = t * per;
  uint32_t sum = 0;
  for (uint32_t f = f0; f < f0 + per && f < nf; ++f) sum += s_cu[f];
  uint32_t ex;
  block_excl_scan_n<kFineThreads>(sum, &ex);
  for (uint32_t f = f0; f < f0 + per && f < nf; ++f) {
    s_st[f] = ex;
    ex += s_cu[f];
  }
  if (t == 0) s_st[nf] = n;
  __syncthreads();
  double* dst = P.sp + s;
  uint32_t* idst = P.sidx ? P.sidx + s : nullptr;
  if (n > static_cast<uint64_t>(P.fine_direct) * cap) {
    // long segment (XL): one pass that scatters every energy to its bin's
    // cursor in the output (the segment's output range stays L2-resident)
    // instead of re-reading the segment once per window
    for (uint32_t f = t; f < nf; f += kFineThreads) s_cu[f] = s_st[f];
    __syncthreads();
    for (uint32_t i0 = t; i0 < n; i0 += kFineIlp * kFineThreads) {
      double pv[kFineIlp];
#pragma unroll
      for (int u = 0; u < kFineIlp; ++u) {
        const uint32_t i = i0 + u * kFineThreads;
        pv[u] = i < n ? src[i] : 0.0;
      }
#pragma unroll
      for (int u = 0; u < kFineIlp; ++u) {
        const uint32_t i = i0 + u * kFineThreads;
        if (i >= n) continue;
        const uint32_t q = atomicAdd(&s_cu[energy_bin(pv[u]) & fmask], 1u);
        dst[q] = pv[u];
        if (idst) idst[q] = isrc[i];
      }
    }
    return;
  }
  uint32_t lo = 0;  // first bin of the window
  while (lo < nf) {
    if (t == 0) {
      // last bin hi with s_st[hi + 1] - s_st[lo] <= cap (at least lo)
      const uint32_t o = s_st[lo];
      uint32_t a = lo, b = nf;  // invariant: bins [lo, a] fit
      while (b - a > 1) {
        const uint32_t m = (a + b) >> 1;
        if (s_st[m + 1] - o <= cap) a = m; else b = m;
      }
      s_win[0] = a;
      s_win[1] = s_st[a + 1] - o <= cap ? 1u : 0u;
    }
    __syncthreads();
    const uint32_t hi = s_win[0];
    const bool fits = s_win[1] != 0;
    const uint32_t o = s_st[lo], wn = s_st[hi + 1] - o;
    if (fits) {
      for (uint32_t f = lo + t; f <= hi; f += kFineThreads) s_cu[f] = s_st[f] - o;
      __syncthreads();
      for (uint32_t i0 = t; i0 < n; i0 += kFineIlp * kFineThreads) {
        double pv[kFineIlp];
#pragma unroll
        for (int u = 0; u < kFineIlp; ++u) {
          const uint32_t i = i0 + u * kFineThreads;
          pv[u] = i < n ? src[i] : 0.0;
        }
#pragma unroll
        for (int u = 0; u < kFineIlp; ++u) {
          if (i0 + u * kFineThreads >= n) continue;
          const uint32_t f = energy_bin(pv[u]) & fmask;
          if (f >= lo && f <= hi) {
            const uint32_t q = atomicAdd(&s_cu[f], 1u);
            s_p[q] = pv[u];
            if (idst) s_i[q] = isrc[i0 + u * kFineThreads];
          }
        }
      }
      __syncthreads();
      for (uint32_t i = t; i < wn; i += kFineThreads) {
        dst[o + i] = s_p[i];
        if (idst) idst[o + i] = s_i[i];
      }
    } else {  // one bin larger than the window (skewed explicit inputs): in place
      if (t == 0) s_cu[lo] = o;
      __syncthreads();
      for (uint32_t i = t; i < n; i += kFineThreads) {
        const double p = src[i];
        if ((energy_bin(p) & fmask) == lo) {
          const uint32_t q = atomicAdd(&s_cu[lo], 1u);
          dst[q] = p;
          if (idst) idst[q] = isrc[i];
        }
      }
    }
    __syncthreads();
    lo = hi + 1;
  }
}

// ------------------------------------------------------------- A4 -- A8 ---
// Bracket index k_n for the lookup's energy through the grid's structure.
template <int GT>
__device__ __forceinline__ int32_t bracket_of(const Params& P, int32_t gidx, int32_t n, double p) {
  if (GT == XS_GRID_UNIONIZED)
    return P.index ? __ldg(P.index + static_cast<int64_t>(gidx) * P.I + n)
                   : __ldg(P.index_t + static_cast<int64_t>(n) * P.NU + gidx);
  const double* rec = P.grid + static_cast<int64_t>(n) * P.N * 6;
  if (GT == XS_GRID_HASH) return hash_bracket(P.index, P.I, P.B, gidx, n, rec, P.N, p);
  return nuclide_bracket(rec, P.N, p);
}

constexpr int kGatherThreads = 256;
constexpr int kG = 3;                 // lanes per lookup
constexpr int kLPT = 32 / kG;         // lookups per warp task (10)

// Record at bucket position pos: A2 batches go through the permutation
// (tmp holds the bin rank in idx; the batch index is the permutation value).
__device__ __forceinline__ LookupRec load_rec(const Params& P, uint32_t pos) {
  if (P.sp) {  // partitioned A2: energies (and positions) in sorted order, no u
    LookupRec r;
    r.p = P.sp[pos];
    r.idx = P.sidx ? P.sidx[pos] : 0u;
    r.gidx = 0;
    return r;
  }
  if (P.perm) {
    const uint32_t i = __ldg(P.perm + pos);
    LookupRec r = P.tmp[i];
    r.idx = i;
    return r;
  }
  return P.recs[pos];
}

struct alignas(16) MatEntry {
  double conc;
  uint32_t noff;  // n * N: first record of nuclide n
  int32_t n;
};

struct alignas(16) GatherSmem {
  int32_t num[kMaxMats];
  uint32_t off[kMaxMats + 1];   // bucket start of material m
  uint32_t cnt[kMaxMats];
  uint32_t toff[kMaxMats + 1];  // first task of material m
};

// Per-lookup view of the acceleration structure for A4: the unionized index
// row IG[u], or the two hash rows HG[b], HG[b+1].
template <int GT>
struct RowView {
  const int32_t* r0;
  const int32_t* r1;
  __device__ __forceinline__ RowView(const Params& P, int32_t gidx) {
    if (GT == XS_GRID_UNIONIZED) {
      r0 = P.index ? P.index + static_cast<int64_t>(gidx) * P.I : nullptr;
      r1 = r0;
    } else if (GT == XS_GRID_HASH) {
      r0 = P.index + static_cast<int64_t>(gidx) * P.I;
      r1 = gidx == P.B - 1 ? nullptr : r0 + P.I;
    } else {
      r0 = r1 = nullptr;
    }
  }
  // bracket k_n(p) of nuclide n whose records start at record index noff
  __device__ __forceinline__ int32_t bracket(const Params& P, int32_t n, uint32_t noff,
                                             double p) const {
    if (GT == XS_GRID_UNIONIZED) return __ldg(r0 + n);
    const double* rec = P.grid + static_cast<uint64_t>(noff) * 6;
    if (GT == XS_GRID_NUCLIDE) return nuclide_bracket(rec, P.N, p);
    const int64_t N = P.N;
    const int64_t u_lo = __ldg(r0 + n);
    const int64_t u_hi = r1 ? static_cast<int64_t>(__ldg(r1 + n)) + 1 : N - 1;
    int64_t lower;
    if (p <= rec_energy(rec, u_lo))
      lower = u_lo;
    else if (p >= rec_energy(rec, u_hi))
      lower = N - 1;
    else
      lower = bracket_search_rec(rec, u_lo, u_hi, p);
    return static_cast<int32_t>(lower == N - 1 ? N - 2 : lower);
  }
};

// U = nuclides per round per group (multiple of kG).
//
// Control flow is warp-uniform by construction (all 10 groups of a warp
// serve the same material, so they walk the same nuclide list); lanes that
// have no lookup (tail of a bucket, lanes 30-31) run the same instructions
// with their loads predicated off.  Every shuffle is executed by all 32
// lanes, outside any branch, and the interpolation weight is computed by
// every lane from its own chunk (only lane r = 0's value, from the energy
// chunk, is used) so the U divisions of a round are independent and
// branch-free.  Record addresses are 32-bit record indices (I*N < 2^31,
// checked at init) scaled once: n*N is precomputed per material slot in
// shared memory.
template <int GT, int U, int MINB, bool CHECK>
__global__ void __launch_bounds__(kGatherThreads, MINB) k_gather(Params P) {
  if (gated_off(P)) return;
  static_assert(U % kG == 0, "U must be a multiple of the group size");
  constexpr int Q = U / kG;
  extern __shared__ __align__(16) unsigned char smem_raw[];
  GatherSmem& S = *reinterpret_cast<GatherSmem*>(smem_raw);
  const int tab = P.n_mats * P.max_nucs;
  // material slot j of material m: {conc, record offset n*N, nuclide n},
  // one 16-B shared-memory entry (a single broadcast load per nuclide step)
  MatEntry* s_tab = reinterpret_cast<MatEntry*>(smem_raw + sizeof(GatherSmem));
  for (int t = threadIdx.x; t < tab; t += blockDim.x) {
    const int32_t n = P.mats[t];
    MatEntry me;
    me.conc = P.concs[t];
    me.noff = n >= 0 ? static_cast<uint32_t>(n) * static_cast<uint32_t>(P.N) : 0u;
    me.n = n;
    s_tab[t] = me;
  }
  if (threadIdx.x == 0) {
    uint32_t run = 0, trun = 0;
    for (int m = 0; m < P.n_mats; ++m) {
      const uint32_t c = P.counts[m];
      S.num[m] = P.num_nucs[m];
      S.off[m] = run;
      S.cnt[m] = c;
      S.toff[m] = trun;
      run += c;
      trun += (c + kLPT - 1) / kLPT;
    }
    S.off[P.n_mats] = run;
    S.toff[P.n_mats] = trun;
  }
  __syncthreads();

  const int lane = threadIdx.x & 31;
  const int g = lane / kG;
  const int r = lane - g * kG;
  const int base = g * kG;
  const uint32_t total_tasks = S.toff[P.n_mats];
  const uint32_t warps_per_block = blockDim.x >> 5;
  const uint32_t gw = blockIdx.x * warps_per_block + (threadIdx.x >> 5);
  const uint32_t nw = gridDim.x * warps_per_block;
  const double2* __restrict__ grid2 = reinterpret_cast<const double2*>(P.grid) + r;

  unsigned long long acc_v = 0, acc_n = 0;
  int m = 0;
  for (uint32_t task = gw; task < total_tasks; task += nw) {
    while (task >= S.toff[m + 1]) ++m;  // tasks are visited in increasing order
    const uint32_t slot = (task - S.toff[m]) * kLPT + g;
    const bool valid = (g < kLPT) && (slot < S.cnt[m]);
    LookupRec rec{0.5, 0u, 0};
    if (valid) {
      rec = load_rec(P, S.off[m] + slot);
    }
    const double p = rec.p;
    const int nn = valid ? S.num[m] : 0;   // invalid lanes load nothing
    const int nw_loop = S.num[m];           // warp-uniform trip count
    const MatEntry* row = s_tab + m * P.max_nucs;
    const RowView<GT> rv(P, valid ? rec.gidx : 0);

    double acc_a = 0.0, acc_b = 0.0;
    int32_t knext[Q];
#pragma unroll
    for (int q = 0; q < Q; ++q) {
      const int j = r + q * kG;
      int32_t kq = 0;
      if (j < nn) {
        const MatEntry me = row[j];
        kq = rv.bracket(P, me.n, me.noff, p);
      }
      knext[q] = kq;
    }
    // One round = U consecutive nuclides of the list.  Full rounds run
    // without any per-nuclide predicate; the (at most one) partial round at
    // the end of the list runs the TAIL instantiation.
    auto round = [&](const int j0, auto tail_tag) {
      constexpr bool TAIL = decltype(tail_tag)::value;
      int32_t kcur[Q];
#pragma unroll
      for (int q = 0; q < Q; ++q) kcur[q] = knext[q];
      // A4 for the next round (overlaps this round's pair gathers)
#pragma unroll
      for (int q = 0; q < Q; ++q) {
        const int j = j0 + U + r + q * kG;
        int32_t kq = 0;
        if (j < nn) {
          const MatEntry me = row[j];
          kq = rv.bracket(P, me.n, me.noff, p);
        }
        knext[q] = kq;
      }
      // A5: 96-B record pairs; lane r loads chunk r of the low and high
      // record.  A lane without a lookup has k = 0 and reads the nuclide's
      // first pair; in the tail round, slots past the end of the list read
      // the grid's first pair: always valid memory, never accumulated.
      double2 lo[U], hi[U];
      double cc[U];
#pragma unroll
      for (int t = 0; t < U; ++t) {
        const int j = j0 + t;
        const int32_t kt = __shfl_sync(0xffffffffu, kcur[t / kG], base + (t % kG));
        const MatEntry me = row[TAIL ? (j < nw_loop ? j : 0) : j];
        cc[t] = me.conc;
        uint32_t off = me.noff + static_cast<uint32_t>(kt);
        if (TAIL) off = j < nw_loop ? off : 0u;
        const double2* pr = grid2 + static_cast<uint64_t>(off) * 3;
        lo[t] = __ldg(pr);
        hi[t] = __ldg(pr + 3);
      }
      // A6: f = (hi.E - p) / (hi.E - lo.E), correctly rounded, every lane
      // (lane r = 0 holds the energies; the other lanes' values are unused)
      double fl[U];
      bool fast = true;
#pragma unroll
      for (int t = 0; t < U; ++t) {
        const double an = dsub(hi[t].x, p), bd = dsub(hi[t].x, lo[t].x);
        fl[t] = div_nr(an, bd);
        if (CHECK) fast &= (r != 0) || div_in_range(an, bd);
      }
      if (CHECK && !__all_sync(0xffffffffu, fast)) {  // rare: extreme data
#pragma unroll
        for (int t = 0; t < U; ++t)
          if (r == 0) fl[t] = ddiv(dsub(hi[t].x, p), dsub(hi[t].x, lo[t].x));
      }
      // A6 + A7 in list order
#pragma unroll
      for (int t = 0; t < U; ++t) {
        const int j = j0 + t;
        const double f = __shfl_sync(0xffffffffu, fl[t], base);
        const double xa = dsub(hi[t].x, dmul(f, dsub(hi[t].x, lo[t].x)));
        const double xb = dsub(hi[t].y, dmul(f, dsub(hi[t].y, lo[t].y)));
        if (!TAIL || j < nw_loop) {  // warp-uniform
          const double c = cc[t];
          acc_a = dadd(acc_a, dmul(xa, c));
          acc_b = dadd(acc_b, dmul(xb, c));
        }
      }
    };
    int j0 = 0;
    for (; j0 + U <= nw_loop; j0 += U) round(j0, std::false_type{});
    if (j0 < nw_loop) round(j0, std::true_type{});
    // A8: channels (t, s, a, f, nf) = (b@r0, a@r1, b@r1, a@r2, b@r2)
    double M[5];
    M[0] = __shfl_sync(0xffffffffu, acc_b, base);
    M[1] = __shfl_sync(0xffffffffu, acc_a, base + 1);
    M[2] = __shfl_sync(0xffffffffu, acc_b, base + 1);
    M[3] = __shfl_sync(0xffffffffu, acc_a, base + 2);
    M[4] = __shfl_sync(0xffffffffu, acc_b, base + 2);
    if (valid && r == 0) {
      double mx = -1.0;
      int vi = 0;
#pragma unroll
      for (int c = 0; c < 5; ++c)
        if (M[c] > mx) {
          mx = M[c];
          vi = c;
        }
      acc_v += static_cast<unsigned long long>(vi + 1);
      acc_n += 1;
      if (P.out_v) P.out_v[rec.idx] = vi + 1;
      if (P.out_M) {
        double* o = P.out_M + static_cast<uint64_t>(rec.idx) * 5;
#pragma unroll
        for (int c = 0; c < 5; ++c) o[c] = M[c];
      }
    }
  }
  // block reduction of the verification sums; one atomic pair per block
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    acc_v += __shfl_xor_sync(0xffffffffu, acc_v, o);
    acc_n += __shfl_xor_sync(0xffffffffu, acc_n, o);
  }
  __shared__ unsigned long long s_red[2][kGatherThreads / 32];
  if (lane == 0) {
    s_red[0][threadIdx.x >> 5] = acc_v;
    s_red[1][threadIdx.x >> 5] = acc_n;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long v = 0, n = 0;
    for (uint32_t w = 0; w < warps_per_block; ++w) {
      v += s_red[0][w];
      n += s_red[1][w];
    }
    if (n) {
      atomicAdd(P.vsum, v);
      atomicAdd(P.vsum + 1, n);
    }
  }
}

// --------------------------------------------- thread-per-lookup gather ---
// k_gather_t: for energy-sorted batches (XS_FLAG_SORT).  A warp takes 32*R
// consecutive lookups of one material bucket; lane l owns the R adjacent
// lookups R*l .. R*l+R-1.  After A2 they lie within ~1e-5 of each other in
// energy, so
//   * for each nuclide the lane's R lookups almost always share one record
//     pair: the lane loads the pair once (6 x 128-bit loads) and reloads
//     only when a later lookup's bracket differs (rare, divergent);
//   * the 32 lanes read the same or neighbouring pairs (1-2 cache lines per
//     load instruction) and, with the column-layout index grid IGT[n][u],
//     neighbouring index entries.
// Each lane does its own exact division and all five channels, and
// accumulates each lookup in list order: no shuffles, every lane's
// arithmetic useful.  R = 1 is plain thread-per-lookup.
template <int GT, int R, int U, int MINB, bool CHECK>
__global__ void __launch_bounds__(kGatherThreads, MINB) k_gather_t(Params P) {
  if (gated_off(P)) return;
  constexpr int kTask = 32 * R;
  extern __shared__ __align__(16) unsigned char smem_raw[];
  GatherSmem& S = *reinterpret_cast<GatherSmem*>(smem_raw);
  const int tab = P.n_mats * P.max_nucs;
  MatEntry* s_tab = reinterpret_cast<MatEntry*>(smem_raw + sizeof(GatherSmem));
  for (int t = threadIdx.x; t < tab; t += blockDim.x) {
    const int32_t n = P.mats[t];
    MatEntry me;
    me.conc = P.concs[t];
    me.noff = n >= 0 ? static_cast<uint32_t>(n) * static_cast<uint32_t>(P.N) : 0u;
    me.n = n;
    s_tab[t] = me;
  }
  if (threadIdx.x == 0) {
    uint32_t run = 0, trun = 0;
    for (int m = 0; m < P.n_mats; ++m) {
      const uint32_t c = P.counts[m];
      S.num[m] = P.num_nucs[m];
      S.off[m] = run;
      S.cnt[m] = c;
      S.toff[m] = trun;
      run += c;
      trun += (c + kTask - 1) / kTask;
    }
    S.off[P.n_mats] = run;
    S.toff[P.n_mats] = trun;
  }
  __syncthreads();

  const int lane = threadIdx.x & 31;
  const uint32_t total_tasks = S.toff[P.n_mats];
  const uint32_t warps_per_block = blockDim.x >> 5;
  const uint32_t gw = blockIdx.x * warps_per_block + (threadIdx.x >> 5);
  const uint32_t nw = gridDim.x * warps_per_block;
  const double2* __restrict__ grid2 = reinterpret_cast<const double2*>(P.grid);

  unsigned long long acc_v = 0, acc_n = 0;
  int m = 0;
  for (uint32_t task = gw; task < total_tasks; task += nw) {
    while (task >= S.toff[m + 1]) ++m;
    const uint32_t slot0 = (task - S.toff[m]) * kTask + lane * R;
    double p[R];
    int32_t gidx[R];
    uint32_t idx[R];
    bool valid[R];
#pragma unroll
    for (int r = 0; r < R; ++r) {
      valid[r] = slot0 + r < S.cnt[m];
      LookupRec rec{0.5, 0u, 0};
      if (valid[r]) {
        const uint32_t pos = S.off[m] + slot0 + r;
        rec = load_rec(P, pos);
      }
      p[r] = rec.p;
      gidx[r] = rec.gidx;
      idx[r] = rec.idx;
    }
    const int nn = S.num[m];
    const MatEntry* row = s_tab + m * P.max_nucs;

    // bracket k_n of lookup r (A4) through the grid's index structure
    auto bracket = [&](const MatEntry& me, int r) -> int32_t {
      if (GT == XS_GRID_UNIONIZED) {
        if (!P.index) return __ldg(P.index_t + static_cast<int64_t>(me.n) * P.NU + gidx[r]);
        return __ldg(P.index + static_cast<int64_t>(gidx[r]) * P.I + me.n);
      }
      const RowView<GT> rv(P, gidx[r]);
      return rv.bracket(P, me.n, me.noff, p[r]);
    };

    double M[R][5];
#pragma unroll
    for (int r = 0; r < R; ++r)
#pragma unroll
      for (int c = 0; c < 5; ++c) M[r][c] = 0.0;

    // A4.  Unionized grid: every lookup reads its own index-grid entry
    // (IGT[n][u]: the lane's R lookups hit neighbouring entries), prefetched
    // one round ahead.  Hash / nuclide grids (whose A4 is a chain of
    // dependent loads): the lane's first lookup runs the full search; each
    // later lookup starts from the bracket before it and, when the pair's
    // energies show it is not its own (E[k] <= p < E[k+1], clamped ends),
    // walks to the neighbouring interval — an exact local search, so every
    // lookup still gets k_n(p).
    constexpr bool kAllIdx = GT == XS_GRID_UNIONIZED;
    constexpr int RK = kAllIdx ? R : 1;
    const int32_t kmax = static_cast<int32_t>(P.N - 2);
    int32_t knext[U][RK];
#pragma unroll
    for (int t = 0; t < U; ++t)
#pragma unroll
      for (int r = 0; r < RK; ++r) knext[t][r] = t < nn ? bracket(row[t], r) : 0;

    for (int j0 = 0; j0 < nn; j0 += U) {
      int32_t kcur[U][RK];
#pragma unroll
      for (int t = 0; t < U; ++t)
#pragma unroll
        for (int r = 0; r < RK; ++r) kcur[t][r] = knext[t][r];
#pragma unroll
      for (int t = 0; t < U; ++t) {
        const int j = j0 + U + t;
#pragma unroll
        for (int r = 0; r < RK; ++r) knext[t][r] = j < nn ? bracket(row[j], r) : 0;
      }
      // A5: the record pair of each nuclide's first bracket
      double2 c[U][6];
      double cc[U];
      uint32_t noff[U];
#pragma unroll
      for (int t = 0; t < U; ++t) {
        const int j = j0 + t;
        const MatEntry me = row[j < nn ? j : 0];
        cc[t] = me.conc;
        noff[t] = j < nn ? me.noff : 0u;
        const double2* pr = grid2 + static_cast<uint64_t>(noff[t] + (j < nn ? kcur[t][0] : 0)) * 3;
#pragma unroll
        for (int q = 0; q < 6; ++q) c[t][q] = __ldg(pr + q);
      }
#pragma unroll
      for (int t = 0; t < U; ++t) {
        if (j0 + t < nn) {  // warp-uniform
          // per pair: lo = (E, t | s, a | f, nf) = c[0..2], hi = c[3..5];
          // bd, its reciprocal and the channel differences are shared by
          // every lookup of the lane that falls in this pair
          int32_t k = kcur[t][0];
          double bd, rc, d0, d1, d2, d3, d4;
          auto pair_terms = [&]() {
            bd = dsub(c[t][3].x, c[t][0].x);
            rc = recip_nr(bd);
            d0 = dsub(c[t][3].y, c[t][0].y);
            d1 = dsub(c[t][4].x, c[t][1].x);
            d2 = dsub(c[t][4].y, c[t][1].y);
            d3 = dsub(c[t][5].x, c[t][2].x);
            d4 = dsub(c[t][5].y, c[t][2].y);
          };
          pair_terms();
#pragma unroll
          for (int r = 0; r < R; ++r) {
            if (r > 0) {
              int32_t kr;
              if (kAllIdx) {
                kr = kcur[t][kAllIdx ? r : 0];
              } else {
                kr = k;
                if (valid[r]) {
                  const double* rec = P.grid + static_cast<uint64_t>(noff[t]) * 6;
                  while (kr > 0 && p[r] < rec_energy(rec, kr)) --kr;
                  while (kr < kmax && p[r] >= rec_energy(rec, kr + 1)) ++kr;
                }
              }
              if (kr != k) {  // rare: this lookup lies in another interval
                k = kr;
                const double2* pr = grid2 + static_cast<uint64_t>(noff[t] + k) * 3;
#pragma unroll
                for (int q = 0; q < 6; ++q) c[t][q] = __ldg(pr + q);
                pair_terms();
              }
            }
            // A6: f = (hi.E - p) / (hi.E - lo.E), correctly rounded
            const double an = dsub(c[t][3].x, p[r]);
            double f = div_by_recip(an, bd, rc);
            if (CHECK && !div_in_range(an, bd)) f = ddiv(an, bd);
            // x_c = hi_c - f * (hi_c - lo_c); A7: M_c += x_c * conc
            const double x0 = dsub(c[t][3].y, dmul(f, d0));
            const double x1 = dsub(c[t][4].x, dmul(f, d1));
            const double x2 = dsub(c[t][4].y, dmul(f, d2));
            const double x3 = dsub(c[t][5].x, dmul(f, d3));
            const double x4 = dsub(c[t][5].y, dmul(f, d4));
            M[r][0] = dadd(M[r][0], dmul(x0, cc[t]));
            M[r][1] = dadd(M[r][1], dmul(x1, cc[t]));
            M[r][2] = dadd(M[r][2], dmul(x2, cc[t]));
            M[r][3] = dadd(M[r][3], dmul(x3, cc[t]));
            M[r][4] = dadd(M[r][4], dmul(x4, cc[t]));
          }
        }
      }
    }
#pragma unroll
    for (int r = 0; r < R; ++r) {
      if (!valid[r]) continue;
      double mx = -1.0;
      int vi = 0;
#pragma unroll
      for (int c = 0; c < 5; ++c)
        if (M[r][c] > mx) {
          mx = M[r][c];
          vi = c;
        }
      acc_v += static_cast<unsigned long long>(vi + 1);
      acc_n += 1;
      if (P.out_v) P.out_v[idx[r]] = vi + 1;
      if (P.out_M) {
        double* o = P.out_M + static_cast<uint64_t>(idx[r]) * 5;
#pragma unroll
        for (int c = 0; c < 5; ++c) o[c] = M[r][c];
      }
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    acc_v += __shfl_xor_sync(0xffffffffu, acc_v, o);
    acc_n += __shfl_xor_sync(0xffffffffu, acc_n, o);
  }
  __shared__ unsigned long long s_red[2][kGatherThreads / 32];
  if (lane == 0) {
    s_red[0][threadIdx.x >> 5] = acc_v;
    s_red[1][threadIdx.x >> 5] = acc_n;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long v = 0, n = 0;
    for (uint32_t w = 0; w < warps_per_block; ++w) {
      v += s_red[0][w];
      n += s_red[1][w];
    }
    if (n) {
      atomicAdd(P.vsum, v);
      atomicAdd(P.vsum + 1, n);
    }
  }
}

// ------------------------------------------- TMA-staged sorted gather ------
// k_gather_s: for energy-sorted batches.  A warp owns a task of 32*R
// consecutive lookups of one material (lane l: lookups R*l..R*l+R-1, ordered
// by energy).  Because the task is energy-sorted, for every nuclide n its
// lookups' brackets lie in [k_lo, k_hi] with k_lo / k_hi the brackets of the
// task's lowest / highest energy (A4 via the index grid for those two
// lookups: IGT is monotone in u).  So per nuclide the warp needs one
// contiguous window of records [k_lo, k_hi + 1].  One lane streams these
// windows into shared memory with TMA bulk copies (cp.async.bulk +
// mbarrier), D nuclides ahead; every lane then walks its lookups through the
// window (an exact search: E[k] <= p < E[k+1], clamped) and interpolates
// from shared memory.  Record pairs never wait in registers for global
// memory and each warp reads each window from L2/HBM once.  Windows larger
// than W records (sparse tasks) are read in place from global memory.
template <int GT, int R, int D, int W, int NW, bool CHECK>
__global__ void __launch_bounds__(32 * NW, 1) k_gather_s(Params P) {
  if (gated_off(P)) return;
  constexpr int kTask = 32 * R;
  extern __shared__ __align__(16) unsigned char smem_raw[];
  GatherSmem& S = *reinterpret_cast<GatherSmem*>(smem_raw);
  const int tab = P.n_mats * P.max_nucs;
  MatEntry* s_tab = reinterpret_cast<MatEntry*>(smem_raw + sizeof(GatherSmem));
  // per warp: D windows of W records, D mbarriers, k_lo/k_hi per nuclide
  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  unsigned char* wbase = reinterpret_cast<unsigned char*>(s_tab + tab);
  const size_t win_bytes = static_cast<size_t>(D) * W * 48;
  const size_t kw_bytes = ((static_cast<size_t>(P.max_nucs) * 2 * 4 + 15) / 16) * 16;
  const size_t per_warp = win_bytes + kw_bytes + ((D * 8 + 15) / 16) * 16;
  unsigned char* mine = wbase + per_warp * warp;
  double2* s_win = reinterpret_cast<double2*>(mine);                  // [D][W*3]
  int32_t* s_klo = reinterpret_cast<int32_t*>(mine + win_bytes);      // [max_nucs]
  int32_t* s_khi = s_klo + P.max_nucs;
  uint64_t* s_bar = reinterpret_cast<uint64_t*>(mine + win_bytes + kw_bytes);

  for (int t = threadIdx.x; t < tab; t += blockDim.x) {
    const int32_t n = P.mats[t];
    MatEntry me;
    me.conc = P.concs[t];
    me.noff = n >= 0 ? static_cast<uint32_t>(n) * static_cast<uint32_t>(P.N) : 0u;
    me.n = n;
    s_tab[t] = me;
  }
  if (threadIdx.x == 0) {
    uint32_t run = 0, trun = 0;
    for (int m = 0; m < P.n_mats; ++m) {
      const uint32_t c = P.counts[m];
      S.num[m] = P.num_nucs[m];
      S.off[m] = run;
      S.cnt[m] = c;
      S.toff[m] = trun;
      run += c;
      trun += (c + kTask - 1) / kTask;
    }
    S.off[P.n_mats] = run;
    S.toff[P.n_mats] = trun;
  }
  if (lane == 0) {
    for (int d = 0; d < D; ++d) mbar_init(&s_bar[d], 1);
    mbar_fence_init();
  }
  __syncthreads();

  const uint32_t total_tasks = S.toff[P.n_mats];
  const uint32_t gw = blockIdx.x * NW + warp;
  const uint32_t nwarps = gridDim.x * NW;
  const double2* __restrict__ grid2 = reinterpret_cast<const double2*>(P.grid);
  const int32_t kmax = static_cast<int32_t>(P.N - 2);
  uint32_t phase = 0;  // parity bit per slot

  unsigned long long acc_v = 0, acc_n = 0;
  int m = 0;
  for (uint32_t task = gw; task < total_tasks; task += nwarps) {
    while (task >= S.toff[m + 1]) ++m;
    const uint32_t slot0 = (task - S.toff[m]) * kTask + lane * R;
    double p[R];
    int32_t gidx[R];
    uint32_t idx[R];
    bool valid[R];
#pragma unroll
    for (int r = 0; r < R; ++r) {
      valid[r] = slot0 + r < S.cnt[m];
      LookupRec rec{0.5, 0u, 0};
      if (valid[r]) rec = load_rec(P, S.off[m] + slot0 + r);
      p[r] = rec.p;
      gidx[r] = rec.gidx;
      idx[r] = rec.idx;
    }
    // order the lane's lookups by energy, valid ones first
#pragma unroll
    for (int pass = 0; pass < R; ++pass) {
#pragma unroll
      for (int r = pass & 1; r + 1 < R; r += 2) {
        const bool swap = (valid[r + 1] && !valid[r]) ||
                          (valid[r] == valid[r + 1] && p[r + 1] < p[r]);
        if (swap) {
          const double tp = p[r]; p[r] = p[r + 1]; p[r + 1] = tp;
          const int32_t tg = gidx[r]; gidx[r] = gidx[r + 1]; gidx[r + 1] = tg;
          const uint32_t ti = idx[r]; idx[r] = idx[r + 1]; idx[r + 1] = ti;
          const bool tv = valid[r]; valid[r] = valid[r + 1]; valid[r + 1] = tv;
        }
      }
    }
    // task extremes: lowest / highest energy (and unionized index) of the
    // task's valid lookups (u is monotone in p)
    double plo = valid[0] ? p[0] : 2.0, phi = -1.0;
    int32_t ulo = valid[0] ? gidx[0] : 0x7fffffff, uhi = -1;
#pragma unroll
    for (int r = 0; r < R; ++r)
      if (valid[r]) {
        phi = p[r];
        uhi = gidx[r];
      }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      const double a = __shfl_xor_sync(0xffffffffu, plo, o);
      const double b = __shfl_xor_sync(0xffffffffu, phi, o);
      plo = a < plo ? a : plo;
      phi = b > phi ? b : phi;
    }
    if (GT == XS_GRID_UNIONIZED && !P.need_gidx) {
      // A3 for the task's extreme energies (u is monotone in p)
      ulo = union_index_tab(P, plo);
      uhi = union_index_tab(P, phi);
    } else {
      ulo = __reduce_min_sync(0xffffffffu, ulo);
      uhi = __reduce_max_sync(0xffffffffu, uhi);
    }
    // slots without a lookup take the lane's last valid energy (or the task
    // minimum) so that the hot loop needs no validity test
#pragma unroll
    for (int r = 0; r < R; ++r)
      if (!valid[r]) p[r] = r > 0 ? p[r - 1] : plo;
    const int nn = S.num[m];
    const MatEntry* row = s_tab + m * P.max_nucs;
    // A4 for the two extremes of every nuclide of the material
    for (int j = lane; j < nn; j += 32) {
      const MatEntry me = row[j];
      int32_t klo, khi;
      if (GT == XS_GRID_UNIONIZED) {
        if (P.index_t) {
          klo = __ldg(P.index_t + static_cast<int64_t>(me.n) * P.NU + ulo);
          khi = __ldg(P.index_t + static_cast<int64_t>(me.n) * P.NU + uhi);
        } else {
          klo = __ldg(P.index + static_cast<int64_t>(ulo) * P.I + me.n);
          khi = __ldg(P.index + static_cast<int64_t>(uhi) * P.I + me.n);
        }
      } else {
        const RowView<GT> rlo(P, GT == XS_GRID_HASH ? hash_bin(plo, P.du, P.B) : 0);
        const RowView<GT> rhi(P, GT == XS_GRID_HASH ? hash_bin(phi, P.du, P.B) : 0);
        klo = rlo.bracket(P, me.n, me.noff, plo);
        khi = rhi.bracket(P, me.n, me.noff, phi);
      }
      s_klo[j] = klo;
      s_khi[j] = khi;
    }
    __syncwarp();
    // A5 producer: window of nuclide j into slot j % D
    auto issue = [&](int j) {
      const int d = j % D;
      const int32_t klo = s_klo[j], khi = s_khi[j];
      const int32_t w = khi - klo + 2;  // records klo .. khi+1
      if (w <= W) {
        const double2* src = grid2 + static_cast<uint64_t>(row[j].noff + static_cast<uint32_t>(klo)) * 3;
        mbar_arrive_expect_tx(&s_bar[d], static_cast<uint32_t>(w) * 48u);
        bulk_copy_g2s(s_win + d * W * 3, src, static_cast<uint32_t>(w) * 48u, &s_bar[d]);
      } else {
        mbar_arrive_expect_tx(&s_bar[d], 0u);  // read in place from global memory
      }
    };
    if (lane == 0)
      for (int j = 0; j < D && j < nn; ++j) issue(j);

    double M[R][5];
#pragma unroll
    for (int r = 0; r < R; ++r)
#pragma unroll
      for (int c = 0; c < 5; ++c) M[r][c] = 0.0;

    for (int j = 0; j < nn; ++j) {
      const int d = j % D;
      mbar_wait(&s_bar[d], (phase >> d) & 1u);
      phase ^= 1u << d;
      const MatEntry me = row[j];
      const int32_t klo = s_klo[j], khi = s_khi[j];
      const double2* win = (khi - klo + 2 <= W)
                               ? s_win + d * W * 3
                               : grid2 + static_cast<uint64_t>(me.noff + static_cast<uint32_t>(klo)) * 3;
      int32_t k = klo;
      double2 c[6];
      auto load_pair = [&]() {
        const double2* pr = win + (k - klo) * 3;
#pragma unroll
        for (int q = 0; q < 6; ++q) c[q] = pr[q];
      };
      load_pair();
      double bd, rc, d0, d1, d2, d3, d4;
      auto pair_terms = [&]() {
        bd = dsub(c[3].x, c[0].x);
        rc = recip_nr(bd);
        d0 = dsub(c[3].y, c[0].y);
        d1 = dsub(c[4].x, c[1].x);
        d2 = dsub(c[4].y, c[1].y);
        d3 = dsub(c[5].x, c[2].x);
        d4 = dsub(c[5].y, c[2].y);
      };
      pair_terms();
#pragma unroll
      for (int r = 0; r < R; ++r) {
        // A4 (exact local search): advance to k_n(p) within [klo, khi] by
        // bisection on the window energies (E[k] <= p is known; k_n(p) <= khi)
        if (k < khi && p[r] >= c[3].x) {
          int32_t lo = k + 1, hi = khi + 1;
          while (hi - lo > 1) {
            const int32_t mid = (lo + hi) >> 1;
            if (win[(mid - klo) * 3].x <= p[r])
              lo = mid;
            else
              hi = mid;
          }
          k = lo;
          load_pair();
          pair_terms();
        }
        const double an = dsub(c[3].x, p[r]);
        double f = div_by_recip(an, bd, rc);
        if (CHECK && !div_in_range(an, bd)) f = ddiv(an, bd);
        const double x0 = dsub(c[3].y, dmul(f, d0));
        const double x1 = dsub(c[4].x, dmul(f, d1));
        const double x2 = dsub(c[4].y, dmul(f, d2));
        const double x3 = dsub(c[5].x, dmul(f, d3));
        const double x4 = dsub(c[5].y, dmul(f, d4));
        M[r][0] = dadd(M[r][0], dmul(x0, me.conc));
        M[r][1] = dadd(M[r][1], dmul(x1, me.conc));
        M[r][2] = dadd(M[r][2], dmul(x2, me.conc));
        M[r][3] = dadd(M[r][3], dmul(x3, me.conc));
        M[r][4] = dadd(M[r][4], dmul(x4, me.conc));
      }
      __syncwarp();  // every lane is done with slot d
      if (lane == 0 && j + D < nn) issue(j + D);
    }
    (void)kmax;
#pragma unroll
    for (int r = 0; r < R; ++r) {
      if (!valid[r]) continue;
      double mx = -1.0;
      int vi = 0;
#pragma unroll
      for (int c = 0; c < 5; ++c)
        if (M[r][c] > mx) {
          mx = M[r][c];
          vi = c;
        }
      acc_v += static_cast<unsigned long long>(vi + 1);
      acc_n += 1;
      if (P.out_v) P.out_v[idx[r]] = vi + 1;
      if (P.out_M) {
        double* o = P.out_M + static_cast<uint64_t>(idx[r]) * 5;
#pragma unroll
        for (int c = 0; c < 5; ++c) o[c] = M[r][c];
      }
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    acc_v += __shfl_xor_sync(0xffffffffu, acc_v, o);
    acc_n += __shfl_xor_sync(0xffffffffu, acc_n, o);
  }
  __shared__ unsigned long long s_red[2][NW];
  if (lane == 0) {
    s_red[0][warp] = acc_v;
    s_red[1][warp] = acc_n;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long v = 0, n = 0;
    for (int w = 0; w < NW; ++w) {
      v += s_red[0][w];
      n += s_red[1][w];
    }
    if (n) {
      atomicAdd(P.vsum, v);
      atomicAdd(P.vsum + 1, n);
    }
  }
}

// ------------------------------- TMA-staged sorted gather, interval table --
// k_gather_s3 (default for energy-sorted batches): the k_gather_s
// decomposition (warp = task of 32*R energy-sorted lookups of one material,
// lane = R consecutive lookups, per-nuclide window [k_lo, k_hi] staged in
// shared memory by TMA bulk copies), with the window holding entries of the
// interval table (grid_build.cu K0d: per record pair {E[k+1], gap,
// recip(gap), hi.c, hi.c - lo.c}) instead of raw records, so no pair-only
// arithmetic (5-DFMA reciprocal chain, 6 subtractions) runs in the timed
// loop: a lookup costs 4 FP64 ops for f and 4 per channel.
//  * Each lane finds the window entries of its first and last lookup by
//    warp-uniform binary lifting over the entries' upper energies (loads
//    clamped, no branches).  When every lane's lookups share one entry (the
//    common case: a fuel task spans ~0.6 intervals of a nuclide) the R
//    interpolations run as one straight-line block (R independent FP64
//    chains); otherwise every lookup reads its own entry.
//  * Windows are read with shared-memory loads on their own code path;
//    windows longer than W entries (sparse tasks) take a global-memory path.
//  * Bulk copies are issued D at a time by D lanes into a ring of 2D slots
//    (D to 2D nuclides ahead), completing on per-slot mbarriers.
// Window access for the staged gathers (16-B units u of an interval-table
// window): through a generic pointer to shared memory, through the read-only
// path from global memory, or through a 32-bit shared-memory address (no
// generic-to-shared conversion in the loop).
struct WinPtr {
  const double2* q;
  __device__ __forceinline__ double2 ld2(int u) const { return q[u]; }
  __device__ __forceinline__ float4 ld4f(int u) const { return *reinterpret_cast<const float4*>(q + u); }
  __device__ __forceinline__ double ld1(int u) const { return reinterpret_cast<const double*>(q + u)[0]; }
  __device__ __forceinline__ WinPtr at(int u) const { return WinPtr{q + u}; }
};
struct WinGlobal {
  const double2* q;
  __device__ __forceinline__ double2 ld2(int u) const { return __ldg(q + u); }
  __device__ __forceinline__ float4 ld4f(int u) const { return __ldg(reinterpret_cast<const float4*>(q + u)); }
  __device__ __forceinline__ double ld1(int u) const { return __ldg(reinterpret_cast<const double*>(q + u)); }
  __device__ __forceinline__ WinGlobal at(int u) const { return WinGlobal{q + u}; }
};
struct WinSmem {
  uint32_t a;  // shared-memory byte address
  __device__ __forceinline__ double2 ld2(int u) const {
    double2 v;
    asm volatile("ld.shared.v2.f64 {%0, %1}, [%2];" : "=d"(v.x), "=d"(v.y) : "r"(a + 16u * u));
    return v;
  }
  __device__ __forceinline__ float4 ld4f(int u) const {
    float4 v;
    asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];"
                 : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w)
                 : "r"(a + 16u * u));
    return v;
  }
  __device__ __forceinline__ double ld1(int u) const {
    double v;
    asm volatile("ld.shared.f64 %0, [%1];" : "=d"(v) : "r"(a + 16u * u));
    return v;
  }
  __device__ __forceinline__ WinSmem at(int u) const { return WinSmem{a + 16u * u}; }
};

// Same operations in the same order as the oracle (bit-identical M).
// Entry layout (7 x 16 B): {E[k+1], gap} {recip(gap), 0} {hi.c, hi.c - lo.c} x 5.
// A6 + A7 for lookups r in [r0, r1) that all lie in entry q (channel terms are
// read from the window per channel to keep register pressure low).
template <int R, bool CHECK, class Win>
__device__ __forceinline__ void iv_interp(const Win q, const double (&p)[R], double conc,
                                          double (&M)[R][5], int r0, int r1) {
  const double2 a0 = q.ld2(0), a1 = q.ld2(1);
  double f[R];
#pragma unroll
  for (int r = 0; r < R; ++r) {
    if (r < r0 || r >= r1) continue;
    const double an = dsub(a0.x, p[r]);
    f[r] = div_by_recip(an, a0.y, a1.x);
    if (CHECK && !div_in_range(an, a0.y)) f[r] = ddiv(an, a0.y);
  }
#pragma unroll
  for (int c = 0; c < 5; ++c) {
    const double2 hd = q.ld2(2 + c);
#pragma unroll
    for (int r = 0; r < R; ++r) {
      if (r < r0 || r >= r1) continue;
      M[r][c] = dadd(M[r][c], dmul(dsub(hd.x, dmul(f[r], hd.y)), conc));
    }
  }
}

// fp32 variant (R18): paired binary32 fused multiply-add (sm_100a FFMA2),
// one rounding per element.  Plain mul/add pairs are avoided on purpose:
// ptxas contracts f32x2 mul + add into FFMA2 even with .rn.
__device__ __forceinline__ float2 ffma2(float2 a, float2 b, float2 c) {
  uint64_t d;
  asm("fma.rn.f32x2 %0, %1, %2, %3;"
      : "=l"(d)
      : "l"(*reinterpret_cast<uint64_t*>(&a)), "l"(*reinterpret_cast<uint64_t*>(&b)),
        "l"(*reinterpret_cast<uint64_t*>(&c)));
  return *reinterpret_cast<float2*>(&d);
}

// Accumulators of the staged gather: M for R lookups and the A6 + A7 update
// from one interval-table entry q for lookups r in [r0, r1).
template <int R, bool CHECK>
struct AccF64 {  // binary64 (R10, R11): entry = K0d, 7 x 16 B
  static constexpr int kE = kIvDoubles / 2;
  double M[R][5];
  __device__ __forceinline__ void zero() {
#pragma unroll
    for (int r = 0; r < R; ++r)
#pragma unroll
      for (int c = 0; c < 5; ++c) M[r][c] = 0.0;
  }
  __device__ __forceinline__ double get(int r, int c) const { return M[r][c]; }
  __device__ __forceinline__ void flush() {}  // one accumulation level (R11)
  template <class Win>
  __device__ __forceinline__ void interp(const Win q, const double (&p)[R], double conc, int r0,
                                         int r1) {
    iv_interp<R, CHECK>(q, p, conc, M, r0, r1);
  }
};

// R18's accumulation block: nuclides are summed in blocks of kF32Block (list
// order); flush() after nuclides 15, 31, ... and after the last one
constexpr int kF32Block = 16;

template <int R, bool CHECK>
struct AccF32 {  // binary32 variant (R18): entry = K0e, 5 x 16 B
  static_assert(R % 2 == 0, "fp32 accumulators pair lookups");
  static constexpr int kE = kIv32Doubles / 2;
  float2 M[R / 2][5];  // block sums {lookup 2q, lookup 2q+1}
  float2 T[R / 2][5];  // totals
  __device__ __forceinline__ void zero() {
#pragma unroll
    for (int q = 0; q < R / 2; ++q)
#pragma unroll
      for (int c = 0; c < 5; ++c) M[q][c] = T[q][c] = make_float2(0.0f, 0.0f);
  }
  // T += B, B = 0 (fma(B, 1, T) is the correctly rounded sum)
  __device__ __forceinline__ void flush() {
#pragma unroll
    for (int q = 0; q < R / 2; ++q)
#pragma unroll
      for (int c = 0; c < 5; ++c) {
        T[q][c] = ffma2(M[q][c], make_float2(1.0f, 1.0f), T[q][c]);
        M[q][c] = make_float2(0.0f, 0.0f);
      }
  }
  __device__ __forceinline__ double get(int r, int c) const {
    return static_cast<double>((r & 1) ? T[r >> 1][c].y : T[r >> 1][c].x);
  }
  template <class Win>
  __device__ __forceinline__ void interp(const Win q, const double (&p)[R], double conc, int r0,
                                         int r1) {
    auto ldf = [&](int u) -> float4 { return q.ld4f(u); };
    const double2 a0 = q.ld2(0), a1 = q.ld2(1);
    float nf[R];  // -f, f = binary64 weight rounded once to binary32
#pragma unroll
    for (int r = 0; r < R; ++r) {
      if (r < r0 || r >= r1) continue;
      const double an = dsub(a0.x, p[r]);
      double f = div_by_recip(an, a0.y, a1.x);
      if (CHECK && !div_in_range(an, a0.y)) f = ddiv(an, a0.y);
      nf[r] = -__double2float_rn(f);
    }
    const float cf = __double2float_rn(conc);
    const float4 t0 = ldf(2), t1 = ldf(3), t2 = ldf(4);
    const float hh[5] = {t0.x, t0.z, t1.x, t1.z, t2.x};
    const float dd[5] = {t0.y, t0.w, t1.y, t1.w, t2.y};
#pragma unroll
    for (int c = 0; c < 5; ++c) {
#pragma unroll
      for (int qq = 0; qq < R / 2; ++qq) {
        const int ra = 2 * qq, rb = 2 * qq + 1;
        const bool ia = ra >= r0 && ra < r1, ib = rb >= r0 && rb < r1;
        if (ia && ib) {
          const float2 x = ffma2(make_float2(nf[ra], nf[rb]), make_float2(dd[c], dd[c]),
                                 make_float2(hh[c], hh[c]));
          M[qq][c] = ffma2(x, make_float2(cf, cf), M[qq][c]);
        } else if (ia) {
          M[qq][c].x = __fmaf_rn(__fmaf_rn(nf[ra], dd[c], hh[c]), cf, M[qq][c].x);
        } else if (ib) {
          M[qq][c].y = __fmaf_rn(__fmaf_rn(nf[rb], dd[c], hh[c]), cf, M[qq][c].y);
        }
      }
    }
  }
};

// One nuclide of a task: win = interval entries k_lo .. k_lo + n_int.
// i(p) = max{t in [0, n_int] : t = 0 or E[k_lo + t] <= p} by binary lifting
// (warp-uniform trip count; loads clamped so the loop has no branches).
template <int R, class Win, class Acc>
__device__ __forceinline__ void stage_nuclide_iv(const Win win, int n_int, double conc,
                                                 const double (&p)[R], Acc& acc) {
  constexpr int kE = Acc::kE;
  // E[k_lo + t] = first double of entry t - 1
  auto E = [&](int t) -> double { return win.ld1((t - 1) * kE); };
  if (n_int == 0) {  // one entry: every lookup of the task lies in it (warp-uniform)
    acc.interp(win, p, conc, 0, R);
    return;
  }
  if (n_int == 1) {  // two entries (the common multi-entry case): one shared probe
    const double e = E(1);
    int i[R];
#pragma unroll
    for (int r = 0; r < R; ++r) i[r] = e <= p[r] ? 1 : 0;
    if (__all_sync(0xffffffffu, i[0] == i[R - 1])) {  // p sorted within the lane
      acc.interp(win.at(i[0] * kE), p, conc, 0, R);
      return;
    }
#pragma unroll
    for (int r = 0; r < R; ++r) acc.interp(win.at(i[r] * kE), p, conc, r, r + 1);
    return;
  }
  int i0, iL;
  const int top = 1 << (31 - __clz(n_int));
  {
    i0 = iL = 0;
    for (int step = top; step > 0; step >>= 1) {
      const int t0 = i0 + step, tL = iL + step;
      const double e0 = E(t0 <= n_int ? t0 : n_int), eL = E(tL <= n_int ? tL : n_int);
      if (t0 <= n_int && e0 <= p[0]) i0 = t0;
      if (tL <= n_int && eL <= p[R - 1]) iL = tL;
    }
  }
  if (__all_sync(0xffffffffu, i0 == iL)) {
    acc.interp(win.at(i0 * kE), p, conc, 0, R);
    return;
  }
  int i[R];
  i[0] = i0;
  i[R - 1] = iL;
#pragma unroll
  for (int r = 1; r < R - 1; ++r) i[r] = i0;
  if (R > 2) {
    for (int step = top; step > 0; step >>= 1) {
#pragma unroll
      for (int r = 1; r < R - 1; ++r) {
        const int t = i[r] + step;
        const double e = E(t <= n_int ? t : n_int);
        if (t <= n_int && e <= p[r]) i[r] = t;
      }
    }
  }
#pragma unroll
  for (int r = 0; r < R; ++r) acc.interp(win.at(i[r] * kE), p, conc, r, r + 1);
}

template <int GT, int R, int D, int W, int NW, bool CHECK, bool DYN = false, bool F32 = false>
__global__ void __launch_bounds__(32 * NW, 1) k_gather_s3(Params P) {
  if (gated_off(P)) return;
  using Acc = typename std::conditional<F32, AccF32<R, CHECK>, AccF64<R, CHECK>>::type;
  constexpr int kTask = 32 * R;
  constexpr int S = 2 * D;               // window slots per warp
  constexpr int kE = Acc::kE;            // 16-B units per interval entry
  constexpr int kEntry = kE * 16;        // bytes per interval entry
  static_assert(S <= 32, "slots");
  extern __shared__ __align__(16) unsigned char smem_raw[];
  GatherSmem& G = *reinterpret_cast<GatherSmem*>(smem_raw);
  const int tab = P.n_mats * P.max_nucs;
  MatEntry* s_tab = reinterpret_cast<MatEntry*>(smem_raw + sizeof(GatherSmem));
  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  unsigned char* wbase = reinterpret_cast<unsigned char*>(s_tab + tab);
  constexpr size_t win_bytes = static_cast<size_t>(S) * W * kEntry;
  const size_t k_bytes = ((static_cast<size_t>(P.max_nucs) * 8 + 15) / 16) * 16;
  constexpr size_t bar_bytes = ((S * 8 + 15) / 16) * 16;
  const size_t per_warp = win_bytes + k_bytes + bar_bytes;
  unsigned char* mine = wbase + per_warp * warp;
  double2* s_win = reinterpret_cast<double2*>(mine);               // [S][W * 7]
  int2* s_k = reinterpret_cast<int2*>(mine + win_bytes);           // [max_nucs] {k_lo, k_hi}
  uint64_t* s_bar = reinterpret_cast<uint64_t*>(mine + win_bytes + k_bytes);

  for (int i = threadIdx.x; i < tab; i += blockDim.x) {
    const int32_t n = P.mats[i];
    MatEntry me;
    me.conc = P.concs[i];
    me.noff = n >= 0 ? static_cast<uint32_t>(n) * static_cast<uint32_t>(P.N) : 0u;
    me.n = n;
    s_tab[i] = me;
  }
  if (threadIdx.x == 0) {
    uint32_t run = 0, trun = 0;
    for (int m = 0; m < P.n_mats; ++m) {
      const uint32_t c = P.counts[m];
      G.num[m] = P.num_nucs[m];
      G.off[m] = run;
      G.cnt[m] = c;
      G.toff[m] = trun;
      run += c;
      trun += (c + kTask - 1) / kTask;
    }
    G.off[P.n_mats] = run;
    G.toff[P.n_mats] = trun;
  }
  if (lane == 0) {
    for (int d = 0; d < S; ++d) mbar_init(&s_bar[d], 1);
    mbar_fence_init();
  }
  __syncthreads();

  const uint32_t total_tasks = G.toff[P.n_mats];
  const uint32_t gw = blockIdx.x * NW + warp;
  const uint32_t nwarps = gridDim.x * NW;
  const double2* __restrict__ iv2 = reinterpret_cast<const double2*>(F32 ? P.iv32 : P.iv);
  uint32_t phase = 0;  // parity bit per slot

  unsigned long long acc_v = 0, acc_n = 0;
  int m = 0;
  // tasks: the first by warp index, later ones from a global counter (fuel
  // tasks, ~25x the work of the others, come first), fetched one task ahead
  uint32_t next = 0;
  if (DYN && lane == 0) next = nwarps + atomicAdd(P.task_next, 1u);
  for (uint32_t task = gw; task < total_tasks;) {
    while (task >= G.toff[m + 1]) ++m;
    const uint32_t slot0 = (task - G.toff[m]) * kTask + lane * R;
    double p[R];
    int32_t gidx[R];
    uint32_t idx[R];
    bool valid[R];
#pragma unroll
    for (int r = 0; r < R; ++r) {
      valid[r] = slot0 + r < G.cnt[m];
      LookupRec rec{0.5, 0u, 0};
      if (valid[r]) rec = load_rec(P, G.off[m] + slot0 + r);
      p[r] = rec.p;
      gidx[r] = rec.gidx;
      idx[r] = rec.idx;
    }
#pragma unroll
    for (int pass = 0; pass < R; ++pass) {
#pragma unroll
      for (int r = pass & 1; r + 1 < R; r += 2) {
        const bool swap = (valid[r + 1] && !valid[r]) ||
                          (valid[r] == valid[r + 1] && p[r + 1] < p[r]);
        if (swap) {
          const double tp = p[r]; p[r] = p[r + 1]; p[r + 1] = tp;
          const int32_t tg = gidx[r]; gidx[r] = gidx[r + 1]; gidx[r + 1] = tg;
          const uint32_t ti = idx[r]; idx[r] = idx[r + 1]; idx[r + 1] = ti;
          const bool tv = valid[r]; valid[r] = valid[r + 1]; valid[r + 1] = tv;
        }
      }
    }
    double plo = valid[0] ? p[0] : 2.0, phi = -1.0;
    int32_t ulo = valid[0] ? gidx[0] : 0x7fffffff, uhi = -1;
#pragma unroll
    for (int r = 0; r < R; ++r)
      if (valid[r]) {
        phi = p[r];
        uhi = gidx[r];
      }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      const double a = __shfl_xor_sync(0xffffffffu, plo, o);
      const double b = __shfl_xor_sync(0xffffffffu, phi, o);
      plo = a < plo ? a : plo;
      phi = b > phi ? b : phi;
    }
    if (GT == XS_GRID_UNIONIZED && !P.need_gidx) {
      ulo = union_lower_tab(P, plo);
      uhi = union_upper_tab(P, phi);
    } else {
      ulo = __reduce_min_sync(0xffffffffu, ulo);
      uhi = __reduce_max_sync(0xffffffffu, uhi);
    }
#pragma unroll
    for (int r = 0; r < R; ++r)
      if (!valid[r]) p[r] = r > 0 ? p[r - 1] : plo;
    const int nn = G.num[m];
    const MatEntry* row = s_tab + m * P.max_nucs;
    // A4 for the two extremes of every nuclide of the material
    for (int j = lane; j < nn; j += 32) {
      const MatEntry me = row[j];
      int32_t klo, khi;
      if (GT == XS_GRID_UNIONIZED) {
        if (!P.index) {  // column layout only without rows (a row read is 2 x ~1.4 KB per task)
          klo = __ldg(P.index_t + static_cast<int64_t>(me.n) * P.NU + ulo);
          khi = __ldg(P.index_t + static_cast<int64_t>(me.n) * P.NU + uhi);
        } else {
          klo = __ldg(P.index + static_cast<int64_t>(ulo) * P.I + me.n);
          khi = __ldg(P.index + static_cast<int64_t>(uhi) * P.I + me.n);
        }
      } else {
        const RowView<GT> rlo(P, GT == XS_GRID_HASH ? hash_bin(plo, P.du, P.B) : 0);
        const RowView<GT> rhi(P, GT == XS_GRID_HASH ? hash_bin(phi, P.du, P.B) : 0);
        klo = rlo.bracket(P, me.n, me.noff, plo);
        khi = rhi.bracket(P, me.n, me.noff, phi);
      }
      s_k[j] = make_int2(klo, khi);
    }
    __syncwarp();
    // A5 producer: lane 0 stages the entries k_lo .. k_hi of nuclides
    // g*D .. g*D+D-1 into their slots; one mbarrier per group (two groups in
    // flight), its transaction count raised per copy before the copy
    auto issue_group = [&](int g) {
      if (lane == 0 && g * D < nn) {
        uint64_t* bar = &s_bar[g & 1];
#pragma unroll
        for (int d = 0; d < D; ++d) {
          const int j = g * D + d;
          if (j < nn) {
            const int2 kk = s_k[j];
            const uint32_t bytes = static_cast<uint32_t>(kk.y - kk.x + 1) * kEntry;
            if (bytes <= static_cast<uint32_t>(W * kEntry)) {
              const double2* src = iv2 + static_cast<uint64_t>(row[j].noff + static_cast<uint32_t>(kk.x)) * kE;
              mbar_expect_tx(bar, bytes);
              bulk_copy_g2s(s_win + (j % S) * W * kE, src, bytes, bar);
            }
          }
        }
        mbar_arrive(bar);
      }
    };
    issue_group(0);
    issue_group(1);

    Acc acc;
    acc.zero();

    for (int j = 0; j < nn; ++j) {
      const int slot = j % S;
      if (j % D == 0) {
        const int g = j / D;
        if (g >= 1) {
          __syncwarp();  // every lane is done with the slots of group g - 1
          issue_group(g + 1);
        }
        mbar_wait(&s_bar[g & 1], (phase >> (g & 1)) & 1u);
        phase ^= 1u << (g & 1);
      }
      const double conc = row[j].conc;
      const int2 kk = s_k[j];
      const int n_int = kk.y - kk.x;
      if (n_int < W) {
        stage_nuclide_iv<R>(WinPtr{s_win + slot * W * kE}, n_int, conc, p, acc);
      } else {
        const double2* g2 = iv2 + static_cast<uint64_t>(row[j].noff + static_cast<uint32_t>(kk.x)) * kE;
        stage_nuclide_iv<R>(WinGlobal{g2}, n_int, conc, p, acc);
      }
      if ((j & (kF32Block - 1)) == kF32Block - 1) acc.flush();
    }
    if (nn & (kF32Block - 1)) acc.flush();
    __syncwarp();
#pragma unroll
    for (int r = 0; r < R; ++r) {
      if (!valid[r]) continue;
      double mx = -1.0;
      int vi = 0;
#pragma unroll
      for (int c = 0; c < 5; ++c)
        if (acc.get(r, c) > mx) {
          mx = acc.get(r, c);
          vi = c;
        }
      acc_v += static_cast<unsigned long long>(vi + 1);
      acc_n += 1;
      if (P.out_v) P.out_v[idx[r]] = vi + 1;
      if (P.out_M) {
        double* o = P.out_M + static_cast<uint64_t>(idx[r]) * 5;
#pragma unroll
        for (int c = 0; c < 5; ++c) o[c] = acc.get(r, c);
      }
    }
    if (DYN) {
      task = __shfl_sync(0xffffffffu, next, 0);
      if (lane == 0 && task < total_tasks) next = nwarps + atomicAdd(P.task_next, 1u);
    } else {
      task += nwarps;
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    acc_v += __shfl_xor_sync(0xffffffffu, acc_v, o);
    acc_n += __shfl_xor_sync(0xffffffffu, acc_n, o);
  }
  __shared__ unsigned long long s_red[2][NW];
  if (lane == 0) {
    s_red[0][warp] = acc_v;
    s_red[1][warp] = acc_n;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long v = 0, n = 0;
    for (int w = 0; w < NW; ++w) {
      v += s_red[0][w];
      n += s_red[1][w];
    }
    if (n) {
      atomicAdd(P.vsum, v);
      atomicAdd(P.vsum + 1, n);
    }
  }
}

// ------------------------------------------------ k_gather_u (unsorted) --
// Unsorted (material-bucketed) batches: every (lookup, nuclide) reads one
// 96-B entry of the 32-B aligned interval table K0u, {E[k+1], gap, h0, d0 |
// h1, d1, h2, d2 | h3, d3, h4, d4} (h = hi.c, d = hi.c - lo.c), as three
// 32-byte loads (LDG.256) by the lookup's three lanes: three DRAM sectors
// and one load instruction per (lookup, nuclide), where the record-pair
// gather (k_gather) needs two loads per lane over 3-4 sectors.  Lane 0
// computes f (R10: correctly rounded division, reciprocal refined on the
// fly) and its channel, lanes 1-2 two channels each.  Same arithmetic as
// every other path (bit-identical M).
constexpr int kGU = 3;                  // lanes per lookup
constexpr int kLPTU = 32 / kGU;         // lookups per warp task (10)
constexpr int kIvuDoubles = 12;         // K0u entry (96 B)

__device__ __forceinline__ double4 ld_nc_256(const double* p) {
  double4 v;
  asm volatile("ld.global.nc.v4.f64 {%0,%1,%2,%3}, [%4];"
               : "=d"(v.x), "=d"(v.y), "=d"(v.z), "=d"(v.w)
               : "l"(p));
  return v;
}

template <int GT, int U, int MINB, bool CHECK>
__global__ void __launch_bounds__(kGatherThreads, MINB) k_gather_u(Params P) {
  if (gated_off(P)) return;
  static_assert(U % kGU == 0, "U must be a multiple of the group size");
  constexpr int Q = U / kGU;
  extern __shared__ __align__(16) unsigned char smem_raw[];
  GatherSmem& S = *reinterpret_cast<GatherSmem*>(smem_raw);
  const int tab = P.n_mats * P.max_nucs;
  MatEntry* s_tab = reinterpret_cast<MatEntry*>(smem_raw + sizeof(GatherSmem));
  for (int t = threadIdx.x; t < tab; t += blockDim.x) {
    const int32_t n = P.mats[t];
    MatEntry me;
    me.conc = P.concs[t];
    me.noff = n >= 0 ? static_cast<uint32_t>(n) * static_cast<uint32_t>(P.N) : 0u;
    me.n = n;
    s_tab[t] = me;
  }
  if (threadIdx.x == 0) {
    uint32_t run = 0, trun = 0;
    for (int m = 0; m < P.n_mats; ++m) {
      const uint32_t c = P.counts[m];
      S.num[m] = P.num_nucs[m];
      S.off[m] = run;
      S.cnt[m] = c;
      S.toff[m] = trun;
      run += c;
      trun += (c + kLPTU - 1) / kLPTU;
    }
    S.off[P.n_mats] = run;
    S.toff[P.n_mats] = trun;
  }
  __syncthreads();

  const int lane = threadIdx.x & 31;
  const int g = lane / kGU;
  const int r = lane - g * kGU;
  const int base = g * kGU;
  const uint32_t total_tasks = S.toff[P.n_mats];
  const uint32_t warps_per_block = blockDim.x >> 5;
  const uint32_t gw = blockIdx.x * warps_per_block + (threadIdx.x >> 5);
  const uint32_t nw = gridDim.x * warps_per_block;
  const double* __restrict__ ivu = P.ivu + r * 4;   // this lane's third of an entry

  unsigned long long acc_v = 0, acc_n = 0;
  int m = 0;
  for (uint32_t task = gw; task < total_tasks; task += nw) {
    while (task >= S.toff[m + 1]) ++m;
    const uint32_t slot = (task - S.toff[m]) * kLPTU + g;
    const bool valid = (g < kLPTU) && (slot < S.cnt[m]);
    LookupRec rec{0.5, 0u, 0};
    if (valid) rec = load_rec(P, S.off[m] + slot);
    const double p = rec.p;
    const int nn = valid ? S.num[m] : 0;
    const int nw_loop = S.num[m];
    const MatEntry* row = s_tab + m * P.max_nucs;
    const RowView<GT> rv(P, valid ? rec.gidx : 0);

    double acc_a = 0.0, acc_b = 0.0;
    int32_t knext[Q];
#pragma unroll
    for (int q = 0; q < Q; ++q) {
      const int j = r + q * kGU;
      int32_t kq = 0;
      if (j < nn) {
        const MatEntry me = row[j];
        kq = rv.bracket(P, me.n, me.noff, p);
      }
      knext[q] = kq;
    }
    auto round = [&](const int j0, auto tail_tag) {
      constexpr bool TAIL = decltype(tail_tag)::value;
      int32_t kcur[Q];
#pragma unroll
      for (int q = 0; q < Q; ++q) kcur[q] = knext[q];
#pragma unroll
      for (int q = 0; q < Q; ++q) {  // A4 for the next round
        const int j = j0 + U + r + q * kGU;
        int32_t kq = 0;
        if (j < nn) {
          const MatEntry me = row[j];
          kq = rv.bracket(P, me.n, me.noff, p);
        }
        knext[q] = kq;
      }
      double4 v[U];
      double cc[U];
#pragma unroll
      for (int t = 0; t < U; ++t) {
        const int j = j0 + t;
        const int32_t kt = __shfl_sync(0xffffffffu, kcur[t / kGU], base + (t % kGU));
        const MatEntry me = row[TAIL ? (j < nw_loop ? j : 0) : j];
        cc[t] = me.conc;
        uint32_t off = me.noff + static_cast<uint32_t>(kt);
        if (TAIL) off = j < nw_loop ? off : 0u;
        v[t] = ld_nc_256(ivu + static_cast<uint64_t>(off) * kIvuDoubles);
      }
      // A6: f from lane 0's third {E[k+1], gap, ...}; every lane computes
      // it from its own third (branch-free), lane 0's value is broadcast
      double fl[U];
      bool fast = true;
#pragma unroll
      for (int t = 0; t < U; ++t) {
        const double an = dsub(v[t].x, p);
        fl[t] = div_nr(an, v[t].y);
        if (CHECK) fast &= (r != 0) || div_in_range(an, v[t].y);
      }
      if (CHECK && !__all_sync(0xffffffffu, fast)) {
#pragma unroll
        for (int t = 0; t < U; ++t)
          if (r == 0) fl[t] = ddiv(dsub(v[t].x, p), v[t].y);
      }
#pragma unroll
      for (int t = 0; t < U; ++t) {
        const int j = j0 + t;
        const double f = __shfl_sync(0xffffffffu, fl[t], base);
        // lane 0: (E, gap | h0, d0) -> channel 0 in acc_b; lanes 1-2: (h, d) x 2
        const double xa = dsub(v[t].x, dmul(f, v[t].y));
        const double xb = dsub(v[t].z, dmul(f, v[t].w));
        if (!TAIL || j < nw_loop) {  // warp-uniform
          const double c = cc[t];
          acc_a = dadd(acc_a, dmul(xa, c));
          acc_b = dadd(acc_b, dmul(xb, c));
        }
      }
    };
    int j0 = 0;
    for (; j0 + U <= nw_loop; j0 += U) round(j0, std::false_type{});
    if (j0 < nw_loop) round(j0, std::true_type{});
    // A8: channels (t, s, a, f, nf) = (b@r0, a@r1, b@r1, a@r2, b@r2)
    double M[5];
    M[0] = __shfl_sync(0xffffffffu, acc_b, base);
    M[1] = __shfl_sync(0xffffffffu, acc_a, base + 1);
    M[2] = __shfl_sync(0xffffffffu, acc_b, base + 1);
    M[3] = __shfl_sync(0xffffffffu, acc_a, base + 2);
    M[4] = __shfl_sync(0xffffffffu, acc_b, base + 2);
    if (valid && r == 0) {
      double mx = -1.0;
      int vi = 0;
#pragma unroll
      for (int c = 0; c < 5; ++c)
        if (M[c] > mx) {
          mx = M[c];
          vi = c;
        }
      acc_v += static_cast<unsigned long long>(vi + 1);
      acc_n += 1;
      if (P.out_v) P.out_v[rec.idx] = vi + 1;
      if (P.out_M) {
        double* o = P.out_M + static_cast<uint64_t>(rec.idx) * 5;
#pragma unroll
        for (int c = 0; c < 5; ++c) o[c] = M[c];
      }
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    acc_v += __shfl_xor_sync(0xffffffffu, acc_v, o);
    acc_n += __shfl_xor_sync(0xffffffffu, acc_n, o);
  }
  __shared__ unsigned long long s_red[2][kGatherThreads / 32];
  if (lane == 0) {
    s_red[0][threadIdx.x >> 5] = acc_v;
    s_red[1][threadIdx.x >> 5] = acc_n;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long v = 0, n = 0;
    for (uint32_t w = 0; w < warps_per_block; ++w) {
      v += s_red[0][w];
      n += s_red[1][w];
    }
    if (n) {
      atomicAdd(P.vsum, v);
      atomicAdd(P.vsum + 1, n);
    }
  }
}

// ------------------------------------------- k_gather_s4 (staged, LDGSTS) --
// The staged gather of k_gather_s3 with a cheaper producer: the windows of a
// group of D nuclides are packed back to back into one of two per-warp
// buffers of C interval entries, copied by all 32 lanes at once with 16-B
// cp.async (32/D lanes per nuclide, no per-copy elected issue), completing
// on the buffer's mbarrier (one cp.async arrive per lane).  Each nuclide's
// place in its group buffer is a segmented warp scan of the window sizes,
// done in the A4 prologue.  A window that does not fit its group's buffer is
// read in place from global memory (rare: C is ~1.5x a group's mean size).
// The material table is staged packed (CSR) instead of [n_mats][max_nucs].
// Arithmetic, operation order and results are those of k_gather_s3 (R10/R11,
// R18 for F32).
struct alignas(16) NucWin {
  int32_t klo, khi;   // bracket range of the task's extreme energies (A4)
  uint32_t noff;      // n * N
  uint32_t off;       // shared-memory byte address of the window in its group
                      // buffer, kNoBuf = read in place from global memory
};
constexpr uint32_t kNoBuf = 0xffffffffu;
#ifndef XS_S4_PREFETCH
#define XS_S4_PREFETCH 1
#endif
constexpr bool kS4Prefetch = XS_S4_PREFETCH;

// Indexed by rank: the materials in decreasing nuclide count (stable), so
// that tasks are numbered longest first (fuel, then 27, 21, ... nuclides)
// and the dynamic task order ends with the shortest tasks.
struct alignas(16) GatherSmem4 {
  int32_t num[kMaxMats];
  uint32_t off[kMaxMats + 1];   // bucket start of the material of rank r
  uint32_t cnt[kMaxMats];
  uint32_t toff[kMaxMats + 1];  // first task of rank r
  uint32_t roff[kMaxMats + 1];  // first table entry of rank r (CSR, rank order)
  int32_t mat[kMaxMats];        // material of rank r
};

// the next task's energies are prefetched (1 KB per warp) by the 4-lookups-
// per-lane shapes with 16 warps (the default for dense batches), whose shared
// memory leaves room for it
template <int R, int NW>
__host__ __device__ constexpr bool s4_prefetch() {
  return kS4Prefetch && R == 4 && NW <= 16;
}
template <int C, bool F32, bool PF = false>
__host__ __device__ constexpr size_t s4_warp_bytes(int max_nucs) {
  return 2 * static_cast<size_t>(C) * (F32 ? kIv32Doubles : kIvDoubles) * 8 +  // buffers
         static_cast<size_t>(max_nucs) * sizeof(NucWin) + 16 +                  // windows + bars
         (PF ? 32 * 4 * 8 : 0);                                                  // next energies
}

// OUT = false: no per-lookup outputs (verification sum only), so the batch
// positions are neither loaded nor kept in registers across the nuclide loop
template <int GT, int R, int D, int C, int NW, bool CHECK, bool F32, bool DYN, bool OUT = true>
__global__ void __launch_bounds__(32 * NW, 1) k_gather_s4(Params P) {
  if (gated_off(P)) return;
  using Acc = typename std::conditional<F32, AccF32<R, CHECK>, AccF64<R, CHECK>>::type;
  constexpr int kTask = 32 * R;
  constexpr int kE = Acc::kE;            // 16-B units per interval entry
  constexpr int LPN = 32 / D;            // copying lanes per nuclide
  static_assert(D >= 1 && D <= 32 && (32 % D) == 0, "group size divides the warp");
  static_assert(C <= 255, "buffer offsets");
  extern __shared__ __align__(16) unsigned char smem_raw[];
  GatherSmem4& G = *reinterpret_cast<GatherSmem4*>(smem_raw);
  MatEntry* s_tab = reinterpret_cast<MatEntry*>(smem_raw + sizeof(GatherSmem4));
  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;

  if (threadIdx.x == 0) {
    uint32_t run = 0;
    for (int m = 0; m < P.n_mats; ++m) {  // bucket starts in material order
      G.off[m] = run;
      run += P.counts[m];
    }
    for (int m = 0; m < P.n_mats; ++m) {  // rank order: insertion by nuclide count
      int r = m;
      while (r > 0 && P.num_nucs[G.mat[r - 1]] < P.num_nucs[m]) {
        G.mat[r] = G.mat[r - 1];
        --r;
      }
      G.mat[r] = m;
    }
    uint32_t start[kMaxMats];
    for (int m = 0; m < P.n_mats; ++m) start[m] = G.off[m];
    uint32_t trun = 0, roff = 0;
    for (int r = 0; r < P.n_mats; ++r) {
      const int m = G.mat[r];
      const uint32_t c = P.counts[m];
      G.num[r] = P.num_nucs[m];
      G.off[r] = start[m];
      G.cnt[r] = c;
      G.toff[r] = trun;
      G.roff[r] = roff;
      trun += (c + kTask - 1) / kTask;
      roff += static_cast<uint32_t>(P.num_nucs[m]);
    }
    G.off[P.n_mats] = run;
    G.toff[P.n_mats] = trun;
    G.roff[P.n_mats] = roff;
  }
  __syncthreads();
  const int tab = static_cast<int>(G.roff[P.n_mats]);
  for (int i = threadIdx.x; i < tab; i += blockDim.x) {
    int r = 0;
    while (static_cast<uint32_t>(i) >= G.roff[r + 1]) ++r;
    const int src = G.mat[r] * P.max_nucs + (i - static_cast<int>(G.roff[r]));
    const int32_t n = P.mats[src];
    MatEntry me;
    me.conc = P.concs[src];
    me.noff = static_cast<uint32_t>(n) * static_cast<uint32_t>(P.N);
    me.n = n;
    s_tab[i] = me;
  }
  unsigned char* wbase = reinterpret_cast<unsigned char*>(s_tab) + ((tab * sizeof(MatEntry) + 15) / 16) * 16;
  constexpr bool PF = s4_prefetch<R, NW>();
  unsigned char* mine = wbase + s4_warp_bytes<C, F32, PF>(P.max_nucs) * warp;
  double2* s_buf = reinterpret_cast<double2*>(mine);                            // [2][C * kE]
  NucWin* s_k = reinterpret_cast<NucWin*>(mine + 2 * static_cast<size_t>(C) * kE * 16);
  uint64_t* s_bar = reinterpret_cast<uint64_t*>(s_k + P.max_nucs);              // [2]
  // the next task's energies, copied by cp.async during this task (R <= 4)
  const uint32_t pf_base = smem_u32(s_bar + 2) + static_cast<uint32_t>(lane) * 32u;
  const uint32_t buf_base = smem_u32(s_buf);
  const uint32_t sk_base = smem_u32(s_k);
  if (lane == 0) {
    mbar_init(&s_bar[0], 32);
    mbar_init(&s_bar[1], 32);
    mbar_fence_init();
  }
  __syncthreads();

  const uint32_t total_tasks = G.toff[P.n_mats];
  const uint32_t gw = blockIdx.x * NW + warp;
  const uint32_t nwarps = gridDim.x * NW;
  const double2* __restrict__ iv2 = reinterpret_cast<const double2*>(F32 ? P.iv32 : P.iv);
  uint32_t phase = 0;  // parity bit per buffer

  unsigned long long acc_v = 0, acc_n = 0;
  int m = 0;
  // DYN: after its first task a warp takes the next one from a global counter
  // (tasks in material order, fuel first), fetched one task ahead
  uint32_t next = 0;
  if (DYN && lane == 0) next = nwarps + atomicAdd(P.task_next, 1u);
  const bool pre = PF && !OUT && P.sp && !P.sidx;
  bool have_pf = false;  // this lane's energies of the task were prefetched
  for (uint32_t task = gw; task < total_tasks;) {
    while (task >= G.toff[m + 1]) ++m;
    const uint32_t slot0 = (task - G.toff[m]) * kTask + lane * R;
    double p[R];
    int32_t gidx[R];
    uint32_t idx[R];
    bool valid[R];
    if (have_pf) asm volatile("cp.async.wait_all;" ::: "memory");
#pragma unroll
    for (int r = 0; r < R; ++r) {
      valid[r] = slot0 + r < G.cnt[m];
      LookupRec rec{0.5, 0u, 0};
      if (have_pf) {
        asm volatile("ld.shared.f64 %0, [%1];" : "=d"(rec.p) : "r"(pf_base + 8u * r));
      } else if (valid[r]) {
        rec = load_rec(P, G.off[m] + slot0 + r);
      }
      p[r] = rec.p;
      gidx[r] = rec.gidx;
      idx[r] = OUT ? rec.idx : 0u;
    }
    if (pre) {  // the next task's energies (whole lane groups only)
      const uint32_t nt = DYN ? __shfl_sync(0xffffffffu, next, 0) : task + nwarps;
      have_pf = false;
      if (nt < total_tasks) {
        int mn = m;
        while (nt >= G.toff[mn + 1]) ++mn;
        const uint32_t s0n = (nt - G.toff[mn]) * kTask + lane * R;
        if (s0n + R <= G.cnt[mn]) {
          const double* src = P.sp + G.off[mn] + s0n;
#pragma unroll
          for (int r = 0; r < R; ++r)
            asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(pf_base + 8u * r),
                         "l"(src + r)
                         : "memory");
          have_pf = true;
        }
      }
    }
#pragma unroll
    for (int pass = 0; pass < R; ++pass) {
#pragma unroll
      for (int r = pass & 1; r + 1 < R; r += 2) {
        const bool swap = (valid[r + 1] && !valid[r]) ||
                          (valid[r] == valid[r + 1] && p[r + 1] < p[r]);
        if (swap) {
          const double tp = p[r]; p[r] = p[r + 1]; p[r + 1] = tp;
          const int32_t tg = gidx[r]; gidx[r] = gidx[r + 1]; gidx[r + 1] = tg;
          const uint32_t ti = idx[r]; idx[r] = idx[r + 1]; idx[r + 1] = ti;
          const bool tv = valid[r]; valid[r] = valid[r + 1]; valid[r + 1] = tv;
        }
      }
    }
    double plo = valid[0] ? p[0] : 2.0, phi = -1.0;
    int32_t ulo = valid[0] ? gidx[0] : 0x7fffffff, uhi = -1;
#pragma unroll
    for (int r = 0; r < R; ++r)
      if (valid[r]) {
        phi = p[r];
        uhi = gidx[r];
      }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      const double a = __shfl_xor_sync(0xffffffffu, plo, o);
      const double b = __shfl_xor_sync(0xffffffffu, phi, o);
      plo = a < plo ? a : plo;
      phi = b > phi ? b : phi;
    }
    if (GT == XS_GRID_UNIONIZED && !P.need_gidx) {
      ulo = union_lower_tab(P, plo);
      uhi = union_upper_tab(P, phi);
    } else {
      ulo = __reduce_min_sync(0xffffffffu, ulo);
      uhi = __reduce_max_sync(0xffffffffu, uhi);
    }
#pragma unroll
    for (int r = 0; r < R; ++r)
      if (!valid[r]) p[r] = r > 0 ? p[r - 1] : plo;
    const int nn = G.num[m];
    const MatEntry* row = s_tab + G.roff[m];
    const uint32_t row_base = smem_u32(row);
    // A4 for the two extremes of every nuclide, and each window's place in
    // its group buffer (segmented scan of the sizes over groups of D lanes;
    // 32 nuclides per round, so groups never straddle rounds)
    for (int j0 = 0; j0 < nn; j0 += 32) {
      const int j = j0 + lane;
      int32_t klo = 0, khi = 0;
      uint32_t noff = 0;
      if (j < nn) {
        const MatEntry me = row[j];
        noff = me.noff;
        if (GT == XS_GRID_UNIONIZED) {
          if (!P.index) {  // column layout only without rows (a row read is 2 x ~1.4 KB per task)
            klo = __ldg(P.index_t + static_cast<int64_t>(me.n) * P.NU + ulo);
            khi = __ldg(P.index_t + static_cast<int64_t>(me.n) * P.NU + uhi);
          } else {
            klo = __ldg(P.index + static_cast<int64_t>(ulo) * P.I + me.n);
            khi = __ldg(P.index + static_cast<int64_t>(uhi) * P.I + me.n);
          }
        } else {
          const RowView<GT> rlo(P, GT == XS_GRID_HASH ? hash_bin(plo, P.du, P.B) : 0);
          const RowView<GT> rhi(P, GT == XS_GRID_HASH ? hash_bin(phi, P.du, P.B) : 0);
          klo = rlo.bracket(P, me.n, me.noff, plo);
          khi = rhi.bracket(P, me.n, me.noff, phi);
        }
      }
      const int32_t n_int = khi - klo;
      const int size = (j < nn && n_int < C) ? n_int + 1 : 0;
      int incl = size;
#pragma unroll
      for (int o = 1; o < D; o <<= 1) {
        const int v = __shfl_up_sync(0xffffffffu, incl, o);
        if ((lane & (D - 1)) >= o) incl += v;
      }
      if (j < nn) {
        NucWin w;
        w.klo = klo;
        w.khi = khi;
        w.noff = noff;
        w.off = (size > 0 && incl <= C)
                    ? buf_base + static_cast<uint32_t>(((j / D) & 1) * C + (incl - size)) * (kE * 16)
                    : kNoBuf;
        s_k[j] = w;
      }
    }
    __syncwarp();
    // A5 producer: all lanes copy group g's windows (LPN lanes per nuclide,
    // 16 B per cp.async) into buffer g & 1, then arrive on its mbarrier
    auto issue_group = [&](int g) {
      if (g * D >= nn) return;  // warp-uniform
      const int j = g * D + lane / LPN;
      if (j < nn) {
        const NucWin w = s_k[j];
        if (w.off != kNoBuf) {
          const double2* src = iv2 + static_cast<uint64_t>(w.noff + static_cast<uint32_t>(w.klo)) * kE;
          const int nch = (w.khi - w.klo + 1) * kE;
          for (int c = lane % LPN; c < nch; c += LPN) cp_async16_s(w.off + 16u * c, src + c);
        }
      }
      cp_async_mbar_arrive(&s_bar[g & 1]);
    };
    issue_group(0);
    issue_group(1);

    Acc acc;
    acc.zero();
    for (int g = 0; g * D < nn; ++g) {  // groups of D nuclides
      if (g >= 1) {
        __syncwarp();  // every lane is done with buffer (g + 1) & 1 (group g - 1)
        issue_group(g + 1);
      }
      mbar_wait(&s_bar[g & 1], (phase >> (g & 1)) & 1u);
      phase ^= 1u << (g & 1);
      const int jend = (g + 1) * D < nn ? (g + 1) * D : nn;
    for (int j = g * D; j < jend; ++j) {
      // the step's window record and concentration through 32-bit shared
      // addresses (no generic-to-shared conversion per step)
      NucWin w;
      asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];"
                   : "=r"(w.klo), "=r"(w.khi), "=r"(w.noff), "=r"(w.off)
                   : "r"(sk_base + 16u * j));
      double conc;
      asm volatile("ld.shared.f64 %0, [%1];" : "=d"(conc) : "r"(row_base + 16u * j));
      const int n_int = w.khi - w.klo;
      if (w.off != kNoBuf) {
        stage_nuclide_iv<R>(WinSmem{w.off}, n_int, conc, p, acc);
      } else {
        const double2* g2 = iv2 + static_cast<uint64_t>(w.noff + static_cast<uint32_t>(w.klo)) * kE;
        stage_nuclide_iv<R>(WinGlobal{g2}, n_int, conc, p, acc);
      }
      if ((j & (kF32Block - 1)) == kF32Block - 1) acc.flush();
    }
    }
    if (nn & (kF32Block - 1)) acc.flush();
    __syncwarp();
#pragma unroll
    for (int r = 0; r < R; ++r) {
      if (!valid[r]) continue;
      double mx = -1.0;
      int vi = 0;
#pragma unroll
      for (int c = 0; c < 5; ++c)
        if (acc.get(r, c) > mx) {
          mx = acc.get(r, c);
          vi = c;
        }
      acc_v += static_cast<unsigned long long>(vi + 1);
      acc_n += 1;
      if (OUT && P.out_v) P.out_v[idx[r]] = vi + 1;
      if (OUT && P.out_M) {
        double* o = P.out_M + static_cast<uint64_t>(idx[r]) * 5;
#pragma unroll
        for (int c = 0; c < 5; ++c) o[c] = acc.get(r, c);
      }
    }
    if (DYN) {
      task = __shfl_sync(0xffffffffu, next, 0);
      if (lane == 0 && task < total_tasks) next = nwarps + atomicAdd(P.task_next, 1u);
    } else {
      task += nwarps;
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    acc_v += __shfl_xor_sync(0xffffffffu, acc_v, o);
    acc_n += __shfl_xor_sync(0xffffffffu, acc_n, o);
  }
  __shared__ unsigned long long s_red[2][NW];
  if (lane == 0) {
    s_red[0][warp] = acc_v;
    s_red[1][warp] = acc_n;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long v = 0, n = 0;
    for (int w = 0; w < NW; ++w) {
      v += s_red[0][w];
      n += s_red[1][w];
    }
    if (n) {
      atomicAdd(P.vsum, v);
      atomicAdd(P.vsum + 1, n);
    }
  }
}

// --------------------------------------------------- XSBench-shape baseline
// One thread per lookup, no bucketing, serial nuclide loop (the shape of the
// CUDA kernels the paper measured).  Same exact
// arithmetic.  For comparison only (XS_FLAG_BASELINE).
template <int GT>
__global__ void __launch_bounds__(256) k_baseline(Params P) {
  unsigned long long acc_v = 0, acc_n = 0;
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < P.count;
       i += gridDim.x * blockDim.x) {
    const Sample s = get_lookup(P, i);
    if (s.mat >= P.n_mats) {
      write_invalid(P, i);
      if (P.out_mat)
        P.out_mat[i] = P.in_mat8 ? static_cast<int32_t>(P.in_mat8[i]) : (P.in_mat ? P.in_mat[i] : -1);
      if (P.out_gidx) P.out_gidx[i] = -1;
      if (P.out_E) P.out_E[i] = s.p;
      continue;
    }
    const int32_t gidx = grid_index_of<GT>(P, s.p);
    double M[5] = {0.0, 0.0, 0.0, 0.0, 0.0};
    const int nn = P.num_nucs[s.mat];
    for (int j = 0; j < nn; ++j) {
      const int32_t n = __ldg(P.mats + s.mat * P.max_nucs + j);
      const double c = __ldg(P.concs + s.mat * P.max_nucs + j);
      const int32_t k = bracket_of<GT>(P, gidx, n, s.p);
      const double2* pr =
          reinterpret_cast<const double2*>(P.grid) + (static_cast<int64_t>(n) * P.N + k) * 3;
      const double2 l0 = __ldg(pr), l1 = __ldg(pr + 1), l2 = __ldg(pr + 2);
      const double2 h0 = __ldg(pr + 3), h1 = __ldg(pr + 4), h2 = __ldg(pr + 5);
      const double f = ddiv(dsub(h0.x, s.p), dsub(h0.x, l0.x));
      const double lo[5] = {l0.y, l1.x, l1.y, l2.x, l2.y};
      const double hi[5] = {h0.y, h1.x, h1.y, h2.x, h2.y};
#pragma unroll
      for (int ch = 0; ch < 5; ++ch) {
        const double x = dsub(hi[ch], dmul(f, dsub(hi[ch], lo[ch])));
        M[ch] = dadd(M[ch], dmul(x, c));
      }
    }
    double mx = -1.0;
    int vi = 0;
#pragma unroll
    for (int ch = 0; ch < 5; ++ch)
      if (M[ch] > mx) {
        mx = M[ch];
        vi = ch;
      }
    acc_v += static_cast<unsigned long long>(vi + 1);
    acc_n += 1;
    if (P.out_v) P.out_v[i] = vi + 1;
    if (P.out_M)
      for (int ch = 0; ch < 5; ++ch) P.out_M[static_cast<uint64_t>(i) * 5 + ch] = M[ch];
    if (P.out_E) P.out_E[i] = s.p;
    if (P.out_mat) P.out_mat[i] = s.mat;
    if (P.out_gidx) P.out_gidx[i] = GT == XS_GRID_NUCLIDE ? -1 : gidx;
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    acc_v += __shfl_xor_sync(0xffffffffu, acc_v, o);
    acc_n += __shfl_xor_sync(0xffffffffu, acc_n, o);
  }
  if ((threadIdx.x & 31) == 0 && acc_n) {
    atomicAdd(P.vsum, acc_v);
    atomicAdd(P.vsum + 1, acc_n);
  }
}

// ------------------------------------------------------------ A8 alone ----
__global__ void k_verify(const double* __restrict__ M, uint64_t count,
                         unsigned long long* __restrict__ vsum) {
  unsigned long long acc_v = 0, acc_n = 0;
  for (uint64_t i = blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x; i < count;
       i += static_cast<uint64_t>(gridDim.x) * blockDim.x) {
    double mx = -1.0;
    int vi = 0;
    for (int c = 0; c < 5; ++c) {
      const double x = M[i * 5 + c];
      if (x > mx) {
        mx = x;
        vi = c;
      }
    }
    acc_v += static_cast<unsigned long long>(vi + 1);
    acc_n += 1;
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    acc_v += __shfl_xor_sync(0xffffffffu, acc_v, o);
    acc_n += __shfl_xor_sync(0xffffffffu, acc_n, o);
  }
  if ((threadIdx.x & 31) == 0 && acc_n) {
    atomicAdd(vsum, acc_v);
    atomicAdd(vsum + 1, acc_n);
  }
}

template <int GT>
__global__ void k_nuclide_index(Params P, const double* __restrict__ energy,
                                const int32_t* __restrict__ nuc, uint64_t count,
                                int32_t* __restrict__ k_out) {
  for (uint64_t i = blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x; i < count;
       i += static_cast<uint64_t>(gridDim.x) * blockDim.x) {
    const double p = energy[i];
    const int32_t n = nuc[i];
    const int32_t gidx = grid_index_of<GT>(P, p);
    k_out[i] = bracket_of<GT>(P, gidx, n, p);
  }
}

// ----------------------------------------------------------------- host ----
static Params make_params(const DeviceGrid& g) {
  Params P{};
  P.grid = g.grid;
  P.iv = g.iv;
  P.iv32 = g.iv32;
  P.ivu = g.ivu;
  P.I = g.I;
  P.N = g.N;
  P.U = g.U;
  P.NU = g.NU;
  P.UB = g.UB;
  P.UBn = g.UBn;
  P.index = g.index;
  P.index_t = g.index_t;
  P.B = g.B;
  P.du = g.du;
  P.num_nucs = g.num_nucs;
  P.mats = g.mats;
  P.concs = g.concs;
  P.n_mats = g.n_mats;
  P.max_nucs = g.max_nucs;
  P.seed = g.lookup_seed;
  return P;
}

static unsigned grid_cap(uint64_t work, int threads, int sm, int per_sm) {
  uint64_t b = (work + threads - 1) / threads;
  uint64_t cap = static_cast<uint64_t>(sm) * per_sm;
  if (b == 0) b = 1;
  return static_cast<unsigned>(b < cap ? b : cap);
}

template <int GT, int U, int MINB, bool CHECK>
static cudaError_t launch_gather(const DeviceGrid& g, const Params& P, cudaStream_t st) {
  const size_t smem = sizeof(GatherSmem) + static_cast<size_t>(g.n_mats) * g.max_nucs * sizeof(MatEntry);
  auto kern = k_gather<GT, U, MINB, CHECK>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       static_cast<int>(smem));
  if (e != cudaSuccess) return e;
  int per_sm = g.blocks_per_sm;
  if (per_sm <= 0) {
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, kGatherThreads, smem);
    if (e != cudaSuccess) return e;
    if (per_sm < 1) per_sm = 1;
  }
  kern<<<g.sm_count * per_sm, kGatherThreads, smem, st>>>(P);
  return cudaGetLastError();
}

// gather variants: (nuclides per round U, min resident blocks of 256 threads)
// CHECK: the division fast path is exact without a range check when every
// energy (grid and lookups) is a multiple of 2^-63 in [0, 1] (DESIGN.md §4:
// then |hi.E - p| and |hi.E - lo.E| are 0 or >= 2^-63), which holds for
// generated grids with sampled lookups; otherwise the checked kernel runs.
template <int GT, int U, int MINB, bool CHECK>
static cudaError_t launch_gather_un(const DeviceGrid& g, const Params& P, cudaStream_t st) {
  const size_t smem = sizeof(GatherSmem) + static_cast<size_t>(g.n_mats) * g.max_nucs * sizeof(MatEntry);
  auto kern = k_gather_u<GT, U, MINB, CHECK>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       static_cast<int>(smem));
  if (e != cudaSuccess) return e;
  int per_sm = g.blocks_per_sm;
  if (per_sm <= 0) {
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, kGatherThreads, smem);
    if (e != cudaSuccess) return e;
    if (per_sm < 1) per_sm = 1;
  }
  kern<<<g.sm_count * per_sm, kGatherThreads, smem, st>>>(P);
  return cudaGetLastError();
}

template <int GT, bool CHECK>
static cudaError_t launch_gather_v(const DeviceGrid& g, const Params& P, cudaStream_t st) {
  if (g.ivu && (g.unroll == 0 || (g.unroll >= 51 && g.unroll <= 54))) {
    switch (g.unroll) {  // k_gather_u (nuclides per round U, min blocks of 256)
      case 51: return launch_gather_un<GT, 3, 3, CHECK>(g, P, st);
      case 53: return launch_gather_un<GT, 3, 4, CHECK>(g, P, st);
      case 54: return launch_gather_un<GT, 6, 3, CHECK>(g, P, st);
      default: return launch_gather_un<GT, 6, 2, CHECK>(g, P, st);  // 52 (measured best, large)
    }
  }
  switch (g.unroll) {
    case 1: return launch_gather<GT, 3, 3, CHECK>(g, P, st);
    case 2: return launch_gather<GT, 3, 4, CHECK>(g, P, st);
    case 4: return launch_gather<GT, 6, 3, CHECK>(g, P, st);
    default: return launch_gather<GT, 6, 2, CHECK>(g, P, st);
  }
}

template <int GT, int R, int U, int MINB, bool CHECK>
static cudaError_t launch_gather_t(const DeviceGrid& g, const Params& P, cudaStream_t st) {
  const size_t smem = sizeof(GatherSmem) + static_cast<size_t>(g.n_mats) * g.max_nucs * sizeof(MatEntry);
  auto kern = k_gather_t<GT, R, U, MINB, CHECK>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       static_cast<int>(smem));
  if (e != cudaSuccess) return e;
  int per_sm = g.blocks_per_sm;
  if (per_sm <= 0) {
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, kGatherThreads, smem);
    if (e != cudaSuccess) return e;
    if (per_sm < 1) per_sm = 1;
  }
  kern<<<g.sm_count * per_sm, kGatherThreads, smem, st>>>(P);
  return cudaGetLastError();
}

template <int GT, int R, int D, int W, int NW, bool CHECK>
static cudaError_t launch_gather_s(const DeviceGrid& g, const Params& P, cudaStream_t st) {
  const size_t win_bytes = static_cast<size_t>(D) * W * 48;
  const size_t kw_bytes = ((static_cast<size_t>(g.max_nucs) * 2 * 4 + 15) / 16) * 16;
  const size_t smem = sizeof(GatherSmem) +
                      static_cast<size_t>(g.n_mats) * g.max_nucs * sizeof(MatEntry) +
                      NW * (win_bytes + kw_bytes + ((D * 8 + 15) / 16) * 16);
  auto kern = k_gather_s<GT, R, D, W, NW, CHECK>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       static_cast<int>(smem));
  if (e != cudaSuccess) return e;
  int per_sm = g.blocks_per_sm;
  if (per_sm <= 0) {
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, 32 * NW, smem);
    if (e != cudaSuccess) return e;
    if (per_sm < 1) per_sm = 1;
  }
  kern<<<g.sm_count * per_sm, 32 * NW, smem, st>>>(P);
  return cudaGetLastError();
}

template <int GT, int R, int D, int W, int NW, bool CHECK, bool DYN = false, bool F32 = false>
static cudaError_t launch_gather_s3(const DeviceGrid& g, const Params& P, cudaStream_t st) {
  constexpr size_t win_bytes = static_cast<size_t>(2 * D) * W * (F32 ? kIv32Doubles : kIvDoubles) * 8;
  const size_t k_bytes = ((static_cast<size_t>(g.max_nucs) * 8 + 15) / 16) * 16;
  const size_t smem = sizeof(GatherSmem) +
                      static_cast<size_t>(g.n_mats) * g.max_nucs * sizeof(MatEntry) +
                      NW * (win_bytes + k_bytes + ((2 * D * 8 + 15) / 16) * 16);
  auto kern = k_gather_s3<GT, R, D, W, NW, CHECK, DYN, F32>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       static_cast<int>(smem));
  if (e != cudaSuccess) return e;
  int per_sm = g.blocks_per_sm;
  if (per_sm <= 0) {
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, 32 * NW, smem);
    if (e != cudaSuccess) return e;
    if (per_sm < 1) per_sm = 1;
  }
  kern<<<g.sm_count * per_sm, 32 * NW, smem, st>>>(P);
  return cudaGetLastError();
}

// SPEC: the default shapes (variants 55-57) also come without per-lookup
// outputs (OUT = false: four registers fewer in the nuclide loop, -0.5 to -1%
// of the gather), chosen per call
template <int GT, int R, int D, int C, int NW, bool CHECK, bool F32 = false, bool DYN = false,
          bool SPEC = false>
static cudaError_t launch_gather_s4(const DeviceGrid& g, const Params& P, cudaStream_t st) {
  // the kernel stages the packed material table: sum(num_nucs) entries
  const size_t smem = sizeof(GatherSmem4) +
                      ((static_cast<size_t>(g.tab_total) * sizeof(MatEntry) + 15) / 16) * 16 +
                      NW * s4_warp_bytes<C, F32, s4_prefetch<R, NW>()>(g.max_nucs);
  auto kern = k_gather_s4<GT, R, D, C, NW, CHECK, F32, DYN, true>;
  if constexpr (SPEC) {
    if (!P.out_v && !P.out_M) kern = k_gather_s4<GT, R, D, C, NW, CHECK, F32, DYN, false>;
  }
  if (smem > 227 * 1024) return cudaErrorInvalidConfiguration;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       static_cast<int>(smem));
  if (e != cudaSuccess) return e;
  int per_sm = g.blocks_per_sm;
  if (per_sm <= 0) {
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, 32 * NW, smem);
    if (e != cudaSuccess) return e;
    if (per_sm < 1) per_sm = 1;
  }
  kern<<<g.sm_count * per_sm, 32 * NW, smem, st>>>(P);
  return cudaGetLastError();
}

template <int GT, bool CHECK>
static cudaError_t launch_gather_tv(const DeviceGrid& g, const Params& P, cudaStream_t st) {
  // variants 1-4: k_gather_t (lookups per lane R, nuclides per round U, min
  // blocks); 9-12 TMA-staged record windows (R, stages D, window W records,
  // warps per block); 17-20 TMA-staged interval-table windows (R, group
  // size D, window W entries, warps per block); 40-58 k_gather_s4 (R, group
  // size D, group buffer C entries, warps per block; 55/56 take tasks from a
  // global counter after their first).  Density d = N * 128 / count (interval
  // entries a 128-lookup task of one material spans per nuclide; for an
  // energy-range shard count is the whole batch's, whose density the shard
  // keeps).  Measured on B200: d < 0.12 (large and small at
  // 17M) variant 59 = variant 55 with 32-entry group buffers (fewer windows
  // read in place: large gather 1.968 vs 1.980 ms, small 0.723 vs 0.734; 55
  // when the shared memory does not fit, and for the hash grid, whose
  // prologue searches read the nuclide grid through L1: large-hash step 2.68
  // vs 2.58 ms with 59); variant 55 = (4, 8, 20, 16,
  // dynamic): large 2.21 ms vs 2.24 static (40) and 2.47 for k_gather_s3
  // (25); 0.12 <= d < 0.25 variant 56 = (2, 8, 16,
  // 24, dynamic): large 8M 1.41 vs 1.42 / 1.48 / 1.61 ms for 44 / 40 / 20;
  // d >= 0.25, N < 100k: k_gather_s3 (2, 2, 8, 24) = variant 20 (large 4M 1.02
  // vs 1.07 ms for 44, small 4M 0.29 vs 0.31); d >= 0.15 on grids of >= 100k
  // points per nuclide (XL 170M, cold 9.5 GB interval table): variant 57 =
  // (2, 4, 16, 24, dynamic): 32.2 vs 33.5 ms for 20 (static); the dynamic
  // task order: gather 30.7 vs 31.5 ms, 8-shard rank 4.74 vs 4.89 ms.
  int v = g.unroll;
  if (v == 0) {
    const double d = static_cast<double>(g.N) * 128.0 / static_cast<double>(P.count ? P.count : 1);
    if (d >= 0.15 && g.N >= 100000)
      v = 57;
    else
      v = d >= 0.25 ? 20 : (d >= 0.12 ? 56 : (GT == XS_GRID_HASH ? 55 : 59));
  }
  switch (v) {
    case 1: return launch_gather_t<GT, 8, 1, 2, CHECK>(g, P, st);
    case 2: return launch_gather_t<GT, 4, 1, 2, CHECK>(g, P, st);
    case 3: return launch_gather_t<GT, 2, 1, 3, CHECK>(g, P, st);
    case 4: return launch_gather_t<GT, 4, 2, 2, CHECK>(g, P, st);
    case 9: return launch_gather_s<GT, 4, 4, 16, 16, CHECK>(g, P, st);
    case 10: return launch_gather_s<GT, 4, 3, 16, 16, CHECK>(g, P, st);
    case 11: return launch_gather_s<GT, 4, 6, 12, 16, CHECK>(g, P, st);
    case 12: return launch_gather_s<GT, 4, 4, 12, 8, CHECK>(g, P, st);
    case 17: return launch_gather_s3<GT, 4, 4, 8, 12, CHECK>(g, P, st);
    case 18: return launch_gather_s3<GT, 4, 4, 8, 16, CHECK>(g, P, st);
    case 19: return launch_gather_s3<GT, 4, 2, 8, 16, CHECK>(g, P, st);
    case 20: return launch_gather_s3<GT, 2, 2, 8, 24, CHECK>(g, P, st);
    case 21: return launch_gather_s3<GT, 4, 2, 8, 16, CHECK, true>(g, P, st);
    case 22: return launch_gather_s3<GT, 4, 1, 8, 16, CHECK, true>(g, P, st);
    case 23: return launch_gather_s3<GT, 4, 2, 6, 16, CHECK, true>(g, P, st);
    case 24: return launch_gather_s3<GT, 4, 2, 8, 20, CHECK>(g, P, st);
    case 25: return launch_gather_s3<GT, 4, 4, 6, 16, CHECK>(g, P, st);
    case 26: return launch_gather_s3<GT, 4, 4, 6, 20, CHECK>(g, P, st);
    case 27: return launch_gather_s3<GT, 4, 2, 6, 24, CHECK>(g, P, st);
    case 28: return launch_gather_s3<GT, 4, 4, 4, 16, CHECK>(g, P, st);
    // k_gather_s4 (R, D, C, NW): LDGSTS-staged group buffers
    case 40: return launch_gather_s4<GT, 4, 8, 20, 16, CHECK>(g, P, st);
    case 41: return launch_gather_s4<GT, 4, 8, 20, 20, CHECK>(g, P, st);
    case 42: return launch_gather_s4<GT, 4, 4, 12, 16, CHECK>(g, P, st);
    case 43: return launch_gather_s4<GT, 4, 4, 12, 20, CHECK>(g, P, st);
    case 44: return launch_gather_s4<GT, 2, 8, 16, 24, CHECK>(g, P, st);
    case 45: return launch_gather_s4<GT, 4, 8, 16, 24, CHECK>(g, P, st);
    case 49: return launch_gather_s4<GT, 3, 4, 8, 24, CHECK>(g, P, st);

    case 50: return launch_gather_s4<GT, 3, 8, 16, 20, CHECK>(g, P, st);
    case 55: return launch_gather_s4<GT, 4, 8, 20, 16, CHECK, false, true, true>(g, P, st);
    case 59: {  // variant 55 with 32-entry group buffers, when the shared memory allows
      const cudaError_t e = launch_gather_s4<GT, 4, 8, 32, 16, CHECK, false, true, true>(g, P, st);
      if (e != cudaErrorInvalidConfiguration) return e;
      return launch_gather_s4<GT, 4, 8, 20, 16, CHECK, false, true, true>(g, P, st);
    }
    case 56: return launch_gather_s4<GT, 2, 8, 16, 24, CHECK, false, true, true>(g, P, st);
    case 57: return launch_gather_s4<GT, 2, 4, 16, 24, CHECK, false, true, true>(g, P, st);
    case 58: return launch_gather_s4<GT, 2, 2, 12, 24, CHECK>(g, P, st);
    default: return launch_gather_t<GT, 2, 2, 2, CHECK>(g, P, st);
  }
}

// fp32 variant (R18): the staged interval-table gather for every batch
// (variants 31-36 and 46-49 select its shape; any other value the default,
// k_gather_s4 with 32-entry group buffers and dynamic tasks).
template <int GT, bool CHECK>
static cudaError_t launch_gather_f32(const DeviceGrid& g, const Params& P, cudaStream_t st) {
  switch (g.unroll) {
    case 32: return launch_gather_s3<GT, 8, 2, 8, 16, CHECK, false, true>(g, P, st);
    case 33: return launch_gather_s3<GT, 4, 2, 8, 16, CHECK, true, true>(g, P, st);
    case 31: return launch_gather_s3<GT, 4, 2, 8, 16, CHECK, false, true>(g, P, st);
    case 34: return launch_gather_s3<GT, 4, 2, 8, 20, CHECK, false, true>(g, P, st);
    case 36: return launch_gather_s3<GT, 4, 4, 6, 24, CHECK, false, true>(g, P, st);
    case 35: return launch_gather_s3<GT, 4, 2, 8, 24, CHECK, false, true>(g, P, st);
    case 47: return launch_gather_s4<GT, 4, 8, 20, 20, CHECK, true>(g, P, st);
    case 48: return launch_gather_s4<GT, 4, 8, 16, 24, CHECK, true>(g, P, st);

    case 46: return launch_gather_s4<GT, 4, 8, 20, 16, CHECK, true, false, true>(g, P, st);
    case 49: return launch_gather_s4<GT, 4, 8, 32, 16, CHECK, true, false, true>(g, P, st);
    default: {
      // = 50: 32-entry group buffers, tasks from the global counter (large
      // gather 1.51 vs 1.54 ms for 46, small 0.594 vs 0.603); 46 for the hash
      // grid (as in binary64) and when the shared memory does not fit
      if (GT != XS_GRID_HASH) {
        const cudaError_t e = launch_gather_s4<GT, 4, 8, 32, 16, CHECK, true, true, true>(g, P, st);
        if (e != cudaErrorInvalidConfiguration) return e;
      }
      return launch_gather_s4<GT, 4, 8, 20, 16, CHECK, true, false, true>(g, P, st);
    }
  }
}

// Kernel choice: energy-sorted batches use the staged gather (variant
// table in launch_gather_tv); unsorted batches the 3-lanes-per-lookup
// kernel, which needs the row layout of the unionized index grid (a
// column-only grid uses the staged gather); the fp32 variant always runs
// the staged gather.
template <int GT>
static cudaError_t launch_gather_u1(const DeviceGrid& g, const Params& P, bool sorted, bool f32,
                                    bool check, cudaStream_t st) {
#ifndef XS_DEV_FAST
  if (f32)
    return check ? launch_gather_f32<GT, true>(g, P, st) : launch_gather_f32<GT, false>(g, P, st);
#endif
  const bool thread_kernel = sorted || (GT == XS_GRID_UNIONIZED && !g.index);
#ifdef XS_DEV_FAST
  // development build (timing experiments only): unionized, unchecked, sorted
  if constexpr (GT == XS_GRID_UNIONIZED) {
    if (!check && thread_kernel) {
      switch (g.unroll) {
        case 56: return launch_gather_s4<GT, 2, 8, 16, 24, false, false, true, true>(g, P, st);
        case 20: return launch_gather_s3<GT, 2, 2, 8, 24, false>(g, P, st);

        case 55: return launch_gather_s4<GT, 4, 8, 20, 16, false, false, true, true>(g, P, st);
        case 57: return launch_gather_s4<GT, 2, 4, 16, 24, false, false, true, true>(g, P, st);
        default: return launch_gather_s4<GT, 4, 8, 32, 16, false, false, true, true>(g, P, st);
      }
    }
  }
  return cudaErrorNotSupported;
#else
  if (thread_kernel)
    return check ? launch_gather_tv<GT, true>(g, P, st) : launch_gather_tv<GT, false>(g, P, st);
  return check ? launch_gather_v<GT, true>(g, P, st) : launch_gather_v<GT, false>(g, P, st);
#endif
}

// Generated energies (dyadic grid) never need the division range checks;
// explicit ones are checked on the device (k_check_energies) and the gather
// runs as a gated pair, so the unchecked kernel does the work whenever the
// batch allows it.  Returns the number of kernels launched in *launches.
template <int GT>
static cudaError_t launch_gather_u(const DeviceGrid& g, const Params& P, bool sorted, bool f32,
                                   uint32_t* gate, cudaStream_t st, int* launches) {
  if (!g.dyadic63) {
    *launches = 1;
    return launch_gather_u1<GT>(g, P, sorted, f32, true, st);
  }
  if (P.in_energy == nullptr || gate == nullptr) {
    *launches = 1;
    return launch_gather_u1<GT>(g, P, sorted, f32, false, st);
  }
  cudaError_t e = cudaMemsetAsync(gate, 0, sizeof(uint32_t), st);
  if (e != cudaSuccess) return e;
  k_check_energies<<<grid_cap(P.count, 256, g.sm_count, 8), 256, 0, st>>>(P.in_energy, P.count,
                                                                             gate);
  Params Q = P;
  Q.gate = gate;
  Q.gate_want = 0;
  e = launch_gather_u1<GT>(g, Q, sorted, f32, false, st);
  if (e != cudaSuccess) return e;
  Q.gate_want = 1;
  *launches = 3;
  return launch_gather_u1<GT>(g, Q, sorted, f32, true, st);
}

static uint32_t part_tiles(uint64_t count, uint32_t tchunks = 0) {
  const uint64_t tlen = static_cast<uint64_t>(tchunks ? tchunks : part_tile_chunks(count)) * kPartChunk;
  const uint64_t t = (count + tlen - 1) / tlen;
  return static_cast<uint32_t>(t < 1 ? 1 : t);
}

// Coarse energy bits of the partitioned A2 (2^7 keys per material).
// A wider key (part_cbits 8, 9) shortens the segments k_part_fine sorts but
// grows the tile histograms and k_part_place's shared memory, and measured
// slower at every size (large 2.85 -> 2.98 ms at 8 bits, XL
// 41.5 -> 42.1 / 42.8 ms at 8 / 9 bits).  Limits: k_part_place holds
// three key arrays and the tile in shared memory, keys are 16 bit, and the
// fine histogram has at most kFineBinsMax bins.
constexpr int kPartCbits = 7, kPartCbitsMin = 6, kPartCbitsMax = 9;

static size_t part_place_smem(uint64_t count, int32_t n_mats, int cbits, bool per_lookup) {
  const size_t nkeys = static_cast<size_t>(n_mats + 1) << cbits;
  const size_t tlen = static_cast<size_t>(part_tile_chunks(count)) * kPartChunk;
  return ((3 * nkeys + 1) * 4 + 15) / 16 * 16 + tlen * (per_lookup ? 14 : 10);
}

bool part_cbits_fit(uint64_t count, int32_t n_mats, int cbits) {
  return cbits >= kPartCbitsMin && cbits <= kPartCbitsMax && (static_cast<size_t>(n_mats + 1) << cbits) <= 65536 &&
         part_place_smem(count, n_mats, cbits, true) + kPickBuckets + 64 <= 227 * 1024;
}

static int part_cbits(uint64_t count, int32_t n_mats, int requested) {
  return requested && part_cbits_fit(count, n_mats, requested) ? requested : kPartCbits;
}

// Bytes the partitioned A2 keeps in the A2 bin area: H [ntiles][nkeys] plus
// the key totals and starts (workspace_layout reserves the larger of this and
// the global-atomic bin array), for the widest coarse key that fits.
static size_t part_bins_need(uint64_t count, size_t nkeys) {
  return (static_cast<size_t>(part_tiles(count)) * nkeys + 2 * nkeys) * 4;
}
size_t part_bins_bytes(uint64_t count, int32_t n_mats) {
  int c = kPartCbits;
  while (c < kPartCbitsMax && part_cbits_fit(count, n_mats, c + 1)) ++c;
  return part_bins_need(count, static_cast<size_t>(n_mats + 1) << c);
}

uint32_t energy_bin_host(double p) { return energy_bin(p); }

// Coarse-key range of the partitioned A2 for a batch: all 2^cbits coarse
// keys per material, or (energy-range shard) only those of [e_lo, e_hi).
struct PartKeys {
  int cbits, kc_lo, nkr;
  size_t nkeys(int32_t n_mats) const { return static_cast<size_t>(n_mats + 1) * nkr; }
};
static PartKeys part_keys(const LookupArgs& a, int cbits) {
  PartKeys k{cbits, 0, 1 << cbits};
  if (a.shard) {
    const int fb = 18 - cbits;
    const uint32_t lo = a.e_lo > 0.0 ? energy_bin(a.e_lo) : 0u;
    const uint32_t hi = a.e_hi < 1.0 ? energy_bin(a.e_hi) : kEnergyBins - 1u;
    k.kc_lo = static_cast<int>(lo >> fb);
    k.nkr = static_cast<int>(hi >> fb) - k.kc_lo + 1;
  }
  return k;
}

template <int GT>
static cudaError_t run_lookup_t(const DeviceGrid& g, const LookupArgs& a, const Workspace& ws,
                                cudaStream_t st) {
  Params P = make_params(g);
  P.first_id = a.first_id;
  P.count = a.count;
  P.in_energy = a.in_energy;
  P.in_mat = a.in_mat;
  P.in_mat8 = a.in_mat8;
  P.counts = ws.counts;
  P.cursor = ws.cursor;
  P.task_next = ws.cursor + (kMaxMats + 1);
  P.recs = ws.recs;
  P.out_M = a.out.macro_xs;
  P.out_E = a.out.energy;
  P.out_mat = a.out.mat;
  P.out_gidx = a.out.grid_index;
  P.out_v = a.out.verification;
  P.vsum = reinterpret_cast<unsigned long long*>(a.out.vsum);
  auto mark = [&](int i) {
    if (a.ev) cudaEventRecord(a.ev[i], st);
  };
  auto launched = [&](uint64_t n) {
    if (a.launches) *a.launches += n;
  };
  cudaError_t e;
  mark(0);
  if (a.flags & XS_FLAG_BASELINE) {
    mark(1);
    mark(2);
    k_baseline<GT><<<grid_cap(a.count, 256, g.sm_count, 16), 256, 0, st>>>(P);
    launched(1);
    mark(3);
    return cudaGetLastError();
  }
  e = cudaMemsetAsync(ws.counts, 0, (2 * (kMaxMats + 1) + 1) * sizeof(uint32_t), st);
  if (e != cudaSuccess) return e;
  const bool binned = a.flags & XS_FLAG_SORT;
  const unsigned nb = grid_cap(a.count, kPrepThreads * kPrepItems, g.sm_count, 16);
  // the staged gather (default for sorted batches) only needs u at each task's
  // extreme energies; per-lookup u is searched when reported or otherwise used
  const int variant = g.unroll;
  P.need_gidx = (!binned || a.out.grid_index ||
                 (!(a.flags & XS_FLAG_F32) && variant != 0 && variant < 9)) ? 1 : 0;
  P.tmp = ws.tmp;
  P.mat8 = ws.mat8;
  const bool f32 = (a.flags & XS_FLAG_F32) != 0;
  const bool staged = f32 || variant == 0 || (variant >= 17 && variant <= 28) ||
                      (variant >= 40 && variant <= 50) || (variant >= 55 && variant <= 59);
  // partitioned A2: the widest coarse key at or below the request whose tile
  // histograms fit the workspace's bin area (a chunk of a host-input batch
  // may allow a wider key than the batch the workspace was sized for)
  PartKeys pk = part_keys(a, part_cbits(a.count, g.n_mats, g.part_cbits));
  if (a.shard && g.part_cbits == 0) {
    // an energy-range shard takes one more coarse bit when its coarse
    // segments would average more than two fine-pass windows (XL) or when its
    // keys would give the fine pass (one block per key and SM) fewer than
    // ~2.5 waves (8 shards): its tile histograms are small (long shard
    // tiles), and more, shorter segments sort faster (A2 per shard, 8 shards:
    // XL 0.73 -> 0.58 ms, large 0.067 -> 0.057 ms)
    const double frac = (a.e_hi < 1.0 ? a.e_hi : 1.0) - (a.e_lo > 0.0 ? a.e_lo : 0.0);
    const double per_key = static_cast<double>(a.count) * (frac > 0.0 ? frac : 0.0) /
                           (static_cast<double>(g.n_mats) * pk.nkr);
    const bool few_keys = 2 * g.n_mats * pk.nkr < 5 * g.sm_count;
    if ((per_key > 2.0 * kFineCapP || few_keys) && part_cbits_fit(a.count, g.n_mats, pk.cbits + 1))
      pk = part_keys(a, pk.cbits + 1);
  }
  while (pk.cbits > kPartCbitsMin &&
         part_bins_need(a.count, pk.nkeys(g.n_mats)) > ws.bins_bytes)
    pk = part_keys(a, pk.cbits - 1);
  const bool part_ok = part_tile_chunks(a.count) <= 12 &&  // k_part_place stages a tile in smem
                       part_cbits_fit(a.count, g.n_mats, pk.cbits) &&
                       part_bins_need(a.count, pk.nkeys(g.n_mats)) <= ws.bins_bytes;
  if (a.shard && !(binned && staged && !g.legacy_sort && part_ok))
    return cudaErrorNotSupported;  // energy-range shards need the partitioned A2
  if (binned && staged && !g.legacy_sort && part_ok) {
    // partitioned A2 (k_part_*) feeding the staged gather: energies (+ batch
    // positions when per-lookup results are written) in sorted order
    P.need_gidx = 0;
    P.cbits = pk.cbits;
    P.kc_lo = pk.kc_lo;
    P.nkr = pk.nkr;
    P.shard = a.shard ? 1 : 0;
    P.e_lo = a.e_lo;
    P.e_hi = a.e_hi;
    if (a.shard) {  // min{s : RN(s) 2^-63 >= e} by bisection (RN is monotone)
      auto first_at_least = [](double e) -> uint64_t {
        if (!(e > 0.0)) return 0;
        if (lcg_double(kMask63) < e) return kMask63 + 1;
        uint64_t lo = 0, hi = kMask63;  // lcg_double(lo) < e <= lcg_double(hi)
        while (hi - lo > 1) {
          const uint64_t mid = lo + (hi - lo) / 2;
          if (lcg_double(mid) >= e) hi = mid; else lo = mid;
        }
        return hi;
      };
      P.s_lo = first_at_least(a.e_lo);
      P.s_hi = first_at_least(a.e_hi);
    }
    P.fine_direct = g.fine_direct;
    const int nkeys = static_cast<int>(pk.nkeys(g.n_mats));
    // an energy-range shard keeps ~1/n of each tile's lookups: its tiles are
    // n/2 times longer (up to 16x), so that the tile histograms, their column
    // scan and the per-tile stream setup shrink while k_part_place still
    // stages few enough lookups per tile for two blocks per SM (measured,
    // large: n/2 beats 1 and n at n = 2, 4, 8)
    uint32_t tmult = 1;
    if (a.shard) {
      const double lo = a.e_lo > 0.0 ? a.e_lo : 0.0, hi = a.e_hi < 1.0 ? a.e_hi : 1.0;
      const double inv = hi > lo ? 0.5 / (hi - lo) : 16.0;
      tmult = inv >= 16.0 ? 16u : static_cast<uint32_t>(inv);
      const uint32_t cap = g.shard_tiles ? static_cast<uint32_t>(g.shard_tiles) : 16u;
      if (tmult > cap) tmult = cap;
      if (tmult < 1) tmult = 1;
    }
    P.tchunks = part_tile_chunks(a.count) * tmult;
    const uint32_t ntiles = part_tiles(a.count, P.tchunks);
    const unsigned nb = ntiles < static_cast<uint32_t>(g.sm_count) * 16 ? ntiles : g.sm_count * 16;
    P.bins = ws.bins;  // H [ntiles][nkeys]
    P.key_tot = ws.bins + static_cast<size_t>(ntiles) * nkeys;
    P.key_start = P.key_tot + nkeys;
    const bool per_lookup = a.out.macro_xs || a.out.verification;
    P.sp_tmp = reinterpret_cast<double*>(ws.tmp);
    P.sidx_tmp = per_lookup ? reinterpret_cast<uint32_t*>(P.sp_tmp + a.count) : nullptr;
    double* sp = reinterpret_cast<double*>(ws.recs);
    P.sp = sp;
    P.sidx = per_lookup ? reinterpret_cast<uint32_t*>(sp + a.count) : nullptr;
    // shard mode: k_part_count keeps the shard's lookups of tile t at slots
    // t * tlen + q, q < the tile's lookups (so every slot is < count): energy
    // and (position << 16 | key) in the record area (16 B per lookup), which
    // k_part_fine writes only after k_part_place has read them
    if (a.shard) {
      P.slab_p = sp;
      P.slab_k = reinterpret_cast<uint64_t*>(sp + a.count);
    }
    const size_t hs = static_cast<size_t>(nkeys) * 4;
    // energy-range shards without per-lookup outputs: the compacting count
    const bool outputs = a.out.energy || a.out.mat || a.out.grid_index;
    if (a.shard && !outputs)
      k_part_count_shard<<<nb, kPrepThreads, hs, st>>>(P);
    else
      k_part_count<GT><<<nb, kPrepThreads, hs, st>>>(P);
    mark(1);
    if (nkeys >= 32 * 148)
      k_part_colscan<32, 32><<<(nkeys + 31) / 32, dim3(32, 32), 0, st>>>(P, static_cast<int>(ntiles));
    else if (nkeys >= 8 * 148)
      k_part_colscan<8, 128><<<(nkeys + 7) / 8, dim3(8, 128), 0, st>>>(P, static_cast<int>(ntiles));
    else
      k_part_colscan<2, 512><<<(nkeys + 1) / 2, dim3(2, 512), 0, st>>>(P, static_cast<int>(ntiles));
    k_part_keyscan<<<1, 1024, 0, st>>>(P);
    {
      // staging: the whole tile, or (shard) its expected share with a wide
      // margin (ranks beyond it are stored directly), so that several blocks
      // share an SM
      const uint32_t tlen = P.tchunks * kPartChunk;
      P.place_cap = tlen;
      if (a.shard) {
        const double lo = a.e_lo > 0.0 ? a.e_lo : 0.0, hi = a.e_hi < 1.0 ? a.e_hi : 1.0;
        const double want = (hi > lo ? hi - lo : 0.0) * 1.25 * tlen + 1024.0;
        if (want < tlen) P.place_cap = (static_cast<uint32_t>(want) + 255u) & ~255u;
      }
      const size_t pl_smem = (static_cast<size_t>(3 * nkeys + 1) * 4 + 15) / 16 * 16 +
                             static_cast<size_t>(P.place_cap) * (per_lookup ? 14 : 10);
      e = cudaFuncSetAttribute(k_part_place<GT, kPlaceThreads>,
                               cudaFuncAttributeMaxDynamicSharedMemorySize, static_cast<int>(pl_smem));
      if (e != cudaSuccess) return e;
      k_part_place<GT, kPlaceThreads><<<nb, kPlaceThreads, pl_smem, st>>>(P);
    }
    {
      // window: fine_cap energies (2/3 of it with batch positions), default
      // the most that fits one 1024-thread block per SM
      const uint32_t cap_p = g.fine_cap ? static_cast<uint32_t>(g.fine_cap) : kFineCapP;
      P.fine_cap = static_cast<int>(per_lookup ? (g.fine_cap ? cap_p * 2 / 3 : kFineCapPI) : cap_p);
      const size_t fine_smem = fine_hist_bytes(1u << (18 - P.cbits)) +
                               static_cast<size_t>(P.fine_cap) * (per_lookup ? 12 : 8);
      e = cudaFuncSetAttribute(k_part_fine, cudaFuncAttributeMaxDynamicSharedMemorySize,
                               static_cast<int>(fine_smem));
      if (e != cudaSuccess) return e;
      k_part_fine<<<g.n_mats * P.nkr, kFineThreads, fine_smem, st>>>(P);
    }
    launched(5);
  } else if (binned) {
    P.bins = ws.bins;
    e = cudaMemsetAsync(ws.bins, 0, static_cast<size_t>(g.n_mats + 1) * kEnergyBins * 4, st);
    if (e != cudaSuccess) return e;
    P.partials = ws.partials;
    P.perm = ws.perm;
    const uint32_t nchunks = static_cast<uint32_t>(g.n_mats + 1) * (kEnergyBins / kScanChunk);
    k_sample<GT, true><<<nb, kPrepThreads, 0, st>>>(P);
    mark(1);
    k_scan_partial<<<nchunks, 1024, 0, st>>>(P);
    k_scan_top<<<1, 1024, 0, st>>>(P, nchunks);
    k_scan_apply<<<nchunks, 1024, 0, st>>>(P);
    k_scatter<true><<<nb, kPrepThreads, 0, st>>>(P);
    launched(5);
  } else {
    k_sample<GT, false><<<nb, kPrepThreads, 0, st>>>(P);
    mark(1);
    k_scatter<false><<<nb, kPrepThreads, 0, st>>>(P);
    launched(2);
  }
  if ((e = cudaGetLastError()) != cudaSuccess) return e;
  mark(2);
  int nl = 0;
  e = launch_gather_u<GT>(g, P, binned, (a.flags & XS_FLAG_F32) != 0,
                         a.energy_sampled ? nullptr : ws.gate, st, &nl);
  launched(nl);
  mark(3);
  return e;
}

cudaError_t run_lookup(const DeviceGrid& g, const LookupArgs& a, const Workspace& ws,
                       cudaStream_t st) {
  switch (g.grid_type) {
    case XS_GRID_UNIONIZED: return run_lookup_t<XS_GRID_UNIONIZED>(g, a, ws, st);
    case XS_GRID_HASH: return run_lookup_t<XS_GRID_HASH>(g, a, ws, st);
    default: return run_lookup_t<XS_GRID_NUCLIDE>(g, a, ws, st);
  }
}

// ------------------------------------------------- history mode (R19) ---
// XSBench's history driver: particle q carries one
// LCG stream through L chained lookups; after each lookup the stream skips
// n_forward = #{c : M_c > 1.0} draws, then draws the next energy and
// material.  On the device the chain runs as L rounds: every round is one
// explicit-lookup batch over all particles (A2-A8 through run_lookup: the
// same kernels as event mode, material-bucketed), then k_hist_advance applies
// the data dependence.  Results are those of the serial chain (each lookup
// depends only on its own energy and material).
__global__ void k_hist_init(uint64_t seed, uint64_t first, uint32_t n, int32_t L, uint64_t* st,
                            double* E, int32_t* mat) {
  for (uint32_t q = blockIdx.x * blockDim.x + threadIdx.x; q < n; q += gridDim.x * blockDim.x) {
    uint64_t s = fast_forward(seed, 10ull * static_cast<uint64_t>(L) * (first + q));
    s = lcg_next(s);
    E[q] = lcg_double(s);
    s = lcg_next(s);
    mat[q] = pick_material_state(s);
    st[q] = s;
  }
}

__global__ void k_hist_advance(HistoryArgs h, int32_t i) {
  for (uint32_t q = blockIdx.x * blockDim.x + threadIdx.x; q < h.n_particles;
       q += gridDim.x * blockDim.x) {
    double M[5];
#pragma unroll
    for (int c = 0; c < 5; ++c) M[c] = h.hist_M[static_cast<uint64_t>(q) * 5 + c];
    const uint64_t o = static_cast<uint64_t>(q) * h.lookups + i;
    if (h.out.macro_xs)
      for (int c = 0; c < 5; ++c) h.out.macro_xs[o * 5 + c] = M[c];
    if (h.out.energy) h.out.energy[o] = h.hist_energy[q];
    if (h.out.mat) h.out.mat[o] = h.hist_mat[q];
    if (h.out.verification) {
      double mx = -1.0;
      int vi = 0;
      for (int c = 0; c < 5; ++c)
        if (M[c] > mx) {
          mx = M[c];
          vi = c;
        }
      h.out.verification[o] = vi + 1;
    }
    int nf = 0;
#pragma unroll
    for (int c = 0; c < 5; ++c) nf += M[c] > 1.0 ? 1 : 0;
    uint64_t s = h.hist_state[q];
    for (int k = 0; k < nf; ++k) s = lcg_next(s);
    s = lcg_next(s);
    h.hist_energy[q] = lcg_double(s);
    s = lcg_next(s);
    h.hist_mat[q] = pick_material_state(s);
    h.hist_state[q] = s;
  }
}

cudaError_t run_history(const DeviceGrid& g, const HistoryArgs& h, const Workspace& ws,
                        cudaStream_t st) {
  const unsigned nb = grid_cap(h.n_particles, 256, g.sm_count, 8);
  k_hist_init<<<nb, 256, 0, st>>>(g.lookup_seed, h.first_particle, h.n_particles, h.lookups,
                                  h.hist_state, h.hist_energy, h.hist_mat);
  if (h.launches) *h.launches += 1;
  cudaError_t e = cudaGetLastError();
  for (int32_t i = 0; i < h.lookups && e == cudaSuccess; ++i) {
    LookupArgs a;
    a.count = h.n_particles;
    a.flags = h.flags & XS_FLAG_SORT;
    a.in_energy = h.hist_energy;
    a.energy_sampled = true;  // LCG draws in [0, 1]: the unchecked gather is exact
    a.in_mat = h.hist_mat;
    a.out.macro_xs = h.hist_M;
    a.out.vsum = h.out.vsum;
    a.launches = h.launches;
    e = run_lookup(g, a, ws, st);
    if (e != cudaSuccess) break;
    k_hist_advance<<<nb, 256, 0, st>>>(h, i);
    if (h.launches) *h.launches += 1;
    e = cudaGetLastError();
  }
  return e;
}

cudaError_t run_verify(const DeviceGrid& g, const double* M, uint64_t count, uint64_t* vsum,
                       cudaStream_t st) {
  k_verify<<<grid_cap(count, 256, g.sm_count, 8), 256, 0, st>>>(
      M, count, reinterpret_cast<unsigned long long*>(vsum));
  return cudaGetLastError();
}

cudaError_t run_nuclide_index(const DeviceGrid& g, const double* energy, const int32_t* nuc,
                              uint64_t count, int32_t* k_out, cudaStream_t st) {
  Params P = make_params(g);
  const unsigned nb = grid_cap(count, 256, g.sm_count, 8);
  switch (g.grid_type) {
    case XS_GRID_UNIONIZED:
      k_nuclide_index<XS_GRID_UNIONIZED><<<nb, 256, 0, st>>>(P, energy, nuc, count, k_out);
      break;
    case XS_GRID_HASH:
      k_nuclide_index<XS_GRID_HASH><<<nb, 256, 0, st>>>(P, energy, nuc, count, k_out);
      break;
    default:
      k_nuclide_index<XS_GRID_NUCLIDE><<<nb, 256, 0, st>>>(P, energy, nuc, count, k_out);
  }
  return cudaGetLastError();
}

}  // namespace xs
