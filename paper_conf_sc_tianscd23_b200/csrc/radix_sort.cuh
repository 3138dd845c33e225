// radix_sort.cuh — in-house stable LSD radix sort (8-bit digits) for u32 or
// u64 keys with optional u32 values.  Used for
//   K0a  the unionized energy grid (u64 keys = order-preserving bit images of
//        the fp64 energies), at init;
//   A2   the optional (material, energy) sort of a lookup batch
//        (north_star: "an optional on-device sort of lookups by material and
//        energy ... built from an in-house radix pass").
//
// One pass = three kernels on the caller's stream:
//   rs_hist     per-tile 256-bin histogram -> hist[digit][tile]
//   rs_scan     per-digit exclusive scan over tiles (+ digit totals)
//   rs_scatter  stable per-tile ranking (warp match + cross-warp prefix in
//               shared memory) and scatter to the output position
// No host synchronisation; the workspace holds hist[256 * tiles] + totals.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace xs {
namespace rs {

constexpr int kThreads = 256;
constexpr int kWarps = kThreads / 32;
constexpr int kItems = 16;                    // keys per thread per tile
constexpr int kTile = kThreads * kItems;      // 4096 keys per tile

__host__ __device__ inline uint64_t num_tiles(uint64_t n) { return (n + kTile - 1) / kTile; }

// workspace bytes for a sort of n keys (histogram + totals)
__host__ inline size_t hist_bytes(uint64_t n) {
  return (256 * num_tiles(n) + 256) * sizeof(uint32_t);
}

template <typename K>
__device__ __forceinline__ uint32_t digit_of(K k, int shift) {
  return static_cast<uint32_t>(k >> shift) & 0xffu;
}

template <typename K>
__global__ void __launch_bounds__(kThreads) rs_hist(const K* __restrict__ keys, uint64_t n,
                                                    int shift, uint32_t* __restrict__ hist,
                                                    uint32_t tiles) {
  __shared__ uint32_t s_h[256];
  s_h[threadIdx.x] = 0;
  __syncthreads();
  uint64_t base = static_cast<uint64_t>(blockIdx.x) * kTile;
#pragma unroll 4
  for (int it = 0; it < kItems; ++it) {
    uint64_t i = base + static_cast<uint64_t>(it) * kThreads + threadIdx.x;
    if (i < n) atomicAdd(&s_h[digit_of(keys[i], shift)], 1u);
  }
  __syncthreads();
  hist[static_cast<uint64_t>(threadIdx.x) * tiles + blockIdx.x] = s_h[threadIdx.x];
}

// grid = 256 blocks (one per digit); block d scans hist[d][0..tiles) in place.
static __global__ void __launch_bounds__(1024) rs_scan(uint32_t* __restrict__ hist, uint32_t tiles,
                                                uint32_t* __restrict__ totals) {
  __shared__ uint32_t s_w[32];
  __shared__ uint32_t s_carry;
  uint32_t* row = hist + static_cast<uint64_t>(blockIdx.x) * tiles;
  if (threadIdx.x == 0) s_carry = 0;
  __syncthreads();
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  for (uint32_t c0 = 0; c0 < tiles; c0 += blockDim.x) {
    uint32_t i = c0 + threadIdx.x;
    uint32_t v = i < tiles ? row[i] : 0u;
    uint32_t x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
      if (lane >= o) x += y;
    }
    if (lane == 31) s_w[w] = x;
    __syncthreads();
    if (w == 0) {
      uint32_t t = lane < (int)(blockDim.x >> 5) ? s_w[lane] : 0u;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        uint32_t y = __shfl_up_sync(0xffffffffu, t, o);
        if (lane >= o) t += y;
      }
      s_w[lane] = t;  // inclusive prefix over warps
    }
    __syncthreads();
    uint32_t carry = s_carry;
    uint32_t excl = carry + (w ? s_w[w - 1] : 0u) + x - v;
    if (i < tiles) row[i] = excl;
    __syncthreads();
    if (threadIdx.x == blockDim.x - 1) s_carry = carry + s_w[(blockDim.x >> 5) - 1];
    __syncthreads();
  }
  if (threadIdx.x == 0) totals[blockIdx.x] = s_carry;
}

template <typename K, bool kHasVal>
__global__ void __launch_bounds__(kThreads) rs_scatter(const K* __restrict__ keys_in,
                                                       const uint32_t* __restrict__ vals_in,
                                                       K* __restrict__ keys_out,
                                                       uint32_t* __restrict__ vals_out,
                                                       uint64_t n, int shift,
                                                       const uint32_t* __restrict__ hist,
                                                       uint32_t tiles,
                                                       const uint32_t* __restrict__ totals) {
  __shared__ uint32_t s_run[256];          // next output position per digit
  __shared__ uint32_t s_wc[kWarps][256];   // per-round per-warp digit counts -> offsets
  __shared__ uint32_t s_tot[256];
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  // digit bases: exclusive scan of totals (256 entries, one per thread)
  {
    uint32_t v = totals[tid];
    s_tot[tid] = v;
    __syncthreads();
    // simple Hillis-Steele scan in shared memory
    for (int o = 1; o < 256; o <<= 1) {
      uint32_t y = tid >= o ? s_tot[tid - o] : 0u;
      __syncthreads();
      s_tot[tid] += y;
      __syncthreads();
    }
    s_run[tid] = s_tot[tid] - v + hist[static_cast<uint64_t>(tid) * tiles + blockIdx.x];
  }
  const uint32_t lt_mask = (1u << lane) - 1u;
  uint64_t base = static_cast<uint64_t>(blockIdx.x) * kTile;
  for (int it = 0; it < kItems; ++it) {
    uint64_t i = base + static_cast<uint64_t>(it) * kThreads + tid;
    const bool valid = i < n;
    K k = valid ? keys_in[i] : K(0);
    uint32_t val = 0;
    if (kHasVal && valid) val = vals_in[i];
    const uint32_t d = valid ? digit_of(k, shift) : 256u;
    const uint32_t peers = __match_any_sync(0xffffffffu, d);
    const uint32_t rank = __popc(peers & lt_mask);
    const bool leader = (__ffs(peers) - 1) == lane;
#pragma unroll
    for (int q = 0; q < kWarps; ++q) s_wc[q][tid] = 0u;
    __syncthreads();
    if (leader && valid) s_wc[w][d] = __popc(peers);
    __syncthreads();
    {
      uint32_t run = s_run[tid];
#pragma unroll
      for (int q = 0; q < kWarps; ++q) {
        uint32_t c = s_wc[q][tid];
        s_wc[q][tid] = run;
        run += c;
      }
      s_run[tid] = run;
    }
    __syncthreads();
    if (valid) {
      uint32_t pos = s_wc[w][d] + rank;
      keys_out[pos] = k;
      if (kHasVal) vals_out[pos] = val;
    }
    __syncthreads();
  }
}

// Sort n keys (with optional values) by bits [0, nbits) (nbits multiple of 8).
// Ping-pongs between (k0, v0) and (k1, v1); returns true if the result ends
// in (k1, v1).  `work` must hold hist_bytes(n).  n < 2^32.
template <typename K, bool kHasVal>
inline cudaError_t sort_pairs(K* k0, uint32_t* v0, K* k1, uint32_t* v1, uint64_t n, int nbits,
                              void* work, cudaStream_t st, bool* result_in_1,
                              const bool* skip_digit = nullptr) {
  *result_in_1 = false;
  if (n == 0) return cudaSuccess;
  const uint32_t tiles = static_cast<uint32_t>(num_tiles(n));
  uint32_t* hist = static_cast<uint32_t*>(work);
  uint32_t* totals = hist + 256ull * tiles;
  K* kin = k0;
  K* kout = k1;
  uint32_t* vin = v0;
  uint32_t* vout = v1;
  for (int shift = 0, pass = 0; shift < nbits; shift += 8, ++pass) {
    if (skip_digit && skip_digit[pass]) continue;
    rs_hist<K><<<tiles, kThreads, 0, st>>>(kin, n, shift, hist, tiles);
    rs_scan<<<256, 1024, 0, st>>>(hist, tiles, totals);
    rs_scatter<K, kHasVal><<<tiles, kThreads, 0, st>>>(kin, vin, kout, vout, n, shift, hist, tiles,
                                                       totals);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    K* tk = kin; kin = kout; kout = tk;
    uint32_t* tv = vin; vin = vout; vout = tv;
    *result_in_1 = !*result_in_1;
  }
  return cudaSuccess;
}

}  // namespace rs
}  // namespace xs
