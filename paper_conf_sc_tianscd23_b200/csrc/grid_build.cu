// grid_build.cu — device construction of the acceleration tables (run once
// per grid at xs_init_grid; not part of the timed lookup step).
//
//   K0a  U  = sorted multiset of all I*N energies      (in-house LSD radix sort)
//   K0b  IG[e][n] = clamp(ub(E_n, U[e]) - 1, 0, N-2)   (chunked search + sweep)
//   K0c  HG[b][n] = clamp(ub(E_n, b du) - 1, 0, N-2)   (one search per entry)
//   K0d  IV[n][k]  = interval terms of record pair (k, k+1) (see below)
//   K0e  IV32[n][k] = the same for the fp32 variant (R18)
// Definitions: DESIGN.md R6, R7 (north_star: "the unionized (or
// hash-accelerated) energy grid").
#include "common.cuh"
#include "radix_sort.cuh"
#include "search.cuh"
#include "xs_internal.h"

namespace xs {

// order-preserving map fp64 bits -> u64 (total order of non-NaN doubles)
__device__ __forceinline__ uint64_t f2key(double x) {
  uint64_t b = static_cast<uint64_t>(__double_as_longlong(x));
  return (b >> 63) ? ~b : (b | 0x8000000000000000ULL);
}
__device__ __forceinline__ double key2f(uint64_t k) {
  uint64_t b = (k >> 63) ? (k & 0x7fffffffffffffffULL) : ~k;
  return __longlong_as_double(static_cast<long long>(b));
}

__global__ void k_extract_energy_keys(const double* __restrict__ grid, uint64_t n,
                                      uint64_t* __restrict__ keys) {
  for (uint64_t i = blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x; i < n;
       i += static_cast<uint64_t>(gridDim.x) * blockDim.x)
    keys[i] = f2key(grid[i * 6]);
}

__global__ void k_keys_to_energy(const uint64_t* __restrict__ keys, uint64_t n,
                                 double* __restrict__ U) {
  for (uint64_t i = blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x; i < n;
       i += static_cast<uint64_t>(gridDim.x) * blockDim.x)
    U[i] = key2f(keys[i]);
}

static int grid_for(uint64_t n, int threads, int sm) {
  uint64_t b = (n + threads - 1) / threads;
  uint64_t cap = static_cast<uint64_t>(sm) * 32;
  return static_cast<int>(b < cap ? (b ? b : 1) : cap);
}

cudaError_t build_union_grid(const DeviceGrid& g, double* U, cudaStream_t st) {
  const uint64_t n = static_cast<uint64_t>(g.NU);
  uint64_t* k0 = nullptr;
  uint64_t* k1 = nullptr;
  void* work = nullptr;
  cudaError_t e = cudaMallocAsync(&k0, n * 8, st);
  if (e == cudaSuccess) e = cudaMallocAsync(&k1, n * 8, st);
  if (e == cudaSuccess) e = cudaMallocAsync(&work, rs::hist_bytes(n), st);
  if (e == cudaSuccess) {
    k_extract_energy_keys<<<grid_for(n, 256, g.sm_count), 256, 0, st>>>(g.grid, n, k0);
    bool in1 = false;
    e = rs::sort_pairs<uint64_t, false>(k0, nullptr, k1, nullptr, n, 64, work, st, &in1);
    if (e == cudaSuccess) {
      k_keys_to_energy<<<grid_for(n, 256, g.sm_count), 256, 0, st>>>(in1 ? k1 : k0, n, U);
      e = cudaGetLastError();
    }
  }
  if (k0) cudaFreeAsync(k0, st);
  if (k1) cudaFreeAsync(k1, st);
  if (work) cudaFreeAsync(work, st);
  return e;
}

// K0b: block b owns rows [b R, (b+1) R); thread t owns nuclides t, t+T, ...
// One binary search per (block, nuclide), then a monotone sweep: writes of a
// row are consecutive in n (coalesced), reads of E_n advance monotonically.
constexpr int kIgRows = 256;

__global__ void __launch_bounds__(384) k_build_index_grid(const double* __restrict__ grid,
                                                          int32_t I, int64_t N,
                                                          const double* __restrict__ U,
                                                          int64_t NU, int32_t* __restrict__ IG) {
  const int64_t e0 = static_cast<int64_t>(blockIdx.x) * kIgRows;
  const int64_t e1 = e0 + kIgRows < NU ? e0 + kIgRows : NU;
  for (int32_t n = threadIdx.x; n < I; n += blockDim.x) {
    const double* rec = grid + static_cast<int64_t>(n) * N * 6;
    int64_t k = bracket_search_rec(rec, 0, N - 1, __ldg(U + e0));
    double e_next = rec_energy(rec, k + 1);
    for (int64_t e = e0; e < e1; ++e) {
      const double q = __ldg(U + e);
      while (k < N - 2 && e_next <= q) {
        ++k;
        e_next = rec_energy(rec, k + 1);
      }
      IG[e * I + n] = static_cast<int32_t>(k);
    }
  }
}

cudaError_t build_index_grid(const DeviceGrid& g, cudaStream_t st) {
  const int64_t blocks = (g.NU + kIgRows - 1) / kIgRows;
  const int threads = g.I >= 384 ? 384 : ((g.I + 31) / 32) * 32;
  k_build_index_grid<<<static_cast<unsigned>(blocks), threads, 0, st>>>(g.grid, g.I, g.N, g.U,
                                                                         g.NU, g.index);
  return cudaGetLastError();
}

// K0b' (column layout): IGT[n][e] = clamp(ub(E_n, U[e]) - 1, 0, N-2).
// Block (x, n): warp w sweeps 256 consecutive unionized energies of nuclide
// n in steps of 32 (one per lane, coalesced 128-B writes).  The bracket of
// the first energy comes from one binary search; each later lane advances
// from its warp's previous bracket (energies increase along e).
constexpr int kIgtPerWarp = 256;

__global__ void __launch_bounds__(256) k_build_index_grid_t(const double* __restrict__ grid,
                                                           int64_t N,
                                                           const double* __restrict__ U,
                                                           int64_t NU, int32_t* __restrict__ IGT) {
  const int32_t n = blockIdx.y;
  const int lane = threadIdx.x & 31;
  const int64_t e_begin = (static_cast<int64_t>(blockIdx.x) * (blockDim.x >> 5) +
                           (threadIdx.x >> 5)) * kIgtPerWarp;
  if (e_begin >= NU) return;
  const double* rec = grid + static_cast<int64_t>(n) * N * 6;
  int64_t kw = bracket_search_rec(rec, 0, N - 1, __ldg(U + e_begin));  // warp-uniform
  int32_t* col = IGT + static_cast<int64_t>(n) * NU;
  for (int64_t e0 = e_begin; e0 < e_begin + kIgtPerWarp && e0 < NU; e0 += 32) {
    const int64_t e = e0 + lane;
    int64_t k = kw;
    if (e < NU) {
      const double q = __ldg(U + e);
      while (k < N - 2 && rec_energy(rec, k + 1) <= q) ++k;
      col[e] = static_cast<int32_t>(k);
    }
    kw = __shfl_sync(0xffffffffu, k, 31);  // last lane's bracket (monotone in e)
    if (e0 + 32 > NU) break;
  }
}

cudaError_t build_index_grid_t(const DeviceGrid& g, cudaStream_t st) {
  const int64_t per_block = 8 * kIgtPerWarp;
  dim3 grid(static_cast<unsigned>((g.NU + per_block - 1) / per_block), static_cast<unsigned>(g.I));
  k_build_index_grid_t<<<grid, 256, 0, st>>>(g.grid, g.N, g.U, g.NU, g.index_t);
  return cudaGetLastError();
}

__global__ void k_build_hash_grid(const double* __restrict__ grid, int32_t I, int64_t N, int32_t B,
                                  double du, int32_t* __restrict__ HG) {
  const uint64_t total = static_cast<uint64_t>(B) * I;
  for (uint64_t t = blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x; t < total;
       t += static_cast<uint64_t>(gridDim.x) * blockDim.x) {
    const int64_t b = static_cast<int64_t>(t / I);
    const int32_t n = static_cast<int32_t>(t % I);
    const double energy = static_cast<double>(b) * du;
    HG[t] = static_cast<int32_t>(
        bracket_search_rec(grid + static_cast<int64_t>(n) * N * 6, 0, N - 1, energy));
  }
}

cudaError_t build_hash_grid(const DeviceGrid& g, cudaStream_t st) {
  const uint64_t total = static_cast<uint64_t>(g.B) * g.I;
  k_build_hash_grid<<<grid_for(total, 256, g.sm_count), 256, 0, st>>>(g.grid, g.I, g.N, g.B,
                                                                        g.du, g.index);
  return cudaGetLastError();
}

// UB[b] = ub(U, b / UBn) = #{U <= b / UBn}, b = 0..UBn: equal-width energy
// bins over the unionized grid, so the A3 search for p in bin b only has to
// run inside [UB[b] - 1, UB[b + 1]] (same result as the full search; DESIGN.md
// §4 "A3").
__global__ void k_union_table(const double* __restrict__ U, int64_t NU, int32_t UBn,
                              int32_t* __restrict__ UB) {
  const double inv = 1.0 / static_cast<double>(UBn);
  for (int64_t b = blockIdx.x * static_cast<int64_t>(blockDim.x) + threadIdx.x; b <= UBn;
       b += static_cast<int64_t>(gridDim.x) * blockDim.x) {
    const double e = static_cast<double>(b) * inv;
    int64_t lo = 0, hi = NU;
    while (lo < hi) {
      const int64_t mid = lo + ((hi - lo) >> 1);
      if (U[mid] <= e)
        lo = mid + 1;
      else
        hi = mid;
    }
    UB[b] = static_cast<int32_t>(lo);
  }
}

cudaError_t build_union_table(const DeviceGrid& g, cudaStream_t st) {
  k_union_table<<<grid_for(static_cast<uint64_t>(g.UBn) + 1, 256, g.sm_count), 256, 0, st>>>(
      g.U, g.NU, g.UBn, g.UB);
  return cudaGetLastError();
}

// K0d: interval table.  For the record pair (k, k+1) of nuclide n, the 14
// doubles {E[k+1], E[k+1] - E[k], recip(E[k+1] - E[k]), 0, then hi.c,
// hi.c - lo.c for c = 0..4}: the pair-only terms of A6 (DESIGN.md
// R10), computed with the same IEEE operations the lookup kernels use
// (dsub, recip_nr), so interpolating from them is bit-identical to
// interpolating from the two records.  Entry k = N-1 (no pair) is zero.
__global__ void k_build_intervals(const double* __restrict__ grid, uint64_t total, int64_t N,
                                  double* __restrict__ IV) {
  for (uint64_t t = blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x; t < total;
       t += static_cast<uint64_t>(gridDim.x) * blockDim.x) {
    double* o = IV + t * kIvDoubles;
    if (static_cast<int64_t>(t % static_cast<uint64_t>(N)) == N - 1) {
      for (int q = 0; q < kIvDoubles; ++q) o[q] = 0.0;
      continue;
    }
    const double* lo = grid + t * 6;
    const double* hi = lo + 6;
    const double bd = dsub(hi[0], lo[0]);
    o[0] = hi[0];
    o[1] = bd;
    o[2] = recip_nr(bd);
    o[3] = 0.0;
    for (int c = 0; c < 5; ++c) {
      o[4 + 2 * c] = hi[1 + c];
      o[5 + 2 * c] = dsub(hi[1 + c], lo[1 + c]);
    }
  }
}

// K0e: fp32-variant interval table (R18), 80-B entries:
// {E[k+1], gap} {recip(gap), 0} then float4 {h0, d0, h1, d1} {h2, d2, h3, d3}
// {h4, d4, 0, 0} with h = (float) hi.c and d = h - (float) lo.c (binary32).
__global__ void k_build_intervals32(const double* __restrict__ grid, uint64_t total, int64_t N,
                                    double* __restrict__ IV) {
  for (uint64_t t = blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x; t < total;
       t += static_cast<uint64_t>(gridDim.x) * blockDim.x) {
    double* o = IV + t * kIv32Doubles;
    float* of = reinterpret_cast<float*>(o + 4);
    if (static_cast<int64_t>(t % static_cast<uint64_t>(N)) == N - 1) {
      for (int q = 0; q < kIv32Doubles; ++q) o[q] = 0.0;
      continue;
    }
    const double* lo = grid + t * 6;
    const double* hi = lo + 6;
    const double bd = dsub(hi[0], lo[0]);
    o[0] = hi[0];
    o[1] = bd;
    o[2] = recip_nr(bd);
    o[3] = 0.0;
    for (int c = 0; c < 5; ++c) {
      const float h = __double2float_rn(hi[1 + c]);
      const float l = __double2float_rn(lo[1 + c]);
      of[2 * c] = h;
      of[2 * c + 1] = __fsub_rn(h, l);
    }
    of[10] = 0.0f;
    of[11] = 0.0f;
  }
}

cudaError_t build_intervals32(const DeviceGrid& g, cudaStream_t st) {
  const uint64_t total = static_cast<uint64_t>(g.I) * g.N;
  k_build_intervals32<<<grid_for(total, 256, g.sm_count), 256, 0, st>>>(g.grid, total, g.N,
                                                                        g.iv32);
  return cudaGetLastError();
}

// K0u: the unsorted gather's interval table (k_gather_u), 96-B entries,
// 32-B aligned: {E[k+1], gap, h0, d0, h1, d1, h2, d2, h3, d3, h4, d4} with
// h = hi.c and d = hi.c - lo.c (the operations of K0d); entry N-1 is zero.
__global__ void k_build_intervals_u(const double* __restrict__ grid, uint64_t total, int64_t N,
                                    double* __restrict__ IV) {
  for (uint64_t t = blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x; t < total;
       t += static_cast<uint64_t>(gridDim.x) * blockDim.x) {
    double* o = IV + t * 12;
    if (static_cast<int64_t>(t % static_cast<uint64_t>(N)) == N - 1) {
      for (int q = 0; q < 12; ++q) o[q] = 0.0;
      continue;
    }
    const double* lo = grid + t * 6;
    const double* hi = lo + 6;
    o[0] = hi[0];
    o[1] = dsub(hi[0], lo[0]);
    for (int c = 0; c < 5; ++c) {
      o[2 + 2 * c] = hi[1 + c];
      o[3 + 2 * c] = dsub(hi[1 + c], lo[1 + c]);
    }
  }
}

cudaError_t build_intervals_u(const DeviceGrid& g, cudaStream_t st) {
  const uint64_t total = static_cast<uint64_t>(g.I) * g.N;
  k_build_intervals_u<<<grid_for(total, 256, g.sm_count), 256, 0, st>>>(g.grid, total, g.N, g.ivu);
  return cudaGetLastError();
}

cudaError_t build_intervals(const DeviceGrid& g, cudaStream_t st) {
  const uint64_t total = static_cast<uint64_t>(g.I) * g.N;
  k_build_intervals<<<grid_for(total, 256, g.sm_count), 256, 0, st>>>(g.grid, total, g.N, g.iv);
  return cudaGetLastError();
}

}  // namespace xs
