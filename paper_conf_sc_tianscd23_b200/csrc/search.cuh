// search.cuh — device searches of the lookup path (A3/A4; R5-R9).
//
//   ub(A, q)        = #{x in A : x <= q}  (upper-bound semantics: an energy
//                     equal to a grid point starts the bracket at that point)
//   bracket k_n(p)  = clamp(ub(E_n, p) - 1, 0, N-2)
//   unionized u     = clamp(ub(U, p) - 1, 0, NU-2);  IG[u][n] = k_n(U[u])
//   hash b          = min(trunc(p / du), B-1), du = 1/B; HG[b][n] = k_n(b du)
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace xs {

// Energy of record k of the nuclide whose records start at `rec` (6 doubles
// per record: E, total, elastic, absorption, fission, nu-fission).
__device__ __forceinline__ double rec_energy(const double* __restrict__ rec, int64_t k) {
  return __ldg(rec + k * 6);
}

// lo in [lo0, hi0-1] with A[lo] <= q < A[lo+1] when A[lo0] <= q < A[hi0];
// the XSBench grid_search loop shape on a strided energy column.
__device__ __forceinline__ int64_t bracket_search_rec(const double* __restrict__ rec, int64_t lo,
                                                      int64_t hi, double q) {
  int64_t len = hi - lo;
  while (len > 1) {
    int64_t mid = lo + (len >> 1);
    if (rec_energy(rec, mid) > q)
      hi = mid;
    else
      lo = mid;
    len = hi - lo;
  }
  return lo;
}

// k_n(p) with a plain binary search over the nuclide's N energies.
__device__ __forceinline__ int32_t nuclide_bracket(const double* __restrict__ rec, int64_t N,
                                                   double p) {
  // ub - 1 clamped to [0, N-2]: search on [0, N-1] gives exactly that
  return static_cast<int32_t>(bracket_search_rec(rec, 0, N - 1, p));
}

// u = clamp(ub(U, p) - 1, 0, NU-2): the same loop on the contiguous U.
__device__ __forceinline__ int64_t union_search(const double* __restrict__ U, int64_t NU,
                                                double p) {
  int64_t lo = 0, hi = NU - 1, len = hi;
  while (len > 1) {
    int64_t mid = lo + (len >> 1);
    if (__ldg(U + mid) > p)
      hi = mid;
    else
      lo = mid;
    len = hi - lo;
  }
  return lo;
}

__device__ __forceinline__ int32_t hash_bin(double p, double du, int32_t B) {
  // trunc toward zero, as a C cast; p < 0 (explicit lookups) -> bin 0
  double q = p / du;
  if (!(q > 0.0)) return 0;
  if (q >= static_cast<double>(B)) return B - 1;
  int32_t b = static_cast<int32_t>(q);
  return b > B - 1 ? B - 1 : b;
}

// XSBench's bracketed hash search (R7), result = k_n(p).
__device__ __forceinline__ int32_t hash_bracket(const int32_t* __restrict__ HG, int32_t I,
                                                int32_t B, int32_t b, int32_t n,
                                                const double* __restrict__ rec, int64_t N,
                                                double p) {
  const int64_t u_lo = __ldg(HG + static_cast<int64_t>(b) * I + n);
  const int64_t u_hi =
      (b == B - 1) ? N - 1 : static_cast<int64_t>(__ldg(HG + static_cast<int64_t>(b + 1) * I + n)) + 1;
  int64_t lower;
  if (p <= rec_energy(rec, u_lo))
    lower = u_lo;
  else if (p >= rec_energy(rec, u_hi))
    lower = N - 1;
  else
    lower = bracket_search_rec(rec, u_lo, u_hi, p);
  return static_cast<int32_t>(lower == N - 1 ? N - 2 : lower);
}

}  // namespace xs
