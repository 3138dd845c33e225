// xs_gen.cpp — seeded synthetic input generator; see xs_gen.h for the contract.
// Input data only: nothing in here is part of the lookup method.
#include "xs_gen.h"

#include <algorithm>
#include <cstring>
#include <thread>
#include <vector>

namespace {

constexpr uint64_t kA = 2806196910506780709ULL;
constexpr uint64_t kC = 1ULL;
constexpr uint64_t kMask63 = (1ULL << 63) - 1ULL;

inline double draw(uint64_t* s) {
  *s = (kA * *s + kC) & kMask63;
  return static_cast<double>(*s) / 9223372036854775808.0;
}

// Jump the generator's stream by n draws (affine-map power; used only so
// that threads can start mid-stream — the resulting sequence is the same as
// drawing serially).
uint64_t jump(uint64_t s, uint64_t n) {
  uint64_t a = kA, c = kC, A = 1, C = 0;
  while (n) {
    if (n & 1) { A = A * a; C = C * a + c; }
    c = c * (a + 1);
    a = a * a;
    n >>= 1;
  }
  return (A * s + C) & kMask63;
}

// XSBench H-M material compositions (public XSBench v20 tables; R1).
const int32_t kFuelSmall[34] = {58, 59, 60, 61, 40, 42, 43, 44, 45, 46, 1,  2,  3,  7,  8,  9,  10,
                                29, 57, 47, 48, 0,  62, 15, 33, 34, 52, 53, 54, 55, 56, 18, 23, 41};
const int32_t kMat1[5] = {63, 64, 65, 66, 67};
const int32_t kMat2[4] = {24, 41, 4, 5};
const int32_t kMat4[27] = {19, 20, 21, 22, 35, 36, 37, 38, 39, 25, 27, 28, 29, 30,
                           31, 32, 26, 49, 50, 51, 11, 12, 13, 14, 6,  16, 17};
const int32_t kMat5[21] = {24, 41, 4,  5,  19, 20, 21, 22, 35, 36, 37,
                           38, 39, 25, 49, 50, 51, 11, 12, 13, 14};
const int32_t kMat10[9] = {24, 41, 4, 5, 63, 64, 65, 66, 67};

// The 12 material id lists for rule 0 with I in {68, 355}; `large` picks the
// 321-nuclide fuel (small list followed by 68..354).
std::vector<std::vector<int32_t>> hm_tables(bool large) {
  std::vector<std::vector<int32_t>> m(XSGEN_N_MATS);
  m[0].assign(kFuelSmall, kFuelSmall + 34);
  if (large)
    for (int32_t i = 0; i < 321 - 34; ++i) m[0].push_back(68 + i);
  m[1].assign(kMat1, kMat1 + 5);
  m[2].assign(kMat2, kMat2 + 4);
  m[3].assign(kMat2, kMat2 + 4);
  m[4].assign(kMat4, kMat4 + 27);
  for (int k = 5; k <= 9; ++k) m[k].assign(kMat5, kMat5 + 21);
  m[10].assign(kMat10, kMat10 + 9);
  m[11].assign(kMat10, kMat10 + 9);
  return m;
}

bool tables(int32_t I, int32_t rule, std::vector<std::vector<int32_t>>* out) {
  if (I < 1) return false;
  if (rule == 0) {
    if (I != 68 && I != 355) return false;
    *out = hm_tables(I == 355);
    return true;
  }
  if (rule == 1) {
    auto big = hm_tables(true);
    out->assign(XSGEN_N_MATS, {});
    for (int m = 0; m < XSGEN_N_MATS; ++m) {
      for (int32_t id : big[m]) {
        int32_t r = id % I;
        if (std::find((*out)[m].begin(), (*out)[m].end(), r) == (*out)[m].end())
          (*out)[m].push_back(r);
      }
    }
    return true;
  }
  return false;
}

struct Rec {
  double v[6];
};

}  // namespace

extern "C" int xsgen_num_nucs(int32_t I, int32_t rule, int32_t num_nucs[XSGEN_N_MATS]) {
  std::vector<std::vector<int32_t>> t;
  if (!tables(I, rule, &t) || !num_nucs) return XSGEN_ERR_INVALID_ARG;
  for (int m = 0; m < XSGEN_N_MATS; ++m) num_nucs[m] = static_cast<int32_t>(t[m].size());
  return XSGEN_OK;
}

extern "C" int32_t xsgen_max_num_nucs(int32_t I, int32_t rule) {
  std::vector<std::vector<int32_t>> t;
  if (!tables(I, rule, &t)) return -1;
  size_t mx = 0;
  for (auto& r : t) mx = std::max(mx, r.size());
  return static_cast<int32_t>(mx);
}

extern "C" int xsgen_mats(int32_t I, int32_t rule, int32_t max_num_nucs, int32_t* mats) {
  std::vector<std::vector<int32_t>> t;
  if (!tables(I, rule, &t) || !mats) return XSGEN_ERR_INVALID_ARG;
  for (auto& r : t)
    if (static_cast<int32_t>(r.size()) > max_num_nucs) return XSGEN_ERR_INVALID_ARG;
  for (int m = 0; m < XSGEN_N_MATS; ++m)
    for (int32_t j = 0; j < max_num_nucs; ++j)
      mats[m * max_num_nucs + j] = j < static_cast<int32_t>(t[m].size()) ? t[m][j] : -1;
  return XSGEN_OK;
}

extern "C" int xsgen_concs(uint64_t conc_seed, const int32_t num_nucs[XSGEN_N_MATS],
                           int32_t max_num_nucs, double* concs) {
  if (!num_nucs || !concs || max_num_nucs < 1) return XSGEN_ERR_INVALID_ARG;
  uint64_t s = conc_seed;
  for (int m = 0; m < XSGEN_N_MATS; ++m) {
    if (num_nucs[m] > max_num_nucs || num_nucs[m] < 0) return XSGEN_ERR_INVALID_ARG;
    for (int32_t j = 0; j < max_num_nucs; ++j)
      concs[m * max_num_nucs + j] = j < num_nucs[m] ? draw(&s) : 0.0;
  }
  return XSGEN_OK;
}

extern "C" int xsgen_nuclide_grid(int32_t I, int64_t N, uint64_t grid_seed, double* grid,
                                  int nthreads) {
  if (I < 1 || N < 2 || !grid) return XSGEN_ERR_INVALID_ARG;
  if (nthreads <= 0) nthreads = static_cast<int>(std::max(1u, std::thread::hardware_concurrency()));
  nthreads = std::min<int>(nthreads, I);
  std::vector<int> bad(nthreads, 0);
  auto work = [&](int t) {
    int32_t n0 = static_cast<int32_t>(static_cast<int64_t>(I) * t / nthreads);
    int32_t n1 = static_cast<int32_t>(static_cast<int64_t>(I) * (t + 1) / nthreads);
    uint64_t s = jump(grid_seed, static_cast<uint64_t>(n0) * static_cast<uint64_t>(N) * 6u);
    for (int32_t n = n0; n < n1; ++n) {
      Rec* r = reinterpret_cast<Rec*>(grid + static_cast<int64_t>(n) * N * 6);
      for (int64_t k = 0; k < N; ++k)
        for (int c = 0; c < 6; ++c) r[k].v[c] = draw(&s);
      std::sort(r, r + N, [](const Rec& x, const Rec& y) { return x.v[0] < y.v[0]; });
      for (int64_t k = 1; k < N; ++k)
        if (!(r[k - 1].v[0] < r[k].v[0])) bad[t] = 1;
    }
  };
  std::vector<std::thread> th;
  for (int t = 1; t < nthreads; ++t) th.emplace_back(work, t);
  work(0);
  for (auto& x : th) x.join();
  for (int b : bad)
    if (b) return XSGEN_ERR_DUP_ENERGY;
  return XSGEN_OK;
}
