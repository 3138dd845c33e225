// rs_gen.cpp — seeded RSBench input generator; see rs_gen.h for the contract.
// Input data only: nothing in here is part of the lookup method.
#include "rs_gen.h"

#include <algorithm>
#include <vector>

#include "xs_gen.h"

namespace {

constexpr uint64_t kA = 2806196910506780709ULL;
constexpr uint64_t kC = 1ULL;
constexpr uint64_t kMask63 = (1ULL << 63) - 1ULL;

inline uint64_t next_int(uint64_t* s) {
  *s = (kA * *s + kC) & kMask63;
  return *s;
}
inline double draw(uint64_t* s) { return static_cast<double>(next_int(s)) / 9223372036854775808.0; }

bool valid(const rsgen_spec* sp) {
  return sp && sp->n_nuclides >= 1 && sp->avg_n_poles >= 1 && sp->avg_n_windows >= 1 &&
         sp->numL >= 1 && xsgen_max_num_nucs(sp->n_nuclides, sp->material_rule) > 0;
}

// Runs the stream through concs (optional), n_poles and n_windows.
int counts(const rsgen_spec* sp, uint64_t* s, int32_t max_num_nucs, double* concs,
           int32_t* np, int32_t* nw) {
  int32_t num_nucs[XSGEN_N_MATS];
  if (xsgen_num_nucs(sp->n_nuclides, sp->material_rule, num_nucs) != XSGEN_OK)
    return RSGEN_ERR_INVALID_ARG;
  for (int m = 0; m < XSGEN_N_MATS; ++m)
    for (int32_t j = 0; j < num_nucs[m]; ++j) {
      double c = draw(s);
      if (concs) concs[m * max_num_nucs + j] = c;
    }
  const int64_t I = sp->n_nuclides;
  for (int pass = 0; pass < 2; ++pass) {
    int32_t* R = pass == 0 ? np : nw;
    const int64_t avg = pass == 0 ? sp->avg_n_poles : sp->avg_n_windows;
    for (int64_t i = 0; i < I; ++i) R[i] = 1;
    for (int64_t k = 0; k < avg * I - I; ++k) R[next_int(s) % static_cast<uint64_t>(I)]++;
  }
  return RSGEN_OK;
}

}  // namespace

extern "C" int rsgen_counts(const rsgen_spec* sp, int32_t* np, int32_t* nw, int32_t* max_p,
                            int32_t* max_w) {
  if (!valid(sp) || !np || !nw || !max_p || !max_w) return RSGEN_ERR_INVALID_ARG;
  uint64_t s = sp->seed;
  int rc = counts(sp, &s, 0, nullptr, np, nw);
  if (rc) return rc;
  *max_p = *std::max_element(np, np + sp->n_nuclides);
  *max_w = *std::max_element(nw, nw + sp->n_nuclides);
  return RSGEN_OK;
}

extern "C" int rsgen_data(const rsgen_spec* sp, int32_t max_num_nucs, int32_t max_p,
                          int32_t max_w, double* concs, int32_t* np, int32_t* nw, double* poles,
                          int32_t* l_value, double* windows, int32_t* wrange, double* k0rs) {
  if (!valid(sp) || !concs || !np || !nw || !poles || !l_value || !windows || !wrange || !k0rs)
    return RSGEN_ERR_INVALID_ARG;
  if (max_num_nucs < xsgen_max_num_nucs(sp->n_nuclides, sp->material_rule))
    return RSGEN_ERR_INVALID_ARG;
  const int64_t I = sp->n_nuclides;
  std::fill(concs, concs + XSGEN_N_MATS * static_cast<int64_t>(max_num_nucs), 0.0);
  uint64_t s = sp->seed;
  int rc = counts(sp, &s, max_num_nucs, concs, np, nw);
  if (rc) return rc;
  for (int64_t n = 0; n < I; ++n)
    if (np[n] > max_p || nw[n] > max_w) return RSGEN_ERR_INVALID_ARG;
  std::fill(poles, poles + I * max_p * 8, 0.0);
  std::fill(l_value, l_value + I * max_p, 0);
  std::fill(windows, windows + I * max_w * 3, 0.0);
  std::fill(wrange, wrange + I * max_w * 2, 0);
  for (int64_t n = 0; n < I; ++n)
    for (int64_t j = 0; j < np[n]; ++j) {
      double* p = poles + (n * max_p + j) * 8;
      for (int c = 0; c < 8; ++c) p[c] = draw(&s);
      l_value[n * max_p + j] = static_cast<int32_t>(next_int(&s) % static_cast<uint64_t>(sp->numL));
    }
  for (int64_t n = 0; n < I; ++n) {
    const int32_t space = np[n] / nw[n];
    const int32_t rem = np[n] - space * nw[n];
    int32_t ctr = 0;
    for (int32_t w = 0; w < nw[n]; ++w) {
      double* t = windows + (n * max_w + w) * 3;
      for (int c = 0; c < 3; ++c) t[c] = draw(&s);
      int32_t* r = wrange + (n * max_w + w) * 2;
      r[0] = ctr;
      r[1] = ctr + space - 1;
      ctr += space;
      if (w < rem) {
        ctr++;
        r[1]++;
      }
    }
  }
  for (int64_t n = 0; n < I; ++n)
    for (int l = 0; l < sp->numL; ++l) k0rs[n * sp->numL + l] = draw(&s);
  return RSGEN_OK;
}
