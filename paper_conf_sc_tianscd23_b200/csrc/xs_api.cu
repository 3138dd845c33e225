// xs_api.cu — the C-ABI (include/xs.h): argument checking, ownership,
// device selection, workspace layout and staging.  All compute is in
// grid_build.cu / lookup.cu; there is no host compute path and no fallback.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <array>
#include <cstdio>
#include <cstring>
#include <memory>
#include <new>
#include <string>
#include <thread>
#include <vector>

#include "../../gen/xs_gen.h"
#include "common.cuh"
#include "radix_sort.cuh"
#include "xs_internal.h"

struct xs_grid {
  xs::DeviceGrid d;
  // chunked host-input pipeline (XS_FLAG_HOST_IO)
  uint64_t host_chunk = 10000000;  // host-input chunk (lookups), measured on B200 (large)
  cudaStream_t copy_stream = nullptr;
  std::vector<cudaEvent_t> chunk_ev;
  // XS_FLAG_HOST_ASYNC: per workspace, the event after the last call that used it
  std::vector<std::pair<const void*, cudaEvent_t>> ws_done;
  // per-phase event timing (xs_timing_enable / xs_timing_read)
  bool timing = false;
  std::vector<std::array<cudaEvent_t, 4>> ev;
  size_t ev_used = 0;
  uint64_t calls = 0;
  uint64_t launches_read = 0;
};

namespace xs {

static thread_local std::string g_err;

static xs_status fail(xs_status code, const std::string& msg, cudaError_t ce = cudaSuccess) {
  g_err = msg;
  if (ce != cudaSuccess) {
    g_err += ": ";
    g_err += cudaGetErrorName(ce);
    g_err += " (";
    g_err += cudaGetErrorString(ce);
    g_err += ")";
    if (ce == cudaErrorMemoryAllocation) code = XS_ERR_OUT_OF_MEMORY;
    cudaGetLastError();  // clear sticky-free errors
  }
  return code;
}

xs_status report_error(xs_status code, const char* msg, cudaError_t ce) {
  return fail(code, msg, ce);
}

#define XS_TRY(expr, what)                                   \
  do {                                                       \
    cudaError_t _e = (expr);                                 \
    if (_e != cudaSuccess) return fail(XS_ERR_CUDA, what, _e); \
  } while (0)

// Switch to the grid's device for the duration of a call.
struct DeviceGuard {
  int prev = -1;
  bool ok = false;
  explicit DeviceGuard(int dev) {
    if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
    ok = cudaSetDevice(dev) == cudaSuccess;
  }
  ~DeviceGuard() {
    if (prev >= 0) cudaSetDevice(prev);
  }
};

static size_t align256(size_t x) { return (x + 255) & ~static_cast<size_t>(255); }

size_t workspace_layout(uint64_t count, uint32_t flags, int32_t n_mats, void* base,
                        Workspace* ws) {
  size_t off = 0;
  auto take = [&](size_t bytes) {
    size_t o = off;
    off += align256(bytes);
    return o;
  };
  const size_t o_counts = take((2 * (kMaxMats + 1) + 2) * sizeof(uint32_t));
  const size_t o_recs = take(count * sizeof(LookupRec));
  const size_t o_tmp = take(count * sizeof(LookupRec));
  const size_t o_mat8 = take(count);
  size_t o_bins = 0, o_part = 0, o_perm = 0, bins_bytes = 0;
  if (flags & XS_FLAG_SORT) {
    o_perm = take(count * 4);
    // the bin area serves both A2 forms: the global-atomic bins and the
    // partitioned A2's tile histograms (whichever is larger for this count)
    bins_bytes = std::max(static_cast<size_t>(n_mats + 1) * kEnergyBins * 4,
                          part_bins_bytes(count, n_mats));
    o_bins = take(bins_bytes);
    o_part = take(static_cast<size_t>(n_mats + 1) * (kEnergyBins / 4096) * 4);
  }
  if (ws) {
    char* b = static_cast<char*>(base);
    ws->counts = reinterpret_cast<uint32_t*>(b + o_counts);
    ws->cursor = ws->counts + (kMaxMats + 1);
    ws->gate = ws->counts + 2 * (kMaxMats + 1) + 1;  // after the task counter
    ws->recs = reinterpret_cast<LookupRec*>(b + o_recs);
    ws->bins = reinterpret_cast<uint32_t*>(b + o_bins);
    ws->partials = reinterpret_cast<uint32_t*>(b + o_part);
    ws->perm = reinterpret_cast<uint32_t*>(b + o_perm);
    ws->tmp = reinterpret_cast<LookupRec*>(b + o_tmp);
    ws->mat8 = reinterpret_cast<uint8_t*>(b + o_mat8);
    ws->bins_bytes = bins_bytes;
    ws->total = off;
  }
  return off;
}

// staging area for XS_FLAG_HOST_IO (after the compute workspace)
struct Staging {
  double* energy;
  int32_t* mat;
  double* M;
  double* E;
  int32_t* omat;
  int64_t* gidx;
  int32_t* v;
  uint64_t* vsum;
};

static size_t staging_layout(uint64_t count, void* base, Staging* s) {
  size_t off = 0;
  auto take = [&](size_t bytes) {
    size_t o = off;
    off += align256(bytes);
    return o;
  };
  const size_t o_e = take(count * 8), o_m = take(count * 4), o_M = take(count * 40),
               o_E = take(count * 8), o_om = take(count * 4), o_g = take(count * 8),
               o_v = take(count * 4), o_s = take(16);
  if (s) {
    char* b = static_cast<char*>(base);
    s->energy = reinterpret_cast<double*>(b + o_e);
    s->mat = reinterpret_cast<int32_t*>(b + o_m);
    s->M = reinterpret_cast<double*>(b + o_M);
    s->E = reinterpret_cast<double*>(b + o_E);
    s->omat = reinterpret_cast<int32_t*>(b + o_om);
    s->gidx = reinterpret_cast<int64_t*>(b + o_g);
    s->v = reinterpret_cast<int32_t*>(b + o_v);
    s->vsum = reinterpret_cast<uint64_t*>(b + o_s);
  }
  return off;
}

static size_t total_workspace(uint64_t count, uint32_t flags, int32_t n_mats) {
  size_t w = workspace_layout(count, flags, n_mats, nullptr, nullptr);
  if (flags & (XS_FLAG_HOST_IO | XS_FLAG_HOST_ASYNC)) w += staging_layout(count, nullptr, nullptr);
  return w;
}

static xs_status check_device(int device, int* sm_count) {
  int n = 0;
  cudaError_t e = cudaGetDeviceCount(&n);
  if (e != cudaSuccess || n == 0) return fail(XS_ERR_CUDA, "no CUDA device available", e);
  if (device < 0 || device >= n) return fail(XS_ERR_INVALID_ARG, "device index out of range");
  cudaDeviceProp prop;
  XS_TRY(cudaGetDeviceProperties(&prop, device), "cudaGetDeviceProperties");
  if (prop.major != 10)
    return fail(XS_ERR_UNSUPPORTED, "libxs is built for sm_100a (B200); device is sm_" +
                                        std::to_string(prop.major * 10 + prop.minor));
  *sm_count = prop.multiProcessorCount;
  return XS_OK;
}

static xs_status init_common(const xs_grid_data* d, int device, cudaStream_t st, xs_grid** out) {
  const int32_t I = d->n_isotopes;
  const int64_t N = d->n_gridpoints;
  if (I < 1 || N < 2 || !d->nuclide_grid || d->n_mats < 1 || d->max_num_nucs < 1 ||
      !d->num_nucs || !d->mats || !d->concs)
    return fail(XS_ERR_INVALID_ARG, "xs_grid_data: missing array or bad size");
  if (N > 0x7fffffffLL || static_cast<int64_t>(I) * N >= 0x7fffffffLL)
    return fail(XS_ERR_UNSUPPORTED, "I*N must be < 2^31 (32-bit grid indices)");
  if (d->n_mats > kMaxMats)
    return fail(XS_ERR_UNSUPPORTED, "more than 64 materials");
  if (d->grid_type < 0 || d->grid_type > 2) return fail(XS_ERR_INVALID_ARG, "bad grid_type");
  if (d->grid_type == XS_GRID_HASH && d->hash_bins < 1)
    return fail(XS_ERR_INVALID_ARG, "hash grid needs hash_bins >= 1");
  const size_t tab = static_cast<size_t>(d->n_mats) * d->max_num_nucs;
  if (tab * 16 > 160 * 1024)
    return fail(XS_ERR_UNSUPPORTED, "material tables exceed the 160 KB shared-memory stage");
  for (int32_t m = 0; m < d->n_mats; ++m) {
    if (d->num_nucs[m] < 0 || d->num_nucs[m] > d->max_num_nucs)
      return fail(XS_ERR_INVALID_ARG, "num_nucs out of range");
    for (int32_t j = 0; j < d->num_nucs[m]; ++j) {
      const int32_t n = d->mats[static_cast<size_t>(m) * d->max_num_nucs + j];
      if (n < 0 || n >= I) return fail(XS_ERR_INVALID_ARG, "mats: nuclide id out of range");
    }
  }
  for (int32_t n = 0; n < I; ++n) {
    const double* E = d->nuclide_grid + static_cast<size_t>(n) * N * 6;
    if (d->grid_type == XS_GRID_HASH && !(E[0] >= 0.0))
      return fail(XS_ERR_INVALID_ARG, "hash grid needs non-negative energies");
    for (int64_t k = 1; k < N; ++k)
      if (!(E[(k - 1) * 6] < E[k * 6]))
        return fail(XS_ERR_DATA, "nuclide " + std::to_string(n) +
                                     ": energies not strictly increasing");
  }
  // energies on the 2^-63 lattice of [0, 1] (all generated grids): lets the
  // gather kernel skip the division range check for sampled lookups
  bool dyadic = true;
  for (int64_t i = 0; i < static_cast<int64_t>(I) * N && dyadic; ++i) {
    const double e = d->nuclide_grid[i * 6];
    const double k = e * 0x1p63;  // exact scaling by a power of two
    dyadic = e >= 0.0 && e <= 1.0 && k == static_cast<double>(static_cast<uint64_t>(k));
  }
  int sm = 0;
  xs_status s = check_device(device, &sm);
  if (s != XS_OK) return s;
  DeviceGuard guard(device);
  if (!guard.ok) return fail(XS_ERR_CUDA, "cudaSetDevice failed");
  XS_TRY(init_constants(), "init_constants");

  std::unique_ptr<xs_grid> g(new (std::nothrow) xs_grid());
  if (!g) return fail(XS_ERR_OUT_OF_MEMORY, "host allocation");
  DeviceGrid& G = g->d;
  G.device = device;
  G.sm_count = sm;
  G.I = I;
  G.N = N;
  G.n_mats = d->n_mats;
  G.max_nucs = d->max_num_nucs;
  for (int32_t m = 0; m < d->n_mats; ++m) G.tab_total += d->num_nucs[m];
  G.grid_type = d->grid_type;
  G.B = d->grid_type == XS_GRID_HASH ? d->hash_bins : 0;
  G.du = G.B ? 1.0 / static_cast<double>(G.B) : 0.0;
  G.lookup_seed = d->lookup_seed;
  G.dyadic63 = dyadic;
  G.NU = d->grid_type == XS_GRID_UNIONIZED ? static_cast<int64_t>(I) * N : 0;
  if (d->index_layout < 0 || d->index_layout > 3)
    return fail(XS_ERR_INVALID_ARG, "index_layout must be XS_INDEX_AUTO/ROW/COL/BOTH");
  if (G.NU) {
    int lay = d->index_layout;
    if (lay == XS_INDEX_AUTO) {
      size_t free_b = 0, total_b = 0;
      cudaMemGetInfo(&free_b, &total_b);
      const double one = static_cast<double>(G.NU) * I * 4.0;
      lay = (2.0 * one <= 0.45 * static_cast<double>(free_b)) ? XS_INDEX_BOTH : XS_INDEX_COL;
    }
    G.index_layout = lay;
  } else {
    G.index_layout = d->grid_type == XS_GRID_HASH ? XS_INDEX_ROW : 0;
  }
  G.index_len = d->grid_type == XS_GRID_UNIONIZED ? G.NU * I
                : d->grid_type == XS_GRID_HASH    ? static_cast<int64_t>(G.B) * I
                                                  : 0;
  if (G.NU) {  // ~8 unionized energies per search-table bin
    G.UBn = 1024;
    while (G.UBn < (1 << 23) && static_cast<int64_t>(G.UBn) * 8 < G.NU) G.UBn <<= 1;
  }
  auto cleanup = [&]() {
    cudaFree(G.grid);
    cudaFree(G.iv);
    cudaFree(G.iv32);
    cudaFree(G.ivu);
    cudaFree(G.U);
    cudaFree(G.UB);
    cudaFree(G.index);
    cudaFree(G.index_t);
    cudaFree(G.num_nucs);
    cudaFree(G.mats);
    cudaFree(G.concs);
  };
  const size_t grid_bytes = static_cast<size_t>(I) * N * 6 * sizeof(double);
  // one padding record after the last nuclide: the windowed gather reads
  // records k..k+2 with k <= N-2 (the padding is never interpolated)
  cudaError_t e = cudaMalloc(&G.grid, grid_bytes + 6 * sizeof(double));
  if (e == cudaSuccess) e = cudaMemsetAsync(reinterpret_cast<char*>(G.grid) + grid_bytes, 0,
                                            6 * sizeof(double), st);
  const size_t iv_bytes = static_cast<size_t>(I) * N * kIvDoubles * sizeof(double);
  if (e == cudaSuccess) e = cudaMalloc(&G.iv, iv_bytes);
  const size_t iv32_bytes = static_cast<size_t>(I) * N * kIv32Doubles * sizeof(double);
  if (e == cudaSuccess) e = cudaMalloc(&G.iv32, iv32_bytes);
  if (e == cudaSuccess && G.NU) e = cudaMalloc(&G.U, G.NU * sizeof(double));
  if (e == cudaSuccess && G.NU) e = cudaMalloc(&G.UB, (static_cast<size_t>(G.UBn) + 1) * 4);
  if (e == cudaSuccess && G.index_len && (G.index_layout & XS_INDEX_ROW))
    e = cudaMalloc(&G.index, G.index_len * sizeof(int32_t));
  if (e == cudaSuccess && G.NU && (G.index_layout & XS_INDEX_COL))
    e = cudaMalloc(&G.index_t, G.index_len * sizeof(int32_t));
  if (e == cudaSuccess) e = cudaMalloc(&G.num_nucs, d->n_mats * sizeof(int32_t));
  if (e == cudaSuccess) e = cudaMalloc(&G.mats, tab * sizeof(int32_t));
  if (e == cudaSuccess) e = cudaMalloc(&G.concs, tab * sizeof(double));
  if (e != cudaSuccess) {
    cleanup();
    return fail(XS_ERR_OUT_OF_MEMORY, "device allocation of the grid tables", e);
  }
  // K0u (unsorted gather): optional, only where it leaves ample memory free
  // (large: 385 MB; XL: 8.1 GB); without it unsorted batches use k_gather.
  // A unionized grid without the row layout (XL) never runs k_gather_u
  // (its unsorted batches take the staged gather): no K0u
  const size_t ivu_bytes = static_cast<size_t>(I) * N * 12 * sizeof(double);
  const bool ivu_usable = !(G.grid_type == XS_GRID_UNIONIZED && !(G.index_layout & XS_INDEX_ROW));
  if (ivu_usable) {
    size_t free_b = 0, total_b = 0;
    cudaMemGetInfo(&free_b, &total_b);
    if (free_b > ivu_bytes + (static_cast<size_t>(24) << 30) && cudaMalloc(&G.ivu, ivu_bytes) != cudaSuccess) {
      G.ivu = nullptr;
      cudaGetLastError();
    }
  }
  G.device_bytes = grid_bytes + iv_bytes + iv32_bytes + (G.ivu ? ivu_bytes : 0) + G.NU * 8 + (G.NU ? (G.UBn + 1) * 4 : 0) + G.index_len * 4 * (G.index_layout == XS_INDEX_BOTH ? 2 : 1) + d->n_mats * 4 + tab * 12;
  e = cudaMemcpyAsync(G.grid, d->nuclide_grid, grid_bytes, cudaMemcpyHostToDevice, st);
  if (e == cudaSuccess)
    e = cudaMemcpyAsync(G.num_nucs, d->num_nucs, d->n_mats * 4, cudaMemcpyHostToDevice, st);
  if (e == cudaSuccess) e = cudaMemcpyAsync(G.mats, d->mats, tab * 4, cudaMemcpyHostToDevice, st);
  if (e == cudaSuccess) e = cudaMemcpyAsync(G.concs, d->concs, tab * 8, cudaMemcpyHostToDevice, st);
  if (e == cudaSuccess) e = build_intervals(G, st);
  if (e == cudaSuccess) e = build_intervals32(G, st);
  if (e == cudaSuccess && G.ivu) e = build_intervals_u(G, st);
  if (e == cudaSuccess && G.grid_type == XS_GRID_UNIONIZED) {
    e = build_union_grid(G, G.U, st);
    if (e == cudaSuccess) e = build_union_table(G, st);
    if (e == cudaSuccess && G.index) e = build_index_grid(G, st);
    if (e == cudaSuccess && G.index_t) e = build_index_grid_t(G, st);
  }
  if (e == cudaSuccess && G.grid_type == XS_GRID_HASH) e = build_hash_grid(G, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  if (e != cudaSuccess) {
    cleanup();
    return fail(XS_ERR_CUDA, "grid upload / build", e);
  }
  *out = g.release();
  return XS_OK;
}

}  // namespace xs

using namespace xs;

extern "C" {

uint32_t xs_abi_version(void) { return XS_ABI_VERSION; }

const char* xs_last_error(void) { return g_err.c_str(); }

uint64_t xs_hash_finalize(uint64_t global_sum) { return global_sum % 999983ULL; }

xs_status xs_init_grid(const xs_grid_spec* spec, int device, void* cuda_stream, xs_grid** out) {
  if (!spec || !out) return fail(XS_ERR_INVALID_ARG, "NULL spec/out");
  *out = nullptr;
  if (spec->abi_version != XS_ABI_VERSION) return fail(XS_ERR_INVALID_ARG, "abi_version mismatch");

  const int32_t I = spec->n_isotopes;
  const int64_t N = spec->n_gridpoints;
  const int32_t mx = xsgen_max_num_nucs(I, spec->material_rule);
  if (I < 1 || N < 2 || mx < 1)
    return fail(XS_ERR_INVALID_ARG, "bad spec (I, N or material_rule; rule 0 needs I in {68,355})");
  if (static_cast<int64_t>(I) * N >= 0x7fffffffLL)
    return fail(XS_ERR_UNSUPPORTED, "I*N must be < 2^31");
  std::vector<int32_t> num(XSGEN_N_MATS), mats(static_cast<size_t>(XSGEN_N_MATS) * mx);
  std::vector<double> concs(static_cast<size_t>(XSGEN_N_MATS) * mx);
  if (xsgen_num_nucs(I, spec->material_rule, num.data()) ||
      xsgen_mats(I, spec->material_rule, mx, mats.data()) ||
      xsgen_concs(spec->conc_seed, num.data(), mx, concs.data()))
    return fail(XS_ERR_INVALID_ARG, "material generation failed");
  std::unique_ptr<double[]> grid(new (std::nothrow) double[static_cast<size_t>(I) * N * 6]);
  if (!grid) return fail(XS_ERR_OUT_OF_MEMORY, "host grid buffer");
  const int ge = xsgen_nuclide_grid(I, N, spec->grid_seed, grid.get(), 0);
  if (ge == XSGEN_ERR_DUP_ENERGY)
    return fail(XS_ERR_DATA, "generated grid has a duplicate energy within a nuclide (seed)");
  if (ge) return fail(XS_ERR_INVALID_ARG, "grid generation failed");
  xs_grid_data d{};
  d.abi_version = XS_ABI_VERSION;
  d.n_isotopes = I;
  d.n_gridpoints = N;
  d.nuclide_grid = grid.get();
  d.n_mats = XSGEN_N_MATS;
  d.max_num_nucs = mx;
  d.num_nucs = num.data();
  d.mats = mats.data();
  d.concs = concs.data();
  d.grid_type = spec->grid_type;
  d.hash_bins = spec->hash_bins;
  d.lookup_seed = spec->lookup_seed;
  d.index_layout = spec->index_layout;
  return init_common(&d, device, static_cast<cudaStream_t>(cuda_stream), out);
}

xs_status xs_init_grid_data(const xs_grid_data* data, int device, void* cuda_stream,
                            xs_grid** out) {
  if (!data || !out) return fail(XS_ERR_INVALID_ARG, "NULL data/out");
  *out = nullptr;
  if (data->abi_version != XS_ABI_VERSION) return fail(XS_ERR_INVALID_ARG, "abi_version mismatch");
  if (data->reserved0 != 0) return fail(XS_ERR_INVALID_ARG, "reserved0 must be 0");
  return init_common(data, device, static_cast<cudaStream_t>(cuda_stream), out);
}

xs_status xs_grid_get_info(const xs_grid* g, xs_grid_info* info) {
  if (!g || !info) return fail(XS_ERR_INVALID_ARG, "NULL grid/info");
  const DeviceGrid& G = g->d;
  info->n_isotopes = G.I;
  info->n_mats = G.n_mats;
  info->max_num_nucs = G.max_nucs;
  info->grid_type = G.grid_type;
  info->hash_bins = G.B;
  info->device = G.device;
  info->n_gridpoints = G.N;
  info->n_union = G.NU;
  info->index_grid_len = G.index_len;
  info->device_bytes = G.device_bytes;
  info->lookup_seed = G.lookup_seed;
  info->index_layout = G.index_layout;
  info->reserved0 = 0;
  return XS_OK;
}

xs_status xs_workspace_size(const xs_grid* g, uint64_t count, uint32_t flags, size_t* bytes) {
  if (!g || !bytes) return fail(XS_ERR_INVALID_ARG, "NULL grid/bytes");
  if (count >= (1ULL << 32)) return fail(XS_ERR_INVALID_ARG, "count must be < 2^32");
  *bytes = total_workspace(count, flags, g->d.n_mats);
  return XS_OK;
}

struct ShardSel {
  bool on = false;
  double e_lo = 0.0, e_hi = 0.0;
};

static xs_status lookup_common(xs_grid* g, uint64_t first_id, const double* energy,
                               const int32_t* mat, uint64_t count, uint32_t flags,
                               const xs_outputs* out, void* workspace, size_t ws_bytes,
                               void* cuda_stream, ShardSel shard = ShardSel()) {
  if (!g || !out) return fail(XS_ERR_INVALID_ARG, "NULL grid/outputs");
  if (!out->vsum) return fail(XS_ERR_INVALID_ARG, "outputs.vsum is required");
  if (count >= (1ULL << 32)) return fail(XS_ERR_INVALID_ARG, "count must be < 2^32");
  if (flags & ~(XS_FLAG_SORT | XS_FLAG_HOST_IO | XS_FLAG_BASELINE | XS_FLAG_F32 | XS_FLAG_MAT_U8 |
                XS_FLAG_HOST_ASYNC))
    return fail(XS_ERR_INVALID_ARG, "unknown flag bits");
  if ((flags & XS_FLAG_HOST_ASYNC) && (flags & XS_FLAG_HOST_IO))
    return fail(XS_ERR_INVALID_ARG, "XS_FLAG_HOST_ASYNC and XS_FLAG_HOST_IO are exclusive");
  const bool async_io = (flags & XS_FLAG_HOST_ASYNC) != 0;
  if (async_io) flags = (flags & ~XS_FLAG_HOST_ASYNC) | XS_FLAG_HOST_IO;  // same staging
  if ((flags & XS_FLAG_MAT_U8) && !energy)
    return fail(XS_ERR_INVALID_ARG, "XS_FLAG_MAT_U8 applies to explicit lookups only");
  const bool mat8 = (flags & XS_FLAG_MAT_U8) != 0;
  const size_t mat_es = mat8 ? 1 : 4;  // bytes per material id
  if ((flags & XS_FLAG_F32) && (flags & XS_FLAG_BASELINE))
    return fail(XS_ERR_UNSUPPORTED, "XS_FLAG_F32 cannot be combined with XS_FLAG_BASELINE");
  if (count == 0) return XS_OK;
  const size_t need = total_workspace(count, flags, g->d.n_mats);
  if (!workspace || ws_bytes < need)
    return fail(XS_ERR_INVALID_ARG, "workspace too small: need " + std::to_string(need) + " bytes");
  if (reinterpret_cast<uintptr_t>(workspace) & 255)
    return fail(XS_ERR_INVALID_ARG, "workspace must be 256-byte aligned");
  DeviceGuard guard(g->d.device);
  if (!guard.ok) return fail(XS_ERR_CUDA, "cudaSetDevice failed");
  cudaStream_t st = static_cast<cudaStream_t>(cuda_stream);
  Workspace ws;
  const size_t wbytes = workspace_layout(count, flags, g->d.n_mats, workspace, &ws);
  LookupArgs a;
  a.first_id = first_id;
  a.count = static_cast<uint32_t>(count);
  a.flags = flags;
  a.in_energy = energy;
  a.in_mat = mat8 ? nullptr : mat;
  a.in_mat8 = mat8 ? reinterpret_cast<const uint8_t*>(mat) : nullptr;
  a.out = *out;
  a.launches = &g->d.launches;
  a.shard = shard.on;
  a.e_lo = shard.e_lo;
  a.e_hi = shard.e_hi;
  if (g->timing) {
    if (g->ev_used == g->ev.size()) {
      std::array<cudaEvent_t, 4> evs{};
      for (auto& x : evs) XS_TRY(cudaEventCreate(&x), "cudaEventCreate");
      g->ev.push_back(evs);
    }
    a.ev = g->ev[g->ev_used++].data();
  }
  ++g->calls;
  Staging sg{};
  const bool host_io = flags & XS_FLAG_HOST_IO;
  // host inputs larger than one chunk are uploaded chunk by chunk on a copy
  // stream while the previous chunk is being looked up (each chunk is a
  // batch of its own: same results, lookups never interact)
  // equal chunks of at most host_chunk lookups
  const uint64_t nch = (count + g->host_chunk - 1) / g->host_chunk;
  const uint64_t chunk = (count + nch - 1) / nch;
  const bool chunked = host_io && energy && nch > 1 && !async_io;
  cudaEvent_t ws_ev = nullptr;  // async: completion of the last call on this workspace
  if (async_io) {
    for (auto& pr : g->ws_done)
      if (pr.first == workspace) ws_ev = pr.second;
    if (!ws_ev) {
      XS_TRY(cudaEventCreateWithFlags(&ws_ev, cudaEventDisableTiming), "cudaEventCreate");
      g->ws_done.emplace_back(workspace, ws_ev);
      XS_TRY(cudaEventRecord(ws_ev, st), "event");
    }
    if (!g->copy_stream)
      XS_TRY(cudaStreamCreateWithFlags(&g->copy_stream, cudaStreamNonBlocking), "copy stream");
    if (g->chunk_ev.empty()) {
      cudaEvent_t ev;
      XS_TRY(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming), "cudaEventCreate");
      g->chunk_ev.push_back(ev);
    }
  }
  if (host_io) {
    staging_layout(count, static_cast<char*>(workspace) + wbytes, &sg);
    if (energy && async_io) {
      // upload on the copy stream once the workspace's previous call is done,
      // overlapping whatever the caller's stream is still running
      XS_TRY(cudaStreamWaitEvent(g->copy_stream, ws_ev, 0), "wait");
      XS_TRY(cudaMemcpyAsync(sg.energy, energy, count * 8, cudaMemcpyHostToDevice, g->copy_stream),
             "H2D energy");
      XS_TRY(cudaMemcpyAsync(sg.mat, mat, count * mat_es, cudaMemcpyHostToDevice, g->copy_stream),
             "H2D mat");
      XS_TRY(cudaEventRecord(g->chunk_ev[0], g->copy_stream), "event");
      XS_TRY(cudaStreamWaitEvent(st, g->chunk_ev[0], 0), "wait");
    } else if (energy && !chunked) {
      XS_TRY(cudaMemcpyAsync(sg.energy, energy, count * 8, cudaMemcpyHostToDevice, st), "H2D energy");
      XS_TRY(cudaMemcpyAsync(sg.mat, mat, count * mat_es, cudaMemcpyHostToDevice, st), "H2D mat");
    }
    if (energy) {
      a.in_energy = sg.energy;
      a.in_mat = mat8 ? nullptr : sg.mat;
      a.in_mat8 = mat8 ? reinterpret_cast<const uint8_t*>(sg.mat) : nullptr;
    }
    XS_TRY(cudaMemcpyAsync(sg.vsum, out->vsum, 16, cudaMemcpyHostToDevice, st), "H2D vsum");
    a.out.vsum = sg.vsum;
    a.out.macro_xs = out->macro_xs ? sg.M : nullptr;
    a.out.energy = out->energy ? sg.E : nullptr;
    a.out.mat = out->mat ? sg.omat : nullptr;
    a.out.grid_index = out->grid_index ? sg.gidx : nullptr;
    a.out.verification = out->verification ? sg.v : nullptr;
  }
  cudaError_t e = cudaSuccess;
  if (!chunked) {
    e = run_lookup(g->d, a, ws, st);
  } else {
    if (!g->copy_stream)
      XS_TRY(cudaStreamCreateWithFlags(&g->copy_stream, cudaStreamNonBlocking), "copy stream");
    const uint64_t nchunks = (count + chunk - 1) / chunk;
    while (g->chunk_ev.size() < nchunks + 1) {
      cudaEvent_t ev;
      XS_TRY(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming), "cudaEventCreate");
      g->chunk_ev.push_back(ev);
    }
    // the copies may only start once earlier work on the caller's stream is done
    XS_TRY(cudaEventRecord(g->chunk_ev[nchunks], st), "event");
    XS_TRY(cudaStreamWaitEvent(g->copy_stream, g->chunk_ev[nchunks], 0), "wait");
    for (uint64_t k = 0; k < nchunks; ++k) {
      const uint64_t b = k * chunk, n = std::min(chunk, count - b);
      XS_TRY(cudaMemcpyAsync(sg.energy + b, energy + b, n * 8, cudaMemcpyHostToDevice,
                             g->copy_stream), "H2D energy");
      XS_TRY(cudaMemcpyAsync(reinterpret_cast<char*>(sg.mat) + b * mat_es,
                             reinterpret_cast<const char*>(mat) + b * mat_es, n * mat_es,
                             cudaMemcpyHostToDevice, g->copy_stream),
             "H2D mat");
      XS_TRY(cudaEventRecord(g->chunk_ev[k], g->copy_stream), "event");
    }
    LookupArgs c = a;
    c.ev = nullptr;  // phase timing covers whole, unchunked batches only
    for (uint64_t k = 0; k < nchunks && e == cudaSuccess; ++k) {
      const uint64_t b = k * chunk, n = std::min(chunk, count - b);
      XS_TRY(cudaStreamWaitEvent(st, g->chunk_ev[k], 0), "wait");
      c.count = static_cast<uint32_t>(n);
      c.in_energy = sg.energy + b;
      c.in_mat = mat8 ? nullptr : sg.mat + b;
      c.in_mat8 = mat8 ? reinterpret_cast<const uint8_t*>(sg.mat) + b : nullptr;
      c.out.macro_xs = a.out.macro_xs ? a.out.macro_xs + b * 5 : nullptr;
      c.out.energy = a.out.energy ? a.out.energy + b : nullptr;
      c.out.mat = a.out.mat ? a.out.mat + b : nullptr;
      c.out.grid_index = a.out.grid_index ? a.out.grid_index + b : nullptr;
      c.out.verification = a.out.verification ? a.out.verification + b : nullptr;
      e = run_lookup(g->d, c, ws, st);
    }
  }
  if (e == cudaErrorNotSupported && shard.on)
    return fail(XS_ERR_UNSUPPORTED, "energy-range shards need the partitioned A2 (XS_FLAG_SORT, "
                                    "staged gather variant, batch <= 268M lookups)");
  if (e != cudaSuccess) return fail(XS_ERR_CUDA, "lookup launch", e);
  if (host_io) {
    struct {
      void* dst;
      const void* src;
      size_t n;
    } cp[] = {{out->macro_xs, sg.M, count * 40}, {out->energy, sg.E, count * 8},
              {out->mat, sg.omat, count * 4},    {out->grid_index, sg.gidx, count * 8},
              {out->verification, sg.v, count * 4}, {out->vsum, sg.vsum, 16}};
    for (auto& c : cp)
      if (c.dst) XS_TRY(cudaMemcpyAsync(c.dst, c.src, c.n, cudaMemcpyDeviceToHost, st), "D2H output");
    if (async_io)
      XS_TRY(cudaEventRecord(ws_ev, st), "event");
    else
      XS_TRY(cudaStreamSynchronize(st), "lookup (host io) completion");
  }
  return XS_OK;
}

xs_status xs_lookup_batch(xs_grid* g, uint64_t first_id, uint64_t count, uint32_t flags,
                          const xs_outputs* out, void* workspace, size_t workspace_bytes,
                          void* cuda_stream) {
  if (g && g->d.n_mats != XSGEN_N_MATS)
    return fail(XS_ERR_UNSUPPORTED, "sampled batches need the 12 XSBench materials");
  return lookup_common(g, first_id, nullptr, nullptr, count, flags, out, workspace,
                       workspace_bytes, cuda_stream);
}

xs_status xs_lookup_batch_shard(xs_grid* g, uint64_t first_id, uint64_t count, int32_t shard,
                                int32_t n_shards, uint32_t flags, const xs_outputs* out,
                                void* workspace, size_t workspace_bytes, void* cuda_stream) {
  if (g && g->d.n_mats != XSGEN_N_MATS)
    return fail(XS_ERR_UNSUPPORTED, "sampled batches need the 12 XSBench materials");
  if (n_shards < 1 || shard < 0 || shard >= n_shards)
    return fail(XS_ERR_INVALID_ARG, "need 0 <= shard < n_shards");
  if (!(flags & XS_FLAG_SORT) || (flags & (XS_FLAG_BASELINE | XS_FLAG_HOST_IO)))
    return fail(XS_ERR_INVALID_ARG, "energy-range shards need XS_FLAG_SORT and device outputs "
                                    "(no XS_FLAG_BASELINE / XS_FLAG_HOST_IO)");
  ShardSel s;
  s.on = true;
  s.e_lo = shard == 0 ? -HUGE_VAL : static_cast<double>(shard) / static_cast<double>(n_shards);
  s.e_hi = shard == n_shards - 1 ? HUGE_VAL
                                 : static_cast<double>(shard + 1) / static_cast<double>(n_shards);
  return lookup_common(g, first_id, nullptr, nullptr, count, flags, out, workspace,
                       workspace_bytes, cuda_stream, s);
}

xs_status xs_lookup_explicit(xs_grid* g, const double* energy, const int32_t* mat, uint64_t count,
                             uint32_t flags, const xs_outputs* out, void* workspace,
                             size_t workspace_bytes, void* cuda_stream) {
  if (count && (!energy || !mat)) return fail(XS_ERR_INVALID_ARG, "NULL energy/mat");
  return lookup_common(g, 0, energy, mat, count, flags, out, workspace, workspace_bytes,
                       cuda_stream);
}

// history mode (R19): event workspace for one round of n lookups
// (flags & XS_FLAG_SORT) + per-particle state
static size_t history_layout(uint64_t n, void* base, HistoryArgs* h) {
  size_t off = 0;
  auto take = [&](size_t bytes) {
    size_t o = off;
    off += align256(bytes);
    return o;
  };
  const size_t o_s = take(n * 8), o_e = take(n * 8), o_m = take(n * 4), o_M = take(n * 40);
  if (h) {
    char* b = static_cast<char*>(base);
    h->hist_state = reinterpret_cast<uint64_t*>(b + o_s);
    h->hist_energy = reinterpret_cast<double*>(b + o_e);
    h->hist_mat = reinterpret_cast<int32_t*>(b + o_m);
    h->hist_M = reinterpret_cast<double*>(b + o_M);
  }
  return off;
}

xs_status xs_history_workspace_size(const xs_grid* g, uint64_t n_particles, uint32_t flags,
                                    size_t* bytes) {
  if (!g || !bytes) return fail(XS_ERR_INVALID_ARG, "NULL argument");
  const uint32_t f = flags & XS_FLAG_SORT;
  *bytes = workspace_layout(n_particles, f, g->d.n_mats, nullptr, nullptr) +
           history_layout(n_particles, nullptr, nullptr);
  return XS_OK;
}

xs_status xs_lookup_history(xs_grid* g, uint64_t first_particle, uint64_t n_particles,
                            int32_t lookups, uint32_t flags, const xs_outputs* out,
                            void* workspace, size_t workspace_bytes, void* cuda_stream) {
  if (!g || !out) return fail(XS_ERR_INVALID_ARG, "NULL grid/outputs");
  if (!out->vsum) return fail(XS_ERR_INVALID_ARG, "outputs.vsum is required");
  if (out->grid_index)
    return fail(XS_ERR_UNSUPPORTED, "history mode does not report grid indices");
  if (flags & ~XS_FLAG_SORT) return fail(XS_ERR_INVALID_ARG, "history mode takes XS_FLAG_SORT only");
  if (lookups < 1) return fail(XS_ERR_INVALID_ARG, "lookups per particle must be >= 1");
  if (n_particles >= (1ULL << 32)) return fail(XS_ERR_INVALID_ARG, "n_particles must be < 2^32");
  if (g->d.n_mats != XSGEN_N_MATS)
    return fail(XS_ERR_UNSUPPORTED, "history mode samples the 12 XSBench materials");
  if (n_particles == 0) return XS_OK;
  size_t need = 0;
  xs_history_workspace_size(g, n_particles, flags, &need);
  if (!workspace || workspace_bytes < need)
    return fail(XS_ERR_INVALID_ARG, "workspace too small: need " + std::to_string(need) + " bytes");
  if (reinterpret_cast<uintptr_t>(workspace) & 255)
    return fail(XS_ERR_INVALID_ARG, "workspace must be 256-byte aligned");
  DeviceGuard guard(g->d.device);
  if (!guard.ok) return fail(XS_ERR_CUDA, "cudaSetDevice failed");
  Workspace ws;
  const size_t wbytes = workspace_layout(n_particles, flags, g->d.n_mats, workspace, &ws);
  HistoryArgs h;
  history_layout(n_particles, static_cast<char*>(workspace) + wbytes, &h);
  h.first_particle = first_particle;
  h.n_particles = static_cast<uint32_t>(n_particles);
  h.lookups = lookups;
  h.flags = flags;
  h.out = *out;
  h.launches = &g->d.launches;
  const cudaError_t e = run_history(g->d, h, ws, static_cast<cudaStream_t>(cuda_stream));
  if (e != cudaSuccess) return fail(XS_ERR_CUDA, "history launch", e);
  return XS_OK;
}

xs_status xs_verify(const xs_grid* g, const double* macro_xs, uint64_t count, uint64_t* vsum,
                    void* cuda_stream) {
  if (!g || !vsum || (count && !macro_xs)) return fail(XS_ERR_INVALID_ARG, "NULL argument");
  if (count == 0) return XS_OK;
  DeviceGuard guard(g->d.device);
  cudaError_t e = run_verify(g->d, macro_xs, count, vsum, static_cast<cudaStream_t>(cuda_stream));
  if (e != cudaSuccess) return fail(XS_ERR_CUDA, "verify launch", e);
  return XS_OK;
}

xs_status xs_nuclide_index(const xs_grid* g, const double* energy, const int32_t* nuclide,
                           uint64_t count, int32_t* k_out, void* cuda_stream) {
  if (!g || (count && (!energy || !nuclide || !k_out)))
    return fail(XS_ERR_INVALID_ARG, "NULL argument");
  if (count == 0) return XS_OK;
  DeviceGuard guard(g->d.device);
  cudaError_t e = run_nuclide_index(g->d, energy, nuclide, count, k_out,
                                    static_cast<cudaStream_t>(cuda_stream));
  if (e != cudaSuccess) return fail(XS_ERR_CUDA, "nuclide_index launch", e);
  return XS_OK;
}

xs_status xs_get_table(const xs_grid* g, int32_t table, uint64_t offset, uint64_t count,
                       void* host_dst) {
  if (!g || (count && !host_dst)) return fail(XS_ERR_INVALID_ARG, "NULL argument");
  const DeviceGrid& G = g->d;
  const void* src = nullptr;
  uint64_t len = 0;
  size_t es = 8;
  switch (table) {
    case XS_TABLE_NUCLIDE_GRID: src = G.grid; len = static_cast<uint64_t>(G.I) * G.N * 6; break;
    case XS_TABLE_UNION_ENERGY: src = G.U; len = G.NU; break;
    case XS_TABLE_INDEX_GRID:
      if (!G.index) return fail(XS_ERR_UNSUPPORTED, "grid has no row-layout index grid");
      src = G.index; len = G.index_len; es = 4; break;
    case XS_TABLE_INDEX_GRID_T:
      if (!G.index_t) return fail(XS_ERR_UNSUPPORTED, "grid has no column-layout index grid");
      src = G.index_t; len = G.index_len; es = 4; break;
    case XS_TABLE_INTERVALS: src = G.iv; len = static_cast<uint64_t>(G.I) * G.N * kIvDoubles; break;
    case XS_TABLE_INTERVALS32:
      src = G.iv32; len = static_cast<uint64_t>(G.I) * G.N * kIv32Doubles; break;
    case XS_TABLE_INTERVALS_U:
      if (!G.ivu) return fail(XS_ERR_UNSUPPORTED, "grid has no K0u table");
      src = G.ivu; len = static_cast<uint64_t>(G.I) * G.N * 12; break;
    case XS_TABLE_NUM_NUCS: src = G.num_nucs; len = G.n_mats; es = 4; break;
    case XS_TABLE_MATS: src = G.mats; len = static_cast<uint64_t>(G.n_mats) * G.max_nucs; es = 4; break;
    case XS_TABLE_CONCS: src = G.concs; len = static_cast<uint64_t>(G.n_mats) * G.max_nucs; break;
    default: return fail(XS_ERR_INVALID_ARG, "unknown table id");
  }
  if (offset > len || count > len - offset) return fail(XS_ERR_INVALID_ARG, "table range out of bounds");
  if (count == 0) return XS_OK;
  DeviceGuard guard(G.device);
  XS_TRY(cudaMemcpy(host_dst, static_cast<const char*>(src) + offset * es, count * es,
                    cudaMemcpyDeviceToHost),
         "table copy");
  return XS_OK;
}

xs_status xs_set_param(xs_grid* g, const char* name, int64_t value) {
  if (!g || !name) return fail(XS_ERR_INVALID_ARG, "NULL argument");
  DeviceGrid& G = g->d;
  if (!std::strcmp(name, "variant")) {
    if (!(value == 0 || (value >= 1 && value <= 4) || (value >= 9 && value <= 12) ||
          (value >= 17 && value <= 28) || (value >= 31 && value <= 36) ||
          (value >= 40 && value <= 59)))
      return fail(XS_ERR_INVALID_ARG, "variant must be 0, 1-4, 9-12, 17-28, 31-36 or 40-59");
    G.unroll = static_cast<int>(value);
  } else if (!std::strcmp(name, "host_chunk")) {
    if (value < 1024) return fail(XS_ERR_INVALID_ARG, "host_chunk >= 1024 lookups");
    g->host_chunk = static_cast<uint64_t>(value);
  } else if (!std::strcmp(name, "blocks_per_sm")) {
    if (value < 0 || value > 32) return fail(XS_ERR_INVALID_ARG, "blocks_per_sm in [0,32]");
    G.blocks_per_sm = static_cast<int>(value);
  } else if (!std::strcmp(name, "legacy_sort")) {
    if (value < 0 || value > 1) return fail(XS_ERR_INVALID_ARG, "legacy_sort is 0 or 1");
    G.legacy_sort = static_cast<int>(value);
  } else if (!std::strcmp(name, "part_cbits")) {
    if (value != 0 && (value < 6 || value > 9))
      return fail(XS_ERR_INVALID_ARG, "part_cbits is 0 (default) or 6-9");
    G.part_cbits = static_cast<int>(value);
  } else if (!std::strcmp(name, "fine_direct")) {
    if (value < 0 || value > 1024) return fail(XS_ERR_INVALID_ARG, "fine_direct in [0,1024]");
    G.fine_direct = static_cast<int>(value);
  } else if (!std::strcmp(name, "fine_cap")) {
    if (value != 0 && (value < 2048 || value > 24576))
      return fail(XS_ERR_INVALID_ARG, "fine_cap is 0 (default) or 2048-24576");
    G.fine_cap = static_cast<int>(value);
  } else if (!std::strcmp(name, "shard_tiles")) {
    if (value < 0 || value > 16) return fail(XS_ERR_INVALID_ARG, "shard_tiles in [0,16]");
    G.shard_tiles = static_cast<int>(value);
  } else {
    return fail(XS_ERR_INVALID_ARG, std::string("unknown parameter ") + name);
  }
  return XS_OK;
}

xs_status xs_timing_enable(xs_grid* g, int enable) {
  if (!g) return fail(XS_ERR_INVALID_ARG, "NULL grid");
  g->timing = enable != 0;
  g->ev_used = 0;
  g->calls = 0;
  g->launches_read = g->d.launches;
  return XS_OK;
}

xs_status xs_timing_read(xs_grid* g, xs_timing* out) {
  if (!g || !out) return fail(XS_ERR_INVALID_ARG, "NULL argument");
  DeviceGuard guard(g->d.device);
  std::memset(out, 0, sizeof(*out));
  out->calls = g->calls;
  out->kernel_launches = g->d.launches - g->launches_read;
  for (size_t i = 0; i < g->ev_used; ++i) {
    auto& e = g->ev[i];
    XS_TRY(cudaEventSynchronize(e[3]), "cudaEventSynchronize");
    float t[3];
    XS_TRY(cudaEventElapsedTime(&t[0], e[0], e[1]), "cudaEventElapsedTime");
    XS_TRY(cudaEventElapsedTime(&t[1], e[1], e[2]), "cudaEventElapsedTime");
    XS_TRY(cudaEventElapsedTime(&t[2], e[2], e[3]), "cudaEventElapsedTime");
    out->ms_count += t[0];
    out->ms_bucket += t[1];
    out->ms_gather += t[2];
  }
  out->ms_total = out->ms_count + out->ms_bucket + out->ms_gather;
  g->ev_used = 0;
  g->calls = 0;
  g->launches_read = g->d.launches;
  return XS_OK;
}

void xs_free_grid(xs_grid* g) {
  if (!g) return;
  DeviceGuard guard(g->d.device);
  for (auto& e : g->ev)
    for (auto x : e) cudaEventDestroy(x);
  for (auto x : g->chunk_ev) cudaEventDestroy(x);
  for (auto& pr : g->ws_done) cudaEventDestroy(pr.second);
  if (g->copy_stream) cudaStreamDestroy(g->copy_stream);
  cudaFree(g->d.grid);
  cudaFree(g->d.iv);
  cudaFree(g->d.iv32);
  cudaFree(g->d.ivu);
  cudaFree(g->d.U);
  cudaFree(g->d.UB);
  cudaFree(g->d.index);
  cudaFree(g->d.index_t);
  cudaFree(g->d.num_nucs);
  cudaFree(g->d.mats);
  cudaFree(g->d.concs);
  delete g;
}

}  // extern "C"
