// FP64 pipe throughput on this GPU (development aid; the number is the
// "alu" roofline peak of the sorted gather).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/fp64_peak tools/fp64_peak.cu
// Prints FP64 instructions/s (lane operations) for DADD, DMUL and DFMA with
// 8 independent dependency chains per thread, 148 x 8 blocks of 256 threads.
#include <cstdio>
#include <cuda_runtime.h>

template <int OP>
__global__ void k_fp64(double* out, int iters, double a, double b) {
  double x[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) x[i] = threadIdx.x * 1e-3 + i;
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      if (OP == 0) x[i] = __dadd_rn(x[i], a);
      if (OP == 1) x[i] = __dmul_rn(x[i], b);
      if (OP == 2) x[i] = __fma_rn(x[i], b, a);
    }
  }
  double s = 0;
#pragma unroll
  for (int i = 0; i < 8; ++i) s += x[i];
  if (s == 12345.678) out[0] = s;  // keep the chains alive
}

// dependent-chain latency: one thread, one chain
__global__ void k_lat(double* out, int iters, double a, long long* cyc) {
  double x = threadIdx.x * 1e-3;
  const long long t0 = clock64();
  for (int it = 0; it < iters; ++it) x = __dadd_rn(x, a);
  const long long t1 = clock64();
  if (x == 12345.678) out[0] = x;
  cyc[0] = t1 - t0;
}

// throughput with C independent chains per thread at a given warps/SM
template <int C>
__global__ void k_ilp(double* out, int iters, double a) {
  double x[C];
#pragma unroll
  for (int i = 0; i < C; ++i) x[i] = threadIdx.x * 1e-3 + i;
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < C; ++i) x[i] = __dadd_rn(x[i], a);
  }
  double s = 0;
#pragma unroll
  for (int i = 0; i < C; ++i) s += x[i];
  if (s == 12345.678) out[0] = s;
}

int main() {
  int dev = 0, sms = 0, mhz = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  cudaDeviceGetAttribute(&mhz, cudaDevAttrClockRate, dev);
  double* out;
  cudaMalloc(&out, 8);
  const int blocks = sms * 8, threads = 256, iters = 20000;
  const char* names[3] = {"DADD", "DMUL", "DFMA"};
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  printf("{\"sms\": %d, \"clock_khz_attr\": %d", sms, mhz);
  for (int op = 0; op < 3; ++op) {
    auto launch = [&]() {
      if (op == 0) k_fp64<0><<<blocks, threads>>>(out, iters, 1e-9, 1.0000001);
      if (op == 1) k_fp64<1><<<blocks, threads>>>(out, iters, 1e-9, 1.0000001);
      if (op == 2) k_fp64<2><<<blocks, threads>>>(out, iters, 1e-9, 1.0000001);
    };
    launch();
    cudaDeviceSynchronize();
    float best = 1e30f;
    for (int r = 0; r < 5; ++r) {
      cudaEventRecord(e0);
      launch();
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms;
      cudaEventElapsedTime(&ms, e0, e1);
      if (ms < best) best = ms;
    }
    const double ops = double(blocks) * threads * iters * 8;
    printf(", \"%s_ops_per_s\": %.4e, \"%s_per_sm_per_clk_at_attr\": %.2f", names[op],
           ops / (best * 1e-3), names[op], ops / (best * 1e-3) / sms / (mhz * 1e3));
  }
  {
    long long* cyc;
    cudaMalloc(&cyc, 8);
    k_lat<<<1, 1>>>(out, 100000, 1e-9, cyc);
    cudaDeviceSynchronize();
    long long c = 0;
    cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost);
    printf(", \"DADD_latency_cycles\": %.2f", c / 100000.0);
  }
  // lane-ops per SM per clock vs warps per SM and chains per thread
  for (int warps : {4, 8, 12, 16, 24}) {
    for (int chains : {1, 2, 4, 8}) {
      auto go = [&]() {
        if (chains == 1) k_ilp<1><<<sms, warps * 32>>>(out, iters * 8, 1e-9);
        if (chains == 2) k_ilp<2><<<sms, warps * 32>>>(out, iters * 4, 1e-9);
        if (chains == 4) k_ilp<4><<<sms, warps * 32>>>(out, iters * 2, 1e-9);
        if (chains == 8) k_ilp<8><<<sms, warps * 32>>>(out, iters, 1e-9);
      };
      go();
      cudaDeviceSynchronize();
      cudaEventRecord(e0);
      go();
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms;
      cudaEventElapsedTime(&ms, e0, e1);
      const double ops = double(sms) * warps * 32 * iters * 8;
      printf(", \"w%d_c%d\": %.1f", warps, chains, ops / (ms * 1e-3) / sms / (mhz * 1e3));
    }
  }
  printf("}\n");
  return 0;
}
