// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o fp64_int_issue tools/fp64_int_issue.cu
// Does an FP64 warp instruction block the SMSP issue slot for 2 cycles?
#include <cstdio>
#include <cstdint>
template <int ND, int NI>
__global__ void k(double* out, int iters, double a, double b) {
  double d[8];
  uint32_t x[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) { d[i] = threadIdx.x + i; x[i] = threadIdx.x * 3 + i; }
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      if (i < ND) d[i] = __dadd_rn(__dmul_rn(d[i], a), b);
      if (i < NI) {
        uint32_t y;
        asm volatile("lop3.b32 %0, %1, %2, %3, 0x96;" : "=r"(y) : "r"(x[i]), "r"(x[(i + 1) & 7]), "r"(it));
        x[i] = y;
        asm volatile("lop3.b32 %0, %1, %2, %3, 0x96;" : "=r"(y) : "r"(x[i]), "r"(x[(i + 3) & 7]), "r"(it));
        x[i] = y;
      }
    }
  }
  double s = 0; uint32_t t = 0;
#pragma unroll
  for (int i = 0; i < 8; ++i) { s += d[i]; t ^= x[i]; }
  out[blockIdx.x * blockDim.x + threadIdx.x] = s + t;
}
template <int ND, int NI>
float run(double* o, int warps) {
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  k<ND, NI><<<148, 32 * warps>>>(o, 1000, 1.0000001, 1e-9);
  cudaEventRecord(e0);
  k<ND, NI><<<148, 32 * warps>>>(o, 20000, 1.0000001, 1e-9);
  cudaEventRecord(e1); cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  return ms;
}
int main() {
  double* o; cudaMalloc(&o, 148 * 1024 * 8);
  for (int w : {8, 16, 32}) {
    float a = run<8, 0>(o, w), b = run<8, 8>(o, w), c = run<0, 8>(o, w), d = run<8, 4>(o, w);
    // per SMSP: warps/4 warps x 20000 iters x instr
    double cyc = 1.965e6;  // cycles per ms
    double n = w / 4.0 * 20000;
    printf("warps %2d: fp64 only %.3f ms (%.2f cyc/iter/warp-slot)  fp64+16int %.3f (%.2f)  16int only %.3f (%.2f)  fp64+8int %.3f (%.2f)\n",
           w, a, a * cyc / n, b, b * cyc / n, c, c * cyc / n, d, d * cyc / n);
  }
}
