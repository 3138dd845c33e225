// Shared-memory wavefronts per LDS.64 / LDS.128 by address pattern.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o lds_wavefronts tools/lds_wavefronts.cu
// ncu --metrics l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,smsp__inst_executed_op_shared_ld.sum ./lds_wavefronts
// wavefronts per LDS.128 / LDS.64 for different address patterns
#include <cstdio>
#include <cstdint>
__global__ void k(double* out, int mode, int iters) {
  __shared__ double2 s[1024];
  for (int i = threadIdx.x; i < 1024; i += blockDim.x) s[i] = make_double2(i, i + 1);
  __syncthreads();
  int lane = threadIdx.x & 31;
  int a;
  if (mode == 0) a = 0;                 // broadcast
  else if (mode == 1) a = (lane >= 16) * 7;  // two addresses
  else if (mode == 2) a = lane;        // 32 distinct consecutive
  else a = (lane / 4) * 7;             // 8 distinct
  double acc = 0;
  for (int it = 0; it < iters; ++it) {
    double2 v = s[(a + it) & 1023];
    acc += v.x * v.y;
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}
__global__ void k64(double* out, int mode, int iters) {
  __shared__ double s[2048];
  for (int i = threadIdx.x; i < 2048; i += blockDim.x) s[i] = i;
  __syncthreads();
  int lane = threadIdx.x & 31;
  int a;
  if (mode == 0) a = 0;
  else if (mode == 1) a = (lane >= 16) * 14;
  else if (mode == 2) a = lane;
  else a = (lane / 4) * 14;
  double acc = 0;
  for (int it = 0; it < iters; ++it) acc += s[(a + 2*it) & 2047];
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}
int main() {
  double* o; cudaMalloc(&o, 148 * 256 * 8);
  for (int m = 0; m < 4; ++m) { k<<<148, 256>>>(o, m, 1000); k64<<<148, 256>>>(o, m, 1000); }
  cudaDeviceSynchronize();
  printf("done\n");
}
