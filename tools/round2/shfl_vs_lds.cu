// Microbenchmark (round 2): does a warp shuffle deliver neighbour values cheaper than a shared load
// on B200?  Per SM throughput of (A) LDS.128, (B) 4x SHFL.32 (the cost of moving one fp64 pair
// between lanes), (C) both interleaved (do they share a pipe?).  nvcc -arch=sm_100a -O3.
#include <cstdio>
#include <cuda_runtime.h>

template <int MODE>
__global__ void k(double* out, int iters) {
  __shared__ double4 sm[1024];
  const int t = threadIdx.x;
  for (int i = t; i < 1024; i += blockDim.x) sm[i] = make_double4(i, i + 1, i + 2, i + 3);
  __syncthreads();
  double a0 = t, a1 = 0;
  unsigned b0 = t, b1 = t + 1, b2 = t + 2, b3 = t + 3;
  int idx = t & 1023;
  for (int it = 0; it < iters; it++) {
    if (MODE == 0 || MODE == 2) {
      const double2 v = reinterpret_cast<const double2*>(sm)[(idx + it) & 2047];
      a0 += v.x;
      a1 += v.y;
    }
    if (MODE == 1 || MODE == 2) {
      b0 = __shfl_down_sync(0xffffffffu, b0, 1) + 1u;
      b1 = __shfl_down_sync(0xffffffffu, b1, 1) + 2u;
      b2 = __shfl_down_sync(0xffffffffu, b2, 1) + 3u;
      b3 = __shfl_down_sync(0xffffffffu, b3, 1) + 4u;
    }
  }
  out[blockIdx.x * blockDim.x + t] = a0 + a1 + double(b0 ^ b1 ^ b2 ^ b3);
}

int main() {
  int blocks = 148 * 8, threads = 256, iters = 4096;
  double* out;
  cudaMalloc(&out, sizeof(double) * blocks * threads);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  int clk;
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  const char* names[] = {"LDS.128 (16 B/lane)", "4x SHFL.32 (16 B/lane)", "LDS.128 + 4x SHFL"};
  for (int m = 0; m < 3; m++) {
    for (int rep = 0; rep < 2; rep++) {
      cudaEventRecord(e0);
      if (m == 0) k<0><<<blocks, threads>>>(out, iters);
      if (m == 1) k<1><<<blocks, threads>>>(out, iters);
      if (m == 2) k<2><<<blocks, threads>>>(out, iters);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms;
      cudaEventElapsedTime(&ms, e0, e1);
      if (rep == 1) {
        const double warp_ops = double(blocks) * threads / 32 * iters;
        const double cyc = ms * 1e-3 * clk * 1e3;   // SM clock cycles (max clock)
        printf("%-24s %.3f ms  %.3f warp-iterations/clk/SM  (%.1f B/clk/SM moved between lanes or from shared)\n", names[m], ms,
               warp_ops / cyc / 148, warp_ops * 512 / cyc / 148);
      }
    }
  }
  return 0;
}
