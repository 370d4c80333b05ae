// Minimal TMA repro: grid_constant tensor map vs tensor map in global memory.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstring>
typedef unsigned long long u64; typedef unsigned u32;
struct __align__(64) KfTmap { u64 v[16]; };
struct Args { KfTmap tm[1]; float* out; };
__device__ __forceinline__ u32 su(const void* p) { return (u32)__cvta_generic_to_shared(p); }
__device__ void body(const KfTmap* map, float* out) {
  __shared__ __align__(128) float s[64 * 4];
  __shared__ __align__(8) u64 mb;
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(su(&mb)), "r"(1));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(su(&mb)), "r"(64*4*4) : "memory");
    asm volatile("cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];"
      :: "r"(su(s)), "l"((u64)map), "r"(0), "r"(0), "r"(0), "r"(su(&mb)) : "memory");
  }
  u32 done = 0;
  do { asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }" : "=r"(done) : "r"(su(&mb)), "r"(0) : "memory"); } while (!done);
  out[threadIdx.x] = s[threadIdx.x];
}
__global__ void k_param(const __grid_constant__ Args a) { body(&a.tm[0], a.out); }
__global__ void k_global(const KfTmap* m, float* out) { body(m, out); }
int main() {
  float *src, *out; cudaMalloc(&src, 64*4*4*4); cudaMalloc(&out, 1024*4);
  float h[1024]; for (int i = 0; i < 1024; i++) h[i] = i; cudaMemcpy(src, h, 64*4*4*4, cudaMemcpyHostToDevice);
  void* fp; cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fp, cudaEnableDefault, &q);
  typedef CUresult (*F)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
  Args a; memset(&a, 0, sizeof a);
  cuuint64_t dims[3] = {64, 4, 4}, str[2] = {64*4, 64*4*4}; cuuint32_t box[3] = {64, 4, 1}, es[3] = {1,1,1};
  CUresult r = ((F)fp)((CUtensorMap*)&a.tm[0], CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, src, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  printf("encode %d sizeof(Args)=%zu\n", r, sizeof(Args));
  a.out = out;
  KfTmap* gm; cudaMalloc(&gm, sizeof(KfTmap)); cudaMemcpy(gm, &a.tm[0], sizeof(KfTmap), cudaMemcpyHostToDevice);
  k_global<<<1, 256>>>(gm, out); printf("global: %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
  cudaMemcpy(h, out, 256*4, cudaMemcpyDeviceToHost); printf("  out[5]=%g out[255]=%g\n", h[5], h[255]);
  k_param<<<1, 256>>>(a); printf("param: %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
  cudaMemcpy(h, out, 256*4, cudaMemcpyDeviceToHost); printf("  out[5]=%g out[255]=%g\n", h[5], h[255]);
}
