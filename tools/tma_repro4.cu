// Parameterised TMA repro: box/dims/coords from argv.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdlib>
#include <cstring>
typedef unsigned long long u64; typedef unsigned u32;
struct __align__(64) KfTmap { u64 v[16]; };
struct Args { KfTmap tm[1]; int c0, c1, c2, bytes; };
__device__ __forceinline__ u32 su(const void* p) { return (u32)__cvta_generic_to_shared(p); }
__global__ void k_param(const __grid_constant__ Args a) {
  extern __shared__ __align__(128) unsigned char s[];
  u64* mb = (u64*)(s + 32768);
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(su(mb)), "r"(1));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(su(mb)), "r"(a.bytes) : "memory");
    asm volatile("cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];"
      :: "r"(su(s)), "l"((u64)&a.tm[0]), "r"(a.c0), "r"(a.c1), "r"(a.c2), "r"(su(mb)) : "memory");
  }
  u32 done = 0;
  do { asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }" : "=r"(done) : "r"(su(mb)), "r"(0) : "memory"); } while (!done);
}
typedef CUresult (*F)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
int main(int argc, char** argv) {
  int d0 = atoi(argv[1]), d1 = atoi(argv[2]), d2 = atoi(argv[3]), b0 = atoi(argv[4]), b1 = atoi(argv[5]);
  int es = atoi(argv[9]);
  void* src; cudaMalloc(&src, (size_t)d0 * d1 * d2 * es);
  void* fp; cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fp, cudaEnableDefault, &q);
  Args a; memset(&a, 0, sizeof a);
  cuuint64_t dims[3] = {(cuuint64_t)d0, (cuuint64_t)d1, (cuuint64_t)d2}, str[2] = {(cuuint64_t)d0 * es, (cuuint64_t)d0 * d1 * es};
  cuuint32_t box[3] = {(cuuint32_t)b0, (cuuint32_t)b1, 1}, est[3] = {1,1,1};
  CUresult r = ((F)fp)((CUtensorMap*)&a.tm[0], es == 4 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32 : CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 3, src, dims, str, box, est, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  a.c0 = atoi(argv[6]); a.c1 = atoi(argv[7]); a.c2 = atoi(argv[8]); a.bytes = b0 * b1 * es;
  cudaFuncSetAttribute(k_param, cudaFuncAttributeMaxDynamicSharedMemorySize, 40000);
  k_param<<<1, 256, 40000>>>(a);
  printf("dims %d %d %d box %d %d coords %d %d %d es %d: encode %d -> %s\n", d0, d1, d2, b0, b1, a.c0, a.c1, a.c2, es, r, cudaGetErrorString(cudaDeviceSynchronize()));
}
