// Launch an NVRTC-generated cubin (KF_DUMP_DIR) via the driver API, two ways.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstring>
#include <vector>
#include <fstream>
#include <iterator>
typedef CUresult (*F)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
int main(int argc, char** argv) {
  std::ifstream f(argv[1], std::ios::binary); std::vector<char> cub((std::istreambuf_iterator<char>(f)), {});
  cudaFree(0);
  float* a; size_t elems = 96 * 20 * 12; cudaMalloc(&a, elems * 4 * 3); cudaMemset(a, 0, elems * 12);
  void* fp; cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fp, cudaEnableDefault, &q);
  alignas(64) unsigned char blob[192]; memset(blob, 0, sizeof blob);
  cuuint64_t dims[3] = {96, 20, 12}, str[2] = {384, 7680}; cuuint32_t box[3] = {36, 18, 1}, es[3] = {1,1,1};
  CUresult r = ((F)fp)((CUtensorMap*)blob, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, a, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  float* out = a + elems + 2*7680/4*0 + 2*96 + 32; memcpy(blob + 128, &out, 8);
  printf("encode %d\n", r);
  for (int variant = 0; variant < 2; variant++) {
    CUmodule m; CUfunction fn;
    CUresult (*load)(CUmodule*, const void*); CUresult (*get)(CUfunction*, CUmodule, const char*);
    CUresult (*attr)(CUfunction, CUfunction_attribute, int);
    CUresult (*launch)(CUfunction, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned, CUstream, void**, void**);
    if (variant == 0) {
      cudaGetDriverEntryPoint("cuModuleLoadData", (void**)&load, cudaEnableDefault, &q);
      cudaGetDriverEntryPoint("cuModuleGetFunction", (void**)&get, cudaEnableDefault, &q);
      cudaGetDriverEntryPoint("cuFuncSetAttribute", (void**)&attr, cudaEnableDefault, &q);
      cudaGetDriverEntryPoint("cuLaunchKernel", (void**)&launch, cudaEnableDefault, &q);
    } else { load = cuModuleLoadData; get = cuModuleGetFunction; attr = cuFuncSetAttribute; launch = cuLaunchKernel; }
    printf("v%d load %d\n", variant, load(&m, cub.data()));
    printf("v%d get %d\n", variant, get(&fn, m, argv[2]));
    attr(fn, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, 10896);
    void* params[] = {blob};
    printf("v%d launch %d\n", variant, launch(fn, 1, 1, 1, 256, 1, 1, 10896, 0, params, nullptr));
    printf("v%d sync %s\n", variant, cudaGetErrorString(cudaDeviceSynchronize()));
  }
}
