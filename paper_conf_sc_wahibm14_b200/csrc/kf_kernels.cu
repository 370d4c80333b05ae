// Ahead-of-time sm_100a helper kernels of the executor (row a10): periodic ghost fill,
// ghost-shell copy for renamed buffers, L2 flush.  The fused-group kernels themselves
// are generated per group and JIT-compiled (kf_codegen.cpp / kf_runtime.cpp).
//
// Layout (kf_array_layout): element (i,j,k), i in [-gx, nx+gx), is at
//   base + (k+gz)*plane + (j+gy)*pitch + xoff + i.
#include <cuda_runtime.h>
#include <stdint.h>

#include "kf_kernels.hpp"

namespace kf {

// Periodic wrap of the ghost layer along x: for every row of the ghosted domain,
// ghost[-1-i] <- interior[nx-1-i], ghost[nx+i] <- interior[i]   (R9, P:82 padding).
template <typename T>
__global__ void fill_x(T* __restrict__ base, Geom g) {
  const int rows = (g.ny + 2 * g.gy) * (g.nz + 2 * g.gz);
  const int w = 2 * g.gx;
  for (long long idx = blockIdx.x * (long long)blockDim.x + threadIdx.x; idx < (long long)rows * w;
       idx += (long long)gridDim.x * blockDim.x) {
    const int r = int(idx / w), e = int(idx % w);
    const int zz = r / (g.ny + 2 * g.gy), yy = r % (g.ny + 2 * g.gy);
    T* row = base + zz * g.plane + yy * g.pitch + g.xoff;
    if (e < g.gx) row[-1 - e] = row[g.nx - 1 - e];
    else row[g.nx + (e - g.gx)] = row[e - g.gx];
  }
}

// Periodic wrap along y: whole padded rows (x ghosts included, so corners are covered
// after fill_x).
template <typename T>
__global__ void fill_y(T* __restrict__ base, Geom g) {
  const int nrow = 2 * g.gy * (g.nz + 2 * g.gz);
  const long long W = g.pitch;
  for (long long idx = blockIdx.x * (long long)blockDim.x + threadIdx.x; idx < nrow * W;
       idx += (long long)gridDim.x * blockDim.x) {
    const int r = int(idx / W), x = int(idx % W);
    const int zz = r / (2 * g.gy), e = r % (2 * g.gy);
    T* pl = base + zz * g.plane;
    int dst, src;
    if (e < g.gy) { dst = g.gy - 1 - e; src = g.gy + g.ny - 1 - e; }
    else { dst = g.gy + g.ny + (e - g.gy); src = g.gy + (e - g.gy); }
    pl[dst * g.pitch + x] = pl[src * g.pitch + x];
  }
}

// Periodic wrap along z: whole planes.
template <typename T>
__global__ void fill_z(T* __restrict__ base, Geom g) {
  const long long P = g.plane;
  for (long long idx = blockIdx.x * (long long)blockDim.x + threadIdx.x; idx < 2LL * g.gz * P;
       idx += (long long)gridDim.x * blockDim.x) {
    const int e = int(idx / P);
    const long long o = idx % P;
    int dst, src;
    if (e < g.gz) { dst = g.gz - 1 - e; src = g.gz + g.nz - 1 - e; }
    else { dst = g.gz + g.nz + (e - g.gz); src = g.gz + (e - g.gz); }
    base[dst * P + o] = base[src * P + o];
  }
}

// Copy every element that is not interior (ghost shell and padding) from src to dst:
// renamed copies of an array share its frozen ghost values (R9).
template <typename T>
__global__ void copy_shell(T* __restrict__ dst, const T* __restrict__ src, Geom g) {
  const long long total = (long long)g.plane * (g.nz + 2 * g.gz);
  for (long long idx = blockIdx.x * (long long)blockDim.x + threadIdx.x; idx < total;
       idx += (long long)gridDim.x * blockDim.x) {
    const int zz = int(idx / g.plane);
    const long long o = idx % g.plane;
    const int yy = int(o / g.pitch), xx = int(o % g.pitch);
    const bool interior = zz >= g.gz && zz < g.gz + g.nz && yy >= g.gy && yy < g.gy + g.ny && xx >= g.xoff &&
                          xx < g.xoff + g.nx;
    if (!interior) dst[idx] = src[idx];
  }
}

// Copy a w x h x d box between two buffers (elements; arbitrary pitches): halo strips for
// domain decomposition (loopback transport) and pack/unpack to contiguous NCCL staging.
template <typename T>
__global__ void copy_box(T* __restrict__ dst, long long dpitch, long long dplane, const T* __restrict__ src,
                         long long spitch, long long splane, int w, int h, int d) {
  const long long total = (long long)w * h * d;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total; i += (long long)gridDim.x * blockDim.x) {
    const int x = int(i % w);
    const long long r = i / w;
    const int y = int(r % h), z = int(r / h);
    dst[z * dplane + y * dpitch + x] = src[z * splane + y * spitch + x];
  }
}

__global__ void flush_kernel(uint4* __restrict__ buf, long long n, unsigned v) {
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
    buf[i] = make_uint4(v, v + 1, v + 2, v + 3);
}

static int blocks_for(long long n) {
  long long b = (n + 255) / 256;
  return int(b < 148 * 16 ? (b < 1 ? 1 : b) : 148 * 16);
}

cudaError_t launch_fill(int axis, void* base, int es, const Geom& g, cudaStream_t s) {
  long long n = axis == 0 ? 2LL * g.gx * (g.ny + 2 * g.gy) * (g.nz + 2 * g.gz)
              : axis == 1 ? 2LL * g.gy * (g.nz + 2 * g.gz) * g.pitch
                          : 2LL * g.gz * g.plane;
  if (n == 0) return cudaSuccess;
  int nb = blocks_for(n);
  if (es == 4) {
    if (axis == 0) fill_x<float><<<nb, 256, 0, s>>>((float*)base, g);
    else if (axis == 1) fill_y<float><<<nb, 256, 0, s>>>((float*)base, g);
    else fill_z<float><<<nb, 256, 0, s>>>((float*)base, g);
  } else {
    if (axis == 0) fill_x<double><<<nb, 256, 0, s>>>((double*)base, g);
    else if (axis == 1) fill_y<double><<<nb, 256, 0, s>>>((double*)base, g);
    else fill_z<double><<<nb, 256, 0, s>>>((double*)base, g);
  }
  return cudaGetLastError();
}

cudaError_t launch_copy_shell(void* dst, const void* src, int es, const Geom& g, cudaStream_t s) {
  long long n = (long long)g.plane * (g.nz + 2 * g.gz);
  int nb = blocks_for(n);
  if (es == 4) copy_shell<float><<<nb, 256, 0, s>>>((float*)dst, (const float*)src, g);
  else copy_shell<double><<<nb, 256, 0, s>>>((double*)dst, (const double*)src, g);
  return cudaGetLastError();
}

cudaError_t launch_copy_box(void* dst, long long dpitch, long long dplane, const void* src, long long spitch,
                            long long splane, int w, int h, int d, int es, cudaStream_t s) {
  long long n = (long long)w * h * d;
  if (n == 0) return cudaSuccess;
  int nb = blocks_for(n);
  if (es == 4) copy_box<float><<<nb, 256, 0, s>>>((float*)dst, dpitch, dplane, (const float*)src, spitch, splane, w, h, d);
  else copy_box<double><<<nb, 256, 0, s>>>((double*)dst, dpitch, dplane, (const double*)src, spitch, splane, w, h, d);
  return cudaGetLastError();
}

cudaError_t launch_flush(void* buf, long long bytes, unsigned v, cudaStream_t s) {
  long long n = bytes / 16;
  flush_kernel<<<148 * 8, 256, 0, s>>>((uint4*)buf, n, v);
  return cudaGetLastError();
}

}  // namespace kf
