// Host-callable launchers of the ahead-of-time helper kernels (kf_kernels.cu).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace kf {
struct Geom {
  int64_t pitch, plane;
  int xoff, nx, ny, nz, gx, gy, gz;
};
cudaError_t launch_fill(int axis, void* base, int es, const Geom& g, cudaStream_t s);
// periodic x/y ghosts of n buffers, batched kMaxFillBufs per launch (px, py: axis periodic)
constexpr int kMaxFillBufs = 32;
cudaError_t launch_fill_xy_multi(void* const* bufs, int n, int px, int py, int es, const Geom& g, cudaStream_t s,
                                 int frozen_only = 0);
cudaError_t launch_copy_shell(void* dst, const void* src, int es, const Geom& g, cudaStream_t s);
cudaError_t launch_copy_box(void* dst, long long dpitch, long long dplane, const void* src, long long spitch,
                            long long splane, int w, int h, int d, int es, cudaStream_t s);
// one box copy (elements; strides in elements): halo strips, pack/unpack (a11)
struct BoxCopy {
  void* dst; const void* src;
  long long dpitch, dplane, spitch, splane;
  int w, h, d, pad;
};
constexpr int kMaxBoxes = 48;
struct BoxList { BoxCopy box[kMaxBoxes]; };
cudaError_t launch_copy_boxes(const BoxCopy* boxes, int n, int es, cudaStream_t s);
cudaError_t launch_flush(void* buf, long long bytes, unsigned v, cudaStream_t s);
}  // namespace kf
