// Ahead-of-time sm_100a helper kernels of the executor (row a10): periodic ghost fill,
// ghost-shell copy for renamed buffers, L2 flush.  The fused-group kernels themselves
// are generated per group and JIT-compiled (kf_codegen.cpp / kf_runtime.cpp).
//
// Layout (kf_array_layout): element (i,j,k), i in [-gx, nx+gx), is at
//   base + (k+gz)*plane + (j+gy)*pitch + xoff + i.
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>

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

// Periodic x and y ghosts of several buffers in one launch (blockIdx.y = buffer): every ghost
// cell takes the interior cell its coordinates wrap to on the periodic axes (a frozen axis keeps
// its coordinate), which is what fill_x followed by fill_y produces, corners included, without
// the ordering between the two passes.  Pieces: the x-ghost columns of every padded row (if x
// is periodic) and the y-ghost rows over the x range not already covered (if y is periodic).
struct FillList { void* base[kMaxFillBufs]; };

// frozen_only: only the ghost cells lying in the ghost layer of a FROZEN axis (bit 0 x, 1 y, 2 z
// frozen) -- the run-start fill of renamed scratch versions, whose other cells are not written yet
// (they are filled or ghost-written after their producer).
template <typename T>
__global__ void fill_xy_multi(FillList L, Geom g, int px, int py, int frozen_only) {
  T* base = (T*)L.base[blockIdx.y];
  const int NZ = g.nz + 2 * g.gz, NYp = g.ny + 2 * g.gy;
  const long long nxs = px ? 2LL * g.gx * NYp * NZ : 0;                  // x-ghost columns
  const int x_lo = px ? 0 : -g.gx, x_w = px ? g.nx : g.nx + 2 * g.gx;    // y rows: x range not in nxs
  const long long nys = py ? (long long)x_w * 2 * g.gy * NZ : 0;
  for (long long idx = blockIdx.x * (long long)blockDim.x + threadIdx.x; idx < nxs + nys;
       idx += (long long)gridDim.x * blockDim.x) {
    int i, j, k;
    if (idx < nxs) {
      const int e = int(idx % (2 * g.gx));
      const long long r = idx / (2 * g.gx);
      j = int(r % NYp) - g.gy;
      k = int(r / NYp) - g.gz;
      i = e < g.gx ? -1 - e : g.nx + (e - g.gx);
    } else {
      const long long q = idx - nxs;
      i = x_lo + int(q % x_w);
      const long long r = q / x_w;
      const int e = int(r % (2 * g.gy));
      k = int(r / (2 * g.gy)) - g.gz;
      j = e < g.gy ? -1 - e : g.ny + (e - g.gy);
    }
    const int si = (px && (i < 0 || i >= g.nx)) ? (i < 0 ? i + g.nx : i - g.nx) : i;
    const int sj = (py && (j < 0 || j >= g.ny)) ? (j < 0 ? j + g.ny : j - g.ny) : j;
    if (frozen_only && !(((frozen_only & 1) && (i < 0 || i >= g.nx)) || ((frozen_only & 2) && (j < 0 || j >= g.ny)) ||
                         ((frozen_only & 4) && (k < 0 || k >= g.nz))))
      continue;
    const long long o = (long long)(k + g.gz) * g.plane + g.xoff;
    base[o + (long long)(j + g.gy) * g.pitch + i] = base[o + (long long)(sj + g.gy) * g.pitch + si];
  }
}

// Periodic x and y ghosts of several buffers in one launch (blockIdx.y = buffer), written in whole
// 32-byte sectors: a ghost span is widened to sector boundaries (padding cells take any wrapped
// value; an interior cell in a shared sector is rewritten with itself), so no store is a partial
// sector (a partial sector costs the L2 a read-modify-write with ECC; measured round 2).  Lanes map
// to consecutive cells of a row span, so a warp stores whole sectors.  Every written cell takes the
// interior cell its coordinates wrap to on the periodic axes (corners included), as fill_xy_multi.
// Pieces: x spans of every row (x periodic; interior rows only if y is periodic as well), then
// whole y-ghost rows (y periodic).  frozen_only (bits x/y/z frozen): only cells inside a frozen
// axis' ghost layer, exact cells (the run-start fill of scratch buffers).
template <typename T>
__global__ void fill_xy_sectors(FillList L, Geom g, int px, int py, int frozen_only) {
  T* base = (T*)L.base[blockIdx.y];
  constexpr int E = 32 / sizeof(T);
  const int NZ = g.nz + 2 * g.gz;
  const int xl0 = -((g.gx + E - 1) / E) * E;                 // left span [xl0, 0)
  const int xr0 = (g.nx / E) * E, xr1 = ((g.nx + g.gx + E - 1) / E) * E;   // right span [xr0, xr1)
  const int cx = px ? (-xl0) + (xr1 - xr0) : 0;              // cells per row of the x pass
  const int rows_x = py ? g.ny : g.ny + 2 * g.gy;
  const int jx0 = py ? 0 : -g.gy;
  const int cy = py ? xr1 - xl0 : 0;                         // cells per y-ghost row: [xl0, xr1)
  const long long nx_cells = (long long)cx * rows_x * NZ, ny_cells = (long long)cy * 2 * g.gy * NZ;
  for (long long idx = blockIdx.x * (long long)blockDim.x + threadIdx.x; idx < nx_cells + ny_cells;
       idx += (long long)gridDim.x * blockDim.x) {
    int i, j, k;
    if (idx < nx_cells) {
      const unsigned q = unsigned(idx);
      const unsigned r = q / unsigned(cx), c = q - r * unsigned(cx);
      k = int(r / unsigned(rows_x)) - g.gz;
      j = jx0 + int(r % unsigned(rows_x));
      i = int(c) < -xl0 ? xl0 + int(c) : xr0 + int(c) + xl0;
    } else {
      const unsigned q = unsigned(idx - nx_cells);
      const unsigned r = q / unsigned(cy), c = q - r * unsigned(cy);
      const int e = int(r % unsigned(2 * g.gy));
      k = int(r / unsigned(2 * g.gy)) - g.gz;
      j = e < g.gy ? -1 - e : g.ny + (e - g.gy);
      i = xl0 + int(c);
    }
    if (frozen_only) {
      const bool gi = i < 0 || i >= g.nx, gj = j < 0 || j >= g.ny, gk = k < 0 || k >= g.nz;
      const bool cell = (px ? (i >= -g.gx && i < g.nx + g.gx) : true) && (py ? (j >= -g.gy && j < g.ny + g.gy) : true);
      if (!cell || (!gi && !gj) || !(((frozen_only & 1) && gi) || ((frozen_only & 2) && gj) || ((frozen_only & 4) && gk)))
        continue;
    }
    int si = i, sj = j;
    if (px && (i < 0 || i >= g.nx)) si = ((i % g.nx) + g.nx) % g.nx;
    if (!px) si = i < -g.gx ? -g.gx : (i >= g.nx + g.gx ? g.nx + g.gx - 1 : i);   // padding: any stored cell
    if (py && (j < 0 || j >= g.ny)) sj = ((j % g.ny) + g.ny) % g.ny;
    const long long o = (long long)(k + g.gz) * g.plane + g.xoff;
    base[o + (long long)(j + g.gy) * g.pitch + i] = base[o + (long long)(sj + g.gy) * g.pitch + si];
  }
}

// Copy every element that is not interior (ghost shell and padding) from src to dst:
// renamed copies of an array share its frozen ghost values (R9).  One CTA per padded row
// (grid-stride): ghost rows / planes whole, interior rows only their x ghost + padding ends.
template <typename T>
__global__ void copy_shell(T* __restrict__ dst, const T* __restrict__ src, Geom g) {
  const int rows = (g.ny + 2 * g.gy) * (g.nz + 2 * g.gz);
  for (int r = blockIdx.x; r < rows; r += gridDim.x) {
    const int zz = r / (g.ny + 2 * g.gy), yy = r - zz * (g.ny + 2 * g.gy);
    const long long o = (long long)zz * g.plane + (long long)yy * g.pitch;
    const bool inner = zz >= g.gz && zz < g.gz + g.nz && yy >= g.gy && yy < g.gy + g.ny;
    const int skip0 = inner ? g.xoff : int(g.pitch), skip1 = inner ? g.xoff + g.nx : int(g.pitch);
    for (int x = threadIdx.x; x < int(g.pitch); x += blockDim.x) {
      if (x >= skip0 && x < skip1) {   // jump over the interior
        x = skip1 - 1 - (skip1 - 1 - x) % int(blockDim.x);
        continue;
      }
      dst[o + x] = src[o + x];
    }
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

// Many w x h x d box copies in one launch (blockIdx.y = box): the strips of every buffer of an
// exchange phase are packed / unpacked / copied together (a11).  Box element counts fit 32 bits
// (ghost-deep strips), so the index arithmetic is 32-bit (division by the box's w and h only).
template <typename T>
__global__ void copy_boxes(BoxList L) {
  const BoxCopy& b = L.box[blockIdx.y];
  T* __restrict__ dst = (T*)b.dst;
  const T* __restrict__ src = (const T*)b.src;
  const unsigned w = unsigned(b.w), wh = unsigned(b.w) * unsigned(b.h);
  const unsigned total = wh * unsigned(b.d);
  for (unsigned i = blockIdx.x * blockDim.x + threadIdx.x; i < total; i += gridDim.x * blockDim.x) {
    const unsigned z = i / wh, r = i - z * wh, y = r / w, x = r - y * w;
    dst[z * b.dplane + (long long)y * b.dpitch + x] = src[z * b.splane + (long long)y * b.spitch + x];
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

cudaError_t launch_fill_xy_multi(void* const* bufs, int n, int px, int py, int es, const Geom& g, cudaStream_t s,
                                 int frozen_only) {
  if (!px && !py) return cudaSuccess;
  const long long NZ = g.nz + 2 * g.gz;
  // sector-wide writes need the row origin (x = 0) 32-byte aligned (kf_array_layout: 128-byte rows)
  const int E = 32 / es;
  const bool sectors = !getenv("KF_FILL_CELLS") && (g.xoff * (long long)es) % 32 == 0 && (g.pitch * (long long)es) % 32 == 0 &&
                       (g.plane * (long long)es) % 32 == 0 && ((g.gx + E - 1) / E) * E <= g.xoff;
  long long per = (px ? 2LL * g.gx * (g.ny + 2 * g.gy) : 0) * NZ +
                  (py ? (long long)(px ? g.nx : g.nx + 2 * g.gx) * 2 * g.gy * NZ : 0);
  if (sectors) {
    const long long xl = ((g.gx + E - 1) / E) * E, xr = ((g.nx + g.gx + E - 1) / E) * E - (g.nx / E) * E;
    per = (px ? (xl + xr) * (long long)(py ? g.ny : g.ny + 2 * g.gy) : 0) * NZ +
          (py ? (xl + (long long)((g.nx + g.gx + E - 1) / E) * E) * 2 * g.gy * NZ : 0);
  }
  if (per == 0) return cudaSuccess;
  for (int b0 = 0; b0 < n; b0 += kMaxFillBufs) {
    const int m = n - b0 < kMaxFillBufs ? n - b0 : kMaxFillBufs;
    FillList L{};
    for (int i = 0; i < m; i++) L.base[i] = bufs[b0 + i];
    long long nb = (per + 255) / 256;
    const long long cap = (148LL * 16 + m - 1) / m;   // ~16 CTAs per SM over all buffers
    dim3 grid(unsigned(nb < cap ? nb : cap), unsigned(m));
    if (sectors && es == 4) fill_xy_sectors<float><<<grid, 256, 0, s>>>(L, g, px, py, frozen_only);
    else if (sectors) fill_xy_sectors<double><<<grid, 256, 0, s>>>(L, g, px, py, frozen_only);
    else if (es == 4) fill_xy_multi<float><<<grid, 256, 0, s>>>(L, g, px, py, frozen_only);
    else fill_xy_multi<double><<<grid, 256, 0, s>>>(L, g, px, py, frozen_only);
  }
  return cudaGetLastError();
}

cudaError_t launch_copy_shell(void* dst, const void* src, int es, const Geom& g, cudaStream_t s) {
  const long long rows = (long long)(g.ny + 2 * g.gy) * (g.nz + 2 * g.gz);
  const int nb = int(rows < 148 * 32 ? rows : 148 * 32);
  if (es == 4) copy_shell<float><<<nb, 128, 0, s>>>((float*)dst, (const float*)src, g);
  else copy_shell<double><<<nb, 128, 0, s>>>((double*)dst, (const double*)src, g);
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

// A box whose rows are whole 16-byte units at 16-byte aligned addresses (ghost-deep x strips of
// fp64 with an even ghost width, whole padded rows of y strips) is copied as uint4 elements.
static bool vec16(const BoxCopy& b, int es) {
  const long long m = 16;
  return (reinterpret_cast<uintptr_t>(b.dst) % m) == 0 && (reinterpret_cast<uintptr_t>(b.src) % m) == 0 &&
         (b.w * (long long)es) % m == 0 && (b.dpitch * es) % m == 0 && (b.spitch * es) % m == 0 &&
         (b.dplane * es) % m == 0 && (b.splane * es) % m == 0;
}

cudaError_t launch_copy_boxes(const BoxCopy* boxes, int n, int es, cudaStream_t s) {
  bool all16 = true;
  for (int i = 0; i < n; i++) all16 = all16 && vec16(boxes[i], es);
  const int f = all16 ? 16 / es : 1;   // elements per copied unit
  for (int b0 = 0; b0 < n; b0 += kMaxBoxes) {
    const int m = n - b0 < kMaxBoxes ? n - b0 : kMaxBoxes;
    BoxList L{};
    long long most = 0;
    for (int i = 0; i < m; i++) {
      BoxCopy b = boxes[b0 + i];
      if (f > 1) {   // geometry in 16-byte units
        b.w /= f;
        b.dpitch /= f;
        b.spitch /= f;
        b.dplane /= f;
        b.splane /= f;
      }
      L.box[i] = b;
      const long long e = (long long)b.w * b.h * b.d;
      if (e >= (1LL << 32)) return cudaErrorInvalidValue;
      most = e > most ? e : most;
    }
    if (most == 0) continue;
    const long long nb = (most + 255) / 256;
    const long long cap = (148LL * 8 + m - 1) / m;   // ~8 CTAs per SM over all boxes
    dim3 grid(unsigned(nb < cap ? nb : cap), unsigned(m));
    if (f > 1) copy_boxes<uint4><<<grid, 256, 0, s>>>(L);
    else if (es == 4) copy_boxes<float><<<grid, 256, 0, s>>>(L);
    else copy_boxes<double><<<grid, 256, 0, s>>>(L);
  }
  return cudaGetLastError();
}

cudaError_t launch_flush(void* buf, long long bytes, unsigned v, cudaStream_t s) {
  long long n = bytes / 16;
  flush_kernel<<<148 * 8, 256, 0, s>>>((uint4*)buf, n, v);
  return cudaGetLastError();
}

}  // namespace kf
