// HotSpot thermal stencil (P229-233 Table II "Rodinia [2]", P319: 8192x8192,
// row-wise split) and the MK-Loop residual kernel (BASELINE configs[3]).
//
// hotspot_rows: HBM-bound, 12 algorithmic bytes per cell (read T, read P,
// write T').  Tiles of kH rows x 1024 columns; every thread batches all its
// loads before computing (see hotspot_vec).  The update uses
// round-to-nearest intrinsics in the oracle's operation order (R16), so the
// result is bit-identical to oracle/numeric.c.
//
// row_residual: rowsum[y] = sum_x ((double)t1 - (double)t0)^2 — one CTA per
// row, FP64 accumulation, fixed shuffle tree (deterministic and independent of
// the partitioning).
#include "kernels.h"

namespace mm {

namespace {

constexpr int kThreads = 256;          // 1024 columns per CTA

__device__ __forceinline__ float cell(float c, float n, float s, float w, float e, float p,
                                      const HotCoef& k) {
  const float two = __fadd_rn(c, c);
  const float dv = __fmul_rn(__fsub_rn(__fadd_rn(s, n), two), k.ry1);
  const float dh = __fmul_rn(__fsub_rn(__fadd_rn(e, w), two), k.rx1);
  const float dz = __fmul_rn(__fsub_rn(k.amb, c), k.rz1);
  const float sum = __fadd_rn(__fadd_rn(__fadd_rn(p, dv), dh), dz);
  return __fadd_rn(c, __fmul_rn(k.sdc, sum));
}

// cols % 4 == 0, 16-B aligned rows.  A CTA owns a tile of kH rows x 1024
// columns of [r0, r1); each thread owns one float4 column group and issues
// ALL its loads first — kH+2 rows of T (rows above/below included) and kH rows
// of P, plus the warp-edge scalars — so each thread has 2kH+2 independent
// 16-B loads in flight, then computes the kH rows from registers (vertical
// reuse) and warp shuffles (horizontal reuse).  Measured on B200
// (tools/hotspot_variants.cu): 6.89 TB/s at 8192^2 and 7.13 TB/s at 16384^2,
// vs 6.13 TB/s for a row-walking strip with one row of prefetch and 4.79 TB/s
// for a single-wave TMA (cp.async.bulk + mbarrier) ring — the halo rows of
// neighbouring tiles are L2 hits, so deep MLP beats smem staging here.
constexpr int kH = 4;

__global__ void __launch_bounds__(kThreads) hotspot_vec(const float* __restrict__ tin,
                                                        const float* __restrict__ pw,
                                                        float* __restrict__ tout, int64_t rows,
                                                        int64_t cols, int64_t r0, int64_t r1,
                                                        HotCoef k, int64_t ncb) {
  const int lane = threadIdx.x & 31;
  const int64_t cb = blockIdx.x % ncb, st = blockIdx.x / ncb;
  const int64_t x0 = (cb * kThreads + threadIdx.x) * 4;
  const int64_t ys = r0 + st * kH;
  const bool active = x0 < cols;
  const int64_t xs = active ? x0 : 0;  // inactive lanes still join the shuffles
  const bool wl = lane == 0 && active && x0 > 0;
  const bool el = lane == 31 && active && x0 + 4 < cols;
  float4 T[kH + 2], P[kH];
  float W[kH], E[kH];
#pragma unroll
  for (int j = 0; j < kH + 2; ++j) {
    int64_t y = ys - 1 + j;
    y = y < 0 ? 0 : (y >= rows ? rows - 1 : y);
    T[j] = *reinterpret_cast<const float4*>(tin + y * cols + xs);
  }
#pragma unroll
  for (int j = 0; j < kH; ++j) {
    int64_t y = ys + j;
    y = y >= rows ? rows - 1 : y;
    P[j] = __ldcs(reinterpret_cast<const float4*>(pw + y * cols + xs));
    W[j] = wl ? tin[y * cols + x0 - 1] : 0.f;
    E[j] = el ? tin[y * cols + x0 + 4] : 0.f;
  }
#pragma unroll
  for (int j = 0; j < kH; ++j) {
    const int64_t y = ys + j;
    if (y >= r1) break;
    const float4 up = T[j], cu = T[j + 1], dn = T[j + 2], p = P[j];
    float w = __shfl_up_sync(0xffffffffu, cu.w, 1);
    float e = __shfl_down_sync(0xffffffffu, cu.x, 1);
    if (lane == 0) w = wl ? W[j] : cu.x;
    if (lane == 31) e = el ? E[j] : cu.w;
    if (x0 == 0) w = cu.x;               // chip edge: neighbour = the cell itself
    if (x0 + 4 >= cols) e = cu.w;
    const bool top = y > 0, bot = y + 1 < rows;
    float4 o;
    o.x = cell(cu.x, top ? up.x : cu.x, bot ? dn.x : cu.x, w, cu.y, p.x, k);
    o.y = cell(cu.y, top ? up.y : cu.y, bot ? dn.y : cu.y, cu.x, cu.z, p.y, k);
    o.z = cell(cu.z, top ? up.z : cu.z, bot ? dn.z : cu.z, cu.y, cu.w, p.z, k);
    o.w = cell(cu.w, top ? up.w : cu.w, bot ? dn.w : cu.w, cu.z, e, p.w, k);
    if (active) __stcs(reinterpret_cast<float4*>(tout + y * cols + x0), o);
  }
}

// Generic shapes: one thread per cell.
__global__ void hotspot_scalar(const float* __restrict__ tin, const float* __restrict__ pw,
                               float* __restrict__ tout, int64_t rows, int64_t cols, int64_t r0,
                               int64_t r1, HotCoef k) {
  const int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int64_t n = (r1 - r0) * cols;
  if (idx >= n) return;
  const int64_t y = r0 + idx / cols, x = idx % cols;
  const float c = tin[y * cols + x];
  const float nn = y > 0 ? tin[(y - 1) * cols + x] : c;
  const float ss = y < rows - 1 ? tin[(y + 1) * cols + x] : c;
  const float w = x > 0 ? tin[y * cols + x - 1] : c;
  const float e = x < cols - 1 ? tin[y * cols + x + 1] : c;
  tout[y * cols + x] = cell(c, nn, ss, w, e, pw[y * cols + x], k);
}

__global__ void __launch_bounds__(kThreads) residual_rows(const float* __restrict__ t0,
                                                          const float* __restrict__ t1,
                                                          double* __restrict__ rowsum, int64_t cols,
                                                          int64_t r0) {
  const int64_t y = r0 + blockIdx.x;
  const float* a = t0 + y * cols;
  const float* b = t1 + y * cols;
  double acc = 0.0;
  if ((cols & 3) == 0) {
    const int64_t n4 = cols / 4;
    for (int64_t i = threadIdx.x; i < n4; i += kThreads) {
      const float4 u = __ldcs(reinterpret_cast<const float4*>(a) + i);
      const float4 v = __ldcs(reinterpret_cast<const float4*>(b) + i);
      double d;
      d = (double)v.x - (double)u.x; acc = fma(d, d, acc);
      d = (double)v.y - (double)u.y; acc = fma(d, d, acc);
      d = (double)v.z - (double)u.z; acc = fma(d, d, acc);
      d = (double)v.w - (double)u.w; acc = fma(d, d, acc);
    }
  } else {
    for (int64_t i = threadIdx.x; i < cols; i += kThreads) {
      const double d = (double)b[i] - (double)a[i];
      acc = fma(d, d, acc);
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
  __shared__ double part[kThreads / 32];
  if ((threadIdx.x & 31) == 0) part[threadIdx.x >> 5] = acc;
  __syncthreads();
  if (threadIdx.x == 0) {
    double s = 0.0;
#pragma unroll
    for (int i = 0; i < kThreads / 32; ++i) s += part[i];
    rowsum[y] = s;
  }
}

}  // namespace

cudaError_t hotspot_rows(const float* tin, const float* pw, float* tout, int64_t rows, int64_t cols,
                         int64_t r0, int64_t r1, HotCoef c, cudaStream_t s, int sms) {
  if (r1 <= r0) return cudaSuccess;
  const bool vec = (cols % 4 == 0) && (((uintptr_t)tin | (uintptr_t)pw | (uintptr_t)tout) & 15u) == 0;
  if (vec) {
    const int64_t ncb = (cols / 4 + kThreads - 1) / kThreads;
    const int64_t tiles = ncb * ((r1 - r0 + kH - 1) / kH);
    hotspot_vec<<<(unsigned)tiles, kThreads, 0, s>>>(tin, pw, tout, rows, cols, r0, r1, c, ncb);
  } else {
    const int64_t n = (r1 - r0) * cols;
    hotspot_scalar<<<(unsigned)((n + 255) / 256), 256, 0, s>>>(tin, pw, tout, rows, cols, r0, r1, c);
  }
  return cudaGetLastError();
}

cudaError_t row_residual(const float* t0, const float* t1, double* rowsum, int64_t cols, int64_t r0,
                         int64_t r1, cudaStream_t s, int) {
  if (r1 <= r0) return cudaSuccess;
  residual_rows<<<(unsigned)(r1 - r0), kThreads, 0, s>>>(t0, t1, rowsum, cols, r0);
  return cudaGetLastError();
}

}  // namespace mm
