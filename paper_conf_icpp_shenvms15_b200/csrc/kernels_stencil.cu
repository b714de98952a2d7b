// HotSpot thermal stencil (P229-233 Table II "Rodinia [2]", P319: 8192x8192,
// row-wise split) and the MK-Loop residual kernel (BASELINE configs[3]).
//
// hotspot_rows: HBM-bound, 12 algorithmic bytes per cell (read T, read P,
// write T').  A CTA owns a strip of kRows rows x 1024 columns; each thread owns
// 4 adjacent columns (one float4) and walks down the strip keeping the rows
// above / at / below in registers (vertical reuse), exchanging its edge
// columns with the neighbouring lanes by warp shuffles (horizontal reuse); only
// the two warp-edge columns are re-read from L1/L2.  HBM traffic per strip is
// (kRows + 2) rows of T + kRows rows of P + kRows rows of T'.  The update uses
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
constexpr int kRows = 32;              // rows per strip

__device__ __forceinline__ float cell(float c, float n, float s, float w, float e, float p,
                                      const HotCoef& k) {
  const float two = __fadd_rn(c, c);
  const float dv = __fmul_rn(__fsub_rn(__fadd_rn(s, n), two), k.ry1);
  const float dh = __fmul_rn(__fsub_rn(__fadd_rn(e, w), two), k.rx1);
  const float dz = __fmul_rn(__fsub_rn(k.amb, c), k.rz1);
  const float sum = __fadd_rn(__fadd_rn(__fadd_rn(p, dv), dh), dz);
  return __fadd_rn(c, __fmul_rn(k.sdc, sum));
}

// cols % 4 == 0 and 16-B aligned rows.
__global__ void __launch_bounds__(kThreads) hotspot_vec(const float* __restrict__ tin,
                                                        const float* __restrict__ pw,
                                                        float* __restrict__ tout, int64_t rows,
                                                        int64_t cols, int64_t r0, int64_t r1,
                                                        HotCoef k) {
  const int64_t x0 = ((int64_t)blockIdx.x * kThreads + threadIdx.x) * 4;
  const int64_t ys = r0 + (int64_t)blockIdx.y * kRows;
  const int64_t ye = min(ys + kRows, r1);
  const int lane = threadIdx.x & 31;
  const bool active = x0 < cols;
  const int64_t xs = active ? x0 : 0;  // inactive lanes still join the shuffles

  auto ld4 = [&](int64_t y) -> float4 { return *reinterpret_cast<const float4*>(tin + y * cols + xs); };
  float4 up = ld4(ys > 0 ? ys - 1 : ys);
  float4 cu = ld4(ys);
  for (int64_t y = ys; y < ye; ++y) {
    const float4 dn = ld4(y + 1 < rows ? y + 1 : y);
    const float4 p = __ldcs(reinterpret_cast<const float4*>(pw + y * cols + xs));
    // west neighbour of column x0 and east neighbour of column x0+3
    float w = __shfl_up_sync(0xffffffffu, cu.w, 1);
    float e = __shfl_down_sync(0xffffffffu, cu.x, 1);
    if (lane == 0) w = (x0 > 0 && active) ? tin[y * cols + x0 - 1] : cu.x;
    if (lane == 31) e = (x0 + 4 < cols && active) ? tin[y * cols + x0 + 4] : cu.w;
    if (x0 == 0) w = cu.x;               // chip edge: neighbour = the cell itself
    if (x0 + 4 >= cols) e = cu.w;
    const float nn0 = (y > 0) ? up.x : cu.x, nn1 = (y > 0) ? up.y : cu.y;
    const float nn2 = (y > 0) ? up.z : cu.z, nn3 = (y > 0) ? up.w : cu.w;
    const float ss0 = (y + 1 < rows) ? dn.x : cu.x, ss1 = (y + 1 < rows) ? dn.y : cu.y;
    const float ss2 = (y + 1 < rows) ? dn.z : cu.z, ss3 = (y + 1 < rows) ? dn.w : cu.w;
    float4 o;
    o.x = cell(cu.x, nn0, ss0, w, cu.y, p.x, k);
    o.y = cell(cu.y, nn1, ss1, cu.x, cu.z, p.y, k);
    o.z = cell(cu.z, nn2, ss2, cu.y, cu.w, p.z, k);
    o.w = cell(cu.w, nn3, ss3, cu.z, e, p.w, k);
    if (active) __stcs(reinterpret_cast<float4*>(tout + y * cols + x0), o);
    up = cu;
    cu = dn;
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
                         int64_t r0, int64_t r1, HotCoef c, cudaStream_t s, int) {
  if (r1 <= r0) return cudaSuccess;
  const bool vec = (cols % 4 == 0) && (((uintptr_t)tin | (uintptr_t)pw | (uintptr_t)tout) & 15u) == 0;
  if (vec) {
    dim3 grid((unsigned)((cols / 4 + kThreads - 1) / kThreads), (unsigned)((r1 - r0 + kRows - 1) / kRows));
    hotspot_vec<<<grid, kThreads, 0, s>>>(tin, pw, tout, rows, cols, r0, r1, c);
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
