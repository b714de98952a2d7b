// Nbody (P223-227 Table II "Mont-Blanc benchmark suite", P319: 1,048,576
// bodies, iterated -> SK-Loop): all-pairs gravitational acceleration with
// Plummer softening, then a semi-implicit Euler step (CUDA SDK integrator
// [ext]).  Bodies [r0, r1) of this device are advanced; every body's position
// is read (the directory pulls the other devices' ranges = an all-gather).
//
// FP32, FMA-pipe bound: ~20 flop per interaction (3 sub, 3 FMA for r^2,
// rsqrt, 3 mul, 3 FMA).  Each thread owns one body; the CTA stages tiles of
// 256 positions in shared memory and every thread sweeps them in ascending j,
// so a body's sum has the same order for any partitioning (bit-identical
// across strategies and device counts).
#include "kernels.h"

namespace mm {

namespace {

constexpr int kTile = 256;

__global__ void __launch_bounds__(kTile) nbody_rows(const float4* __restrict__ pin, const float4* __restrict__ vin,
                                                    float4* __restrict__ pout, float4* __restrict__ vout, int64_t n,
                                                    int64_t r0, int64_t r1, float dt, float eps2) {
  __shared__ float4 sp[kTile];
  const int64_t i = r0 + (int64_t)blockIdx.x * kTile + threadIdx.x;
  const bool live = i < r1;
  const float4 pi = live ? pin[i] : make_float4(0.f, 0.f, 0.f, 0.f);
  float ax = 0.f, ay = 0.f, az = 0.f;
  for (int64_t j0 = 0; j0 < n; j0 += kTile) {
    const int64_t j = j0 + threadIdx.x;
    sp[threadIdx.x] = j < n ? pin[j] : make_float4(0.f, 0.f, 0.f, 0.f);   // m = 0 pads
    __syncthreads();
    const int m = n - j0 < kTile ? (int)(n - j0) : kTile;
#pragma unroll 8
    for (int q = 0; q < m; ++q) {
      const float4 pj = sp[q];
      const float dx = pj.x - pi.x, dy = pj.y - pi.y, dz = pj.z - pi.z;
      const float d2 = fmaf(dx, dx, fmaf(dy, dy, fmaf(dz, dz, eps2)));
      const float inv = rsqrtf(d2);
      const float s = pj.w * inv * inv * inv;
      ax = fmaf(dx, s, ax);
      ay = fmaf(dy, s, ay);
      az = fmaf(dz, s, az);
    }
    __syncthreads();
  }
  if (live) {
    const float4 v = vin[i];
    const float4 vn = make_float4(fmaf(ax, dt, v.x), fmaf(ay, dt, v.y), fmaf(az, dt, v.z), v.w);
    vout[i] = vn;
    pout[i] = make_float4(fmaf(vn.x, dt, pi.x), fmaf(vn.y, dt, pi.y), fmaf(vn.z, dt, pi.z), pi.w);
  }
}

}  // namespace

cudaError_t nbody_rows_launch(const float* pin, const float* vin, float* pout, float* vout, int64_t n, int64_t r0,
                              int64_t r1, float dt, float eps2, cudaStream_t s) {
  if (r1 <= r0) return cudaSuccess;
  if ((((uintptr_t)pin | (uintptr_t)vin | (uintptr_t)pout | (uintptr_t)vout) & 15u) != 0) return cudaErrorInvalidValue;
  nbody_rows<<<(unsigned)((r1 - r0 + kTile - 1) / kTile), kTile, 0, s>>>(
      reinterpret_cast<const float4*>(pin), reinterpret_cast<const float4*>(vin), reinterpret_cast<float4*>(pout),
      reinterpret_cast<float4*>(vout), n, r0, r1, dt, eps2);
  return cudaGetLastError();
}

}  // namespace mm
