// Nbody (P223-227 Table II "Mont-Blanc benchmark suite", P319: 1,048,576
// bodies, iterated -> SK-Loop): all-pairs gravitational acceleration with
// Plummer softening, then a semi-implicit Euler step (CUDA SDK integrator
// [ext]).  Bodies [r0, r1) of this device are advanced; every body's position
// is read (the directory pulls the other devices' ranges = an all-gather).
//
// FP32-pipe bound: 20 flop per interaction by the usual count; the kernel
// issues 12 FP32 lane-ops (3 sub, 3 FMA for r^2, 3 mul for m/r^3, 3 FMA into
// the sum) + 1 MUFU.RSQ.  Each thread owns TWO bodies (i and i + kTile of the
// CTA's 2*kTile block) held in the two lanes of f32x2 registers, so every
// FP32 instruction is a packed FFMA2/FADD2/FMUL2 (half the issue slots; the
// FP32 lane rate is unchanged, tools/pipe_rates.cu) and every shared-memory
// position load feeds two interactions.  rsqrt.approx.ftz = the bare MUFU.RSQ
// (d2 >= eps2 >= FLT_MIN is normal, so it equals rsqrtf, without its
// denormal scaling).  The CTA stages tiles of kTile positions in shared memory
// and every body sweeps them in ascending j, so a body's sum has the same
// order for any partitioning (bit-identical across strategies and device
// counts).  Ceiling: 128 FP32 lanes/clk/SM / 12 = 10.67 interactions/clk/SM.
#include "kernels.h"

namespace mm {

namespace {

constexpr int kTile = 256;

struct f2 {
  unsigned long long v;
};
__device__ __forceinline__ f2 pack(float a, float b) {
  f2 r;
  asm("mov.b64 %0, {%1, %2};" : "=l"(r.v) : "f"(a), "f"(b));
  return r;
}
__device__ __forceinline__ void unpack(f2 x, float& a, float& b) { asm("mov.b64 {%0, %1}, %2;" : "=f"(a), "=f"(b) : "l"(x.v)); }
__device__ __forceinline__ f2 sub2(f2 a, f2 b) {
  f2 r;
  asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(r.v) : "l"(a.v), "l"(b.v));
  return r;
}
__device__ __forceinline__ f2 mul2(f2 a, f2 b) {
  f2 r;
  asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(r.v) : "l"(a.v), "l"(b.v));
  return r;
}
__device__ __forceinline__ f2 fma2(f2 a, f2 b, f2 c) {
  f2 r;
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(r.v) : "l"(a.v), "l"(b.v), "l"(c.v));
  return r;
}
__device__ __forceinline__ float rsq(float x) {
  float r;
  asm("rsqrt.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
  return r;
}

// BP f32x2 pairs of bodies per thread (2 * BP bodies: i + kTile * m of the
// CTA's 2 * BP * kTile block): every shared-memory position load feeds 2 * BP
// interactions, and the BP pairs' chains interleave.  BP = 2 (64 registers,
// 4 CTAs per SM) measured equal to BP = 1 (433 ms for 2^20 bodies); BP = 1
// with the compiler free to use 84 registers runs 2 % faster than at 48.
template <int BP>
__global__ void __launch_bounds__(kTile, BP == 2 ? 4 : 1) nbody_rows(const float4* __restrict__ pin, const float4* __restrict__ vin,
                                                    float4* __restrict__ pout, float4* __restrict__ vout, int64_t n,
                                                    int64_t r0, int64_t r1, float dt, float eps2) {
  __shared__ float4 sp[kTile];
  int64_t ib[2 * BP];
  float4 pb[2 * BP];
#pragma unroll
  for (int m = 0; m < 2 * BP; ++m) {
    ib[m] = r0 + (int64_t)blockIdx.x * 2 * BP * kTile + m * kTile + threadIdx.x;
    pb[m] = ib[m] < r1 ? pin[ib[m]] : make_float4(0.f, 0.f, 0.f, 0.f);
  }
  const f2 e2 = pack(eps2, eps2);
  f2 px[BP], py[BP], pz[BP], ax[BP], ay[BP], az[BP];
#pragma unroll
  for (int u = 0; u < BP; ++u) {
    px[u] = pack(pb[2 * u].x, pb[2 * u + 1].x);
    py[u] = pack(pb[2 * u].y, pb[2 * u + 1].y);
    pz[u] = pack(pb[2 * u].z, pb[2 * u + 1].z);
    ax[u] = ay[u] = az[u] = pack(0.f, 0.f);
  }
  for (int64_t j0 = 0; j0 < n; j0 += kTile) {
    const int64_t j = j0 + threadIdx.x;
    sp[threadIdx.x] = j < n ? pin[j] : make_float4(0.f, 0.f, 0.f, 0.f);   // m = 0 pads
    __syncthreads();
    const int m = n - j0 < kTile ? (int)(n - j0) : kTile;
#pragma unroll 8
    for (int q = 0; q < m; ++q) {
      const float4 pj = sp[q];
#pragma unroll
      for (int u = 0; u < BP; ++u) {
        const f2 dx = sub2(pack(pj.x, pj.x), px[u]), dy = sub2(pack(pj.y, pj.y), py[u]),
                 dz = sub2(pack(pj.z, pj.z), pz[u]);
        const f2 d2 = fma2(dx, dx, fma2(dy, dy, fma2(dz, dz, e2)));
        float d2a, d2b;
        unpack(d2, d2a, d2b);
        const f2 inv = pack(rsq(d2a), rsq(d2b));
        const f2 s = mul2(mul2(mul2(pack(pj.w, pj.w), inv), inv), inv);
        ax[u] = fma2(dx, s, ax[u]);
        ay[u] = fma2(dy, s, ay[u]);
        az[u] = fma2(dz, s, az[u]);
      }
    }
    __syncthreads();
  }
#pragma unroll
  for (int u = 0; u < BP; ++u) {
    float axv[2], ayv[2], azv[2];
    unpack(ax[u], axv[0], axv[1]);
    unpack(ay[u], ayv[0], ayv[1]);
    unpack(az[u], azv[0], azv[1]);
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      const int mm = 2 * u + h;
      if (ib[mm] < r1) {
        const float4 v = vin[ib[mm]];
        const float4 vn = make_float4(fmaf(axv[h], dt, v.x), fmaf(ayv[h], dt, v.y), fmaf(azv[h], dt, v.z), v.w);
        vout[ib[mm]] = vn;
        const float4 p0 = pb[mm];
        pout[ib[mm]] = make_float4(fmaf(vn.x, dt, p0.x), fmaf(vn.y, dt, p0.y), fmaf(vn.z, dt, p0.z), p0.w);
      }
    }
  }
}

}  // namespace

cudaError_t nbody_rows_launch(const float* pin, const float* vin, float* pout, float* vout, int64_t n, int64_t r0,
                              int64_t r1, float dt, float eps2, cudaStream_t s) {
  if (r1 <= r0) return cudaSuccess;
  if ((((uintptr_t)pin | (uintptr_t)vin | (uintptr_t)pout | (uintptr_t)vout) & 15u) != 0) return cudaErrorInvalidValue;
  if (!(eps2 >= 1.17549435e-38f)) return cudaErrorInvalidValue;   // normal eps^2 > 0 (rsqrt.ftz)
  note_launch();
  nbody_rows<1><<<(unsigned)((r1 - r0 + 2 * kTile - 1) / (2 * kTile)), kTile, 0, s>>>(
      reinterpret_cast<const float4*>(pin), reinterpret_cast<const float4*>(vin), reinterpret_cast<float4*>(pout),
      reinterpret_cast<float4*>(vout), n, r0, r1, dt, eps2);
  return cudaGetLastError();
}

}  // namespace mm
