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

__global__ void __launch_bounds__(kTile) nbody_rows(const float4* __restrict__ pin, const float4* __restrict__ vin,
                                                    float4* __restrict__ pout, float4* __restrict__ vout, int64_t n,
                                                    int64_t r0, int64_t r1, float dt, float eps2) {
  __shared__ float4 sp[kTile];
  const int64_t ia = r0 + (int64_t)blockIdx.x * 2 * kTile + threadIdx.x, ib = ia + kTile;
  const bool la = ia < r1, lb = ib < r1;
  const float4 pa = la ? pin[ia] : make_float4(0.f, 0.f, 0.f, 0.f);
  const float4 pb = lb ? pin[ib] : make_float4(0.f, 0.f, 0.f, 0.f);
  const f2 px = pack(pa.x, pb.x), py = pack(pa.y, pb.y), pz = pack(pa.z, pb.z), e2 = pack(eps2, eps2);
  f2 ax = pack(0.f, 0.f), ay = ax, az = ax;
  for (int64_t j0 = 0; j0 < n; j0 += kTile) {
    const int64_t j = j0 + threadIdx.x;
    sp[threadIdx.x] = j < n ? pin[j] : make_float4(0.f, 0.f, 0.f, 0.f);   // m = 0 pads
    __syncthreads();
    const int m = n - j0 < kTile ? (int)(n - j0) : kTile;
#pragma unroll 8
    for (int q = 0; q < m; ++q) {
      const float4 pj = sp[q];
      const f2 dx = sub2(pack(pj.x, pj.x), px), dy = sub2(pack(pj.y, pj.y), py), dz = sub2(pack(pj.z, pj.z), pz);
      const f2 d2 = fma2(dx, dx, fma2(dy, dy, fma2(dz, dz, e2)));
      float d2a, d2b;
      unpack(d2, d2a, d2b);
      const f2 inv = pack(rsq(d2a), rsq(d2b));
      const f2 s = mul2(mul2(mul2(pack(pj.w, pj.w), inv), inv), inv);
      ax = fma2(dx, s, ax);
      ay = fma2(dy, s, ay);
      az = fma2(dz, s, az);
    }
    __syncthreads();
  }
  float axa, axb, aya, ayb, aza, azb;
  unpack(ax, axa, axb);
  unpack(ay, aya, ayb);
  unpack(az, aza, azb);
  if (la) {
    const float4 v = vin[ia];
    const float4 vn = make_float4(fmaf(axa, dt, v.x), fmaf(aya, dt, v.y), fmaf(aza, dt, v.z), v.w);
    vout[ia] = vn;
    pout[ia] = make_float4(fmaf(vn.x, dt, pa.x), fmaf(vn.y, dt, pa.y), fmaf(vn.z, dt, pa.z), pa.w);
  }
  if (lb) {
    const float4 v = vin[ib];
    const float4 vn = make_float4(fmaf(axb, dt, v.x), fmaf(ayb, dt, v.y), fmaf(azb, dt, v.z), v.w);
    vout[ib] = vn;
    pout[ib] = make_float4(fmaf(vn.x, dt, pb.x), fmaf(vn.y, dt, pb.y), fmaf(vn.z, dt, pb.z), pb.w);
  }
}

}  // namespace

cudaError_t nbody_rows_launch(const float* pin, const float* vin, float* pout, float* vout, int64_t n, int64_t r0,
                              int64_t r1, float dt, float eps2, cudaStream_t s) {
  if (r1 <= r0) return cudaSuccess;
  if ((((uintptr_t)pin | (uintptr_t)vin | (uintptr_t)pout | (uintptr_t)vout) & 15u) != 0) return cudaErrorInvalidValue;
  if (!(eps2 >= 1.17549435e-38f)) return cudaErrorInvalidValue;   // normal eps^2 > 0 (rsqrt.ftz)
  note_launch();
  nbody_rows<<<(unsigned)((r1 - r0 + 2 * kTile - 1) / (2 * kTile)), kTile, 0, s>>>(
      reinterpret_cast<const float4*>(pin), reinterpret_cast<const float4*>(vin), reinterpret_cast<float4*>(pout),
      reinterpret_cast<float4*>(vout), n, r0, r1, dt, eps2);
  return cudaGetLastError();
}

}  // namespace mm
