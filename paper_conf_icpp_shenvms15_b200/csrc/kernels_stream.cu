// STREAM copy / scale / add / triad (P235-245 Table II, P473; McCalpin [22]).
//
// HBM-bound: 8 / 8 / 12 / 12 algorithmic bytes per element.  Each thread moves
// kUnroll float4 per array with all loads issued before any store (>= 4
// independent 16-B loads in flight per thread, SURVEY §8(a) requirement).
// Loads use the streaming (.cs, evict-first) cache policy for inputs that are
// read once per kernel; stores use .cs as well so the 1 GiB arrays do not
// thrash L2 for the next kernel's reads.  Arithmetic is written with explicit
// round-to-nearest intrinsics so the result equals the FP32 oracle bit for bit
// (no FMA contraction except the triad's single fused multiply-add, R14).
#include "kernels.h"

namespace mm {

namespace {

constexpr int kThreads = 256;
constexpr int kUnroll = 4;
constexpr int64_t kVecPerBlock = (int64_t)kThreads * kUnroll;

enum { OP_COPY = 0, OP_SCALE = 1, OP_ADD = 2, OP_TRIAD = 3 };

__device__ __forceinline__ float4 ld_cs(const float4* p) { return __ldcs(p); }
__device__ __forceinline__ void st_cs(float4* p, float4 v) { __stcs(p, v); }

template <int OP>
__device__ __forceinline__ float apply(float x, float y, float q) {
  if (OP == OP_COPY) return x;
  if (OP == OP_SCALE) return __fmul_rn(q, x);
  if (OP == OP_ADD) return __fadd_rn(x, y);
  return __fmaf_rn(q, y, x);  // triad: a = b + q*c with x=b, y=c
}

template <int OP>
__device__ __forceinline__ float4 apply4(float4 x, float4 y, float q) {
  return make_float4(apply<OP>(x.x, y.x, q), apply<OP>(x.y, y.y, q), apply<OP>(x.z, y.z, q),
                     apply<OP>(x.w, y.w, q));
}

// z[i] = op(x[i], y[i]) over float4 indices [0, n4) of pointers already
// offset to the range start.
template <int OP>
__global__ void __launch_bounds__(kThreads) stream_vec(const float4* __restrict__ x,
                                                       const float4* __restrict__ y,
                                                       float4* __restrict__ z, int64_t n4, float q) {
  const int64_t base = (int64_t)blockIdx.x * kVecPerBlock + threadIdx.x;
  constexpr bool two = (OP == OP_ADD || OP == OP_TRIAD);
  float4 vx[kUnroll], vy[kUnroll];
  if (base + (kUnroll - 1) * kThreads < n4) {
#pragma unroll
    for (int u = 0; u < kUnroll; ++u) {
      vx[u] = ld_cs(x + base + u * kThreads);
      if (two) vy[u] = ld_cs(y + base + u * kThreads);
    }
#pragma unroll
    for (int u = 0; u < kUnroll; ++u) st_cs(z + base + u * kThreads, apply4<OP>(vx[u], two ? vy[u] : vx[u], q));
  } else {
#pragma unroll
    for (int u = 0; u < kUnroll; ++u) {
      const int64_t i = base + u * kThreads;
      if (i < n4) {
        float4 a = ld_cs(x + i);
        float4 b = two ? ld_cs(y + i) : a;
        st_cs(z + i, apply4<OP>(a, b, q));
      }
    }
  }
}

template <int OP>
__global__ void stream_scalar(const float* __restrict__ x, const float* __restrict__ y,
                              float* __restrict__ z, int64_t n, float q) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) {
    const float a = x[i];
    const float b = (OP == OP_ADD || OP == OP_TRIAD) ? y[i] : a;
    z[i] = apply<OP>(a, b, q);
  }
}

template <int OP>
cudaError_t run(const float* x, const float* y, float* z, float q, int64_t lo, int64_t hi,
                cudaStream_t s) {
  if (hi <= lo) return cudaSuccess;
  const float* xs = x + lo;
  const float* ys = y ? y + lo : nullptr;
  float* zs = z + lo;
  const int64_t n = hi - lo;
  auto aligned = [](const void* p) { return ((uintptr_t)p & 15u) == 0; };
  int64_t done = 0;
  if (aligned(xs) && aligned(zs) && (!ys || aligned(ys))) {
    const int64_t n4 = n / 4;
    if (n4 > 0) {
      const int64_t blocks = (n4 + kVecPerBlock - 1) / kVecPerBlock;
      note_launch();
      stream_vec<OP><<<(unsigned)blocks, kThreads, 0, s>>>(
          reinterpret_cast<const float4*>(xs), reinterpret_cast<const float4*>(ys ? ys : xs),
          reinterpret_cast<float4*>(zs), n4, q);
      done = n4 * 4;
    }
  }
  if (done < n) {
    const int64_t m = n - done;
    note_launch();
    stream_scalar<OP><<<(unsigned)((m + 255) / 256), 256, 0, s>>>(xs + done, ys ? ys + done : xs + done,
                                                                   zs + done, m, q);
  }
  return cudaGetLastError();
}

}  // namespace

cudaError_t stream_copy(const float* a, float* c, int64_t lo, int64_t hi, cudaStream_t s, int) {
  return run<OP_COPY>(a, nullptr, c, 0.f, lo, hi, s);
}
cudaError_t stream_scale(const float* c, float* b, float q, int64_t lo, int64_t hi, cudaStream_t s, int) {
  return run<OP_SCALE>(c, nullptr, b, q, lo, hi, s);
}
cudaError_t stream_add(const float* a, const float* b, float* c, int64_t lo, int64_t hi, cudaStream_t s, int) {
  return run<OP_ADD>(a, b, c, 0.f, lo, hi, s);
}
cudaError_t stream_triad(const float* b, const float* c, float* a, float q, int64_t lo, int64_t hi,
                         cudaStream_t s, int) {
  return run<OP_TRIAD>(b, c, a, q, lo, hi, s);
}

}  // namespace mm
