// Microbenchmark of all-pairs Nbody inner loops (development tool).
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cmath>

constexpr int T = 256;

__global__ void __launch_bounds__(T) v1(const float4* __restrict__ p, float4* __restrict__ acc, int n, float eps2) {
  __shared__ float4 sp[T];
  int i = blockIdx.x * T + threadIdx.x;
  float4 pi = p[i];
  float ax = 0, ay = 0, az = 0;
  for (int j0 = 0; j0 < n; j0 += T) {
    sp[threadIdx.x] = p[j0 + threadIdx.x];
    __syncthreads();
#pragma unroll 8
    for (int q = 0; q < T; ++q) {
      float4 pj = sp[q];
      float dx = pj.x - pi.x, dy = pj.y - pi.y, dz = pj.z - pi.z;
      float d2 = fmaf(dx, dx, fmaf(dy, dy, fmaf(dz, dz, eps2)));
      float inv = rsqrtf(d2);
      float s = pj.w * inv * inv * inv;
      ax = fmaf(dx, s, ax); ay = fmaf(dy, s, ay); az = fmaf(dz, s, az);
    }
    __syncthreads();
  }
  acc[i] = make_float4(ax, ay, az, 0);
}

// two bodies per thread (i and i + T within the CTA's 2T block), scalar
__global__ void __launch_bounds__(T) v2(const float4* __restrict__ p, float4* __restrict__ acc, int n, float eps2) {
  __shared__ float4 sp[T];
  int i0 = blockIdx.x * 2 * T + threadIdx.x, i1 = i0 + T;
  float4 a = p[i0], b = p[i1];
  float ax = 0, ay = 0, az = 0, bx = 0, by = 0, bz = 0;
  for (int j0 = 0; j0 < n; j0 += T) {
    sp[threadIdx.x] = p[j0 + threadIdx.x];
    __syncthreads();
#pragma unroll 8
    for (int q = 0; q < T; ++q) {
      float4 pj = sp[q];
      {
        float dx = pj.x - a.x, dy = pj.y - a.y, dz = pj.z - a.z;
        float d2 = fmaf(dx, dx, fmaf(dy, dy, fmaf(dz, dz, eps2)));
        float inv = rsqrtf(d2);
        float s = pj.w * inv * inv * inv;
        ax = fmaf(dx, s, ax); ay = fmaf(dy, s, ay); az = fmaf(dz, s, az);
      }
      {
        float dx = pj.x - b.x, dy = pj.y - b.y, dz = pj.z - b.z;
        float d2 = fmaf(dx, dx, fmaf(dy, dy, fmaf(dz, dz, eps2)));
        float inv = rsqrtf(d2);
        float s = pj.w * inv * inv * inv;
        bx = fmaf(dx, s, bx); by = fmaf(dy, s, by); bz = fmaf(dz, s, bz);
      }
    }
    __syncthreads();
  }
  acc[i0] = make_float4(ax, ay, az, 0);
  acc[i1] = make_float4(bx, by, bz, 0);
}

__device__ __forceinline__ float2 sub2(float2 a, float2 b) {
  float2 r;
  asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(*(unsigned long long*)&r) : "l"(*(unsigned long long*)&a), "l"(*(unsigned long long*)&b));
  return r;
}
__device__ __forceinline__ float2 mul2(float2 a, float2 b) {
  float2 r;
  asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(*(unsigned long long*)&r) : "l"(*(unsigned long long*)&a), "l"(*(unsigned long long*)&b));
  return r;
}
__device__ __forceinline__ float2 fma2(float2 a, float2 b, float2 c) {
  float2 r;
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(*(unsigned long long*)&r)
      : "l"(*(unsigned long long*)&a), "l"(*(unsigned long long*)&b), "l"(*(unsigned long long*)&c));
  return r;
}

// two bodies per thread packed in f32x2 lanes
__global__ void __launch_bounds__(T) v3(const float4* __restrict__ p, float4* __restrict__ acc, int n, float eps2) {
  __shared__ float4 sp[T];
  int i0 = blockIdx.x * 2 * T + threadIdx.x, i1 = i0 + T;
  float4 a = p[i0], b = p[i1];
  float2 px = make_float2(a.x, b.x), py = make_float2(a.y, b.y), pz = make_float2(a.z, b.z);
  float2 e2 = make_float2(eps2, eps2);
  float2 ax = make_float2(0, 0), ay = ax, az = ax;
  for (int j0 = 0; j0 < n; j0 += T) {
    sp[threadIdx.x] = p[j0 + threadIdx.x];
    __syncthreads();
#pragma unroll 8
    for (int q = 0; q < T; ++q) {
      float4 pj = sp[q];
      float2 dx = sub2(make_float2(pj.x, pj.x), px);
      float2 dy = sub2(make_float2(pj.y, pj.y), py);
      float2 dz = sub2(make_float2(pj.z, pj.z), pz);
      float2 d2 = fma2(dx, dx, fma2(dy, dy, fma2(dz, dz, e2)));
      float2 inv = make_float2(rsqrtf(d2.x), rsqrtf(d2.y));
      float2 s = mul2(mul2(mul2(make_float2(pj.w, pj.w), inv), inv), inv);
      ax = fma2(dx, s, ax); ay = fma2(dy, s, ay); az = fma2(dz, s, az);
    }
    __syncthreads();
  }
  acc[i0] = make_float4(ax.x, ay.x, az.x, 0);
  acc[i1] = make_float4(ax.y, ay.y, az.y, 0);
}

// four bodies per thread packed in two f32x2 groups
__global__ void __launch_bounds__(T) v4(const float4* __restrict__ p, float4* __restrict__ acc, int n, float eps2) {
  __shared__ float4 sp[T];
  int i0 = blockIdx.x * 4 * T + threadIdx.x;
  float2 px[2], py[2], pz[2], ax[2], ay[2], az[2];
  for (int g = 0; g < 2; ++g) {
    float4 a = p[i0 + (2 * g) * T], b = p[i0 + (2 * g + 1) * T];
    px[g] = make_float2(a.x, b.x); py[g] = make_float2(a.y, b.y); pz[g] = make_float2(a.z, b.z);
    ax[g] = ay[g] = az[g] = make_float2(0, 0);
  }
  float2 e2 = make_float2(eps2, eps2);
  for (int j0 = 0; j0 < n; j0 += T) {
    sp[threadIdx.x] = p[j0 + threadIdx.x];
    __syncthreads();
#pragma unroll 4
    for (int q = 0; q < T; ++q) {
      float4 pj = sp[q];
#pragma unroll
      for (int g = 0; g < 2; ++g) {
        float2 dx = sub2(make_float2(pj.x, pj.x), px[g]);
        float2 dy = sub2(make_float2(pj.y, pj.y), py[g]);
        float2 dz = sub2(make_float2(pj.z, pj.z), pz[g]);
        float2 d2 = fma2(dx, dx, fma2(dy, dy, fma2(dz, dz, e2)));
        float2 inv = make_float2(rsqrtf(d2.x), rsqrtf(d2.y));
        float2 s = mul2(mul2(mul2(make_float2(pj.w, pj.w), inv), inv), inv);
        ax[g] = fma2(dx, s, ax[g]); ay[g] = fma2(dy, s, ay[g]); az[g] = fma2(dz, s, az[g]);
      }
    }
    __syncthreads();
  }
  for (int g = 0; g < 2; ++g) {
    acc[i0 + (2 * g) * T] = make_float4(ax[g].x, ay[g].x, az[g].x, 0);
    acc[i0 + (2 * g + 1) * T] = make_float4(ax[g].y, ay[g].y, az[g].y, 0);
  }
}

__device__ __forceinline__ float rsq(float x) { float r; asm("rsqrt.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x)); return r; }

__global__ void __launch_bounds__(T) v5(const float4* __restrict__ p, float4* __restrict__ acc, int n, float eps2) {
  __shared__ float4 sp[T];
  int i = blockIdx.x * T + threadIdx.x;
  float4 pi = p[i];
  float ax = 0, ay = 0, az = 0;
  for (int j0 = 0; j0 < n; j0 += T) {
    sp[threadIdx.x] = p[j0 + threadIdx.x];
    __syncthreads();
#pragma unroll 8
    for (int q = 0; q < T; ++q) {
      float4 pj = sp[q];
      float dx = pj.x - pi.x, dy = pj.y - pi.y, dz = pj.z - pi.z;
      float d2 = fmaf(dx, dx, fmaf(dy, dy, fmaf(dz, dz, eps2)));
      float inv = rsq(d2);
      float s = pj.w * inv * inv * inv;
      ax = fmaf(dx, s, ax); ay = fmaf(dy, s, ay); az = fmaf(dz, s, az);
    }
    __syncthreads();
  }
  acc[i] = make_float4(ax, ay, az, 0);
}

__global__ void __launch_bounds__(T) v6(const float4* __restrict__ p, float4* __restrict__ acc, int n, float eps2) {
  __shared__ float4 sp[T];
  int i0 = blockIdx.x * 2 * T + threadIdx.x, i1 = i0 + T;
  float4 a = p[i0], b = p[i1];
  float2 px = make_float2(a.x, b.x), py = make_float2(a.y, b.y), pz = make_float2(a.z, b.z);
  float2 e2 = make_float2(eps2, eps2);
  float2 ax = make_float2(0, 0), ay = ax, az = ax;
  for (int j0 = 0; j0 < n; j0 += T) {
    sp[threadIdx.x] = p[j0 + threadIdx.x];
    __syncthreads();
#pragma unroll 8
    for (int q = 0; q < T; ++q) {
      float4 pj = sp[q];
      float2 dx = sub2(make_float2(pj.x, pj.x), px);
      float2 dy = sub2(make_float2(pj.y, pj.y), py);
      float2 dz = sub2(make_float2(pj.z, pj.z), pz);
      float2 d2 = fma2(dx, dx, fma2(dy, dy, fma2(dz, dz, e2)));
      float2 inv = make_float2(rsq(d2.x), rsq(d2.y));
      float2 s = mul2(mul2(mul2(make_float2(pj.w, pj.w), inv), inv), inv);
      ax = fma2(dx, s, ax); ay = fma2(dy, s, ay); az = fma2(dz, s, az);
    }
    __syncthreads();
  }
  acc[i0] = make_float4(ax.x, ay.x, az.x, 0);
  acc[i1] = make_float4(ax.y, ay.y, az.y, 0);
}

int main() {
  const int n = 1 << 20;
  std::vector<float4> h(n);
  uint64_t s = 1;
  auto rnd = [&] { s = s * 6364136223846793005ULL + 1442695040888963407ULL; return (float)((s >> 40) * 0x1p-24); };
  for (auto& q : h) q = make_float4(2 * rnd() - 1, 2 * rnd() - 1, 2 * rnd() - 1, 0.5f + 0.5f * rnd());
  float4 *p, *a;
  cudaMalloc(&p, n * 16); cudaMalloc(&a, n * 16);
  cudaMemcpy(p, h.data(), n * 16, cudaMemcpyHostToDevice);
  std::vector<float4> ref(n), out(n);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  auto bench = [&](const char* name, auto launch) {
    launch();
    cudaDeviceSynchronize();
    cudaEventRecord(e0);
    for (int r = 0; r < 5; ++r) launch();
    cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1); ms /= 5;
    cudaMemcpy(out.data(), a, n * 16, cudaMemcpyDeviceToHost);
    bool first = ref[0].x == 0 && ref[0].y == 0;
    if (first) ref = out;
    size_t diff = 0;
    for (int i = 0; i < n; ++i) diff += memcmp(&ref[i], &out[i], 12) != 0;
    printf("%-28s %8.3f ms  %6.2f TF/s (20 flop/int)  bitdiff=%zu err=%s\n", name, ms, 20.0 * n * n / (ms * 1e-3) / 1e12,
           diff, cudaGetErrorString(cudaGetLastError()));
  };
  for (auto& q : ref) q = make_float4(0, 0, 0, 0);
  bench("v1 1 body/thread", [&] { v1<<<n / T, T>>>(p, a, n, 1e-4f); });
  bench("v2 2 bodies scalar", [&] { v2<<<n / (2 * T), T>>>(p, a, n, 1e-4f); });
  bench("v3 2 bodies f32x2", [&] { v3<<<n / (2 * T), T>>>(p, a, n, 1e-4f); });
  bench("v4 4 bodies f32x2", [&] { v4<<<n / (4 * T), T>>>(p, a, n, 1e-4f); });
  bench("v5 1 body ftz rsqrt", [&] { v5<<<n / T, T>>>(p, a, n, 1e-4f); });
  bench("v6 2 bodies f32x2 ftz", [&] { v6<<<n / (2 * T), T>>>(p, a, n, 1e-4f); });
  bench("v1 again", [&] { v1<<<n / T, T>>>(p, a, n, 1e-4f); });
  return 0;
}
