// Measured issue rates of the pipes the Nbody kernel uses (development tool):
// MUFU.RSQ, FFMA, FFMA2 (f32x2) per SM per clock, on 148 SMs.
#include <cuda_runtime.h>
#include <cstdio>

__global__ void k_rsq(float* out, int iters) {
  float x[8];
  for (int u = 0; u < 8; ++u) x[u] = 1.0f + threadIdx.x * 1e-3f + u;
  for (int i = 0; i < iters; ++i)
#pragma unroll
    for (int u = 0; u < 8; ++u) asm volatile("rsqrt.approx.ftz.f32 %0, %0;" : "+f"(x[u]));
  float s = 0; for (int u = 0; u < 8; ++u) s += x[u];
  if (s == 12345.f) out[0] = s;
}
__global__ void k_ffma(float* out, int iters) {
  float x[8];
  float a = 1.0001f + threadIdx.x * 1e-7f, b = 1e-7f;
  for (int u = 0; u < 8; ++u) x[u] = threadIdx.x * 1e-3f + u;
  for (int i = 0; i < iters; ++i)
#pragma unroll
    for (int u = 0; u < 8; ++u) asm volatile("fma.rn.f32 %0, %0, %1, %2;" : "+f"(x[u]) : "f"(a), "f"(b));
  float s = 0; for (int u = 0; u < 8; ++u) s += x[u];
  if (s == 12345.f) out[0] = s;
}
__global__ void k_ffma2(float* out, int iters) {
  unsigned long long x[8];
  float2 av = make_float2(1.0001f, 1.0002f), bv = make_float2(1e-7f, 2e-7f);
  unsigned long long a = *(unsigned long long*)&av, b = *(unsigned long long*)&bv;
  for (int u = 0; u < 8; ++u) { float2 t = make_float2(threadIdx.x * 1e-3f + u, u); x[u] = *(unsigned long long*)&t; }
  for (int i = 0; i < iters; ++i)
#pragma unroll
    for (int u = 0; u < 8; ++u) asm volatile("fma.rn.f32x2 %0, %0, %1, %2;" : "+l"(x[u]) : "l"(a), "l"(b));
  float s = 0; for (int u = 0; u < 8; ++u) { float2 t = *(float2*)&x[u]; s += t.x + t.y; }
  if (s == 12345.f) out[0] = s;
}
__global__ void k_mix(float* out, int iters) {   // 1 rsqrt + 6 ffma2 (the Nbody v6 ratio)
  float r[4]; unsigned long long x[8];
  float2 av = make_float2(1.0001f, 1.0002f), bv = make_float2(1e-7f, 2e-7f);
  unsigned long long a = *(unsigned long long*)&av, b = *(unsigned long long*)&bv;
  for (int u = 0; u < 8; ++u) { float2 t = make_float2(threadIdx.x * 1e-3f + u, u); x[u] = *(unsigned long long*)&t; }
  for (int u = 0; u < 4; ++u) r[u] = 1.0f + u + threadIdx.x;
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int u = 0; u < 4; ++u) asm volatile("rsqrt.approx.ftz.f32 %0, %0;" : "+f"(r[u]));
#pragma unroll
    for (int v = 0; v < 3; ++v)
#pragma unroll
      for (int u = 0; u < 8; ++u) asm volatile("fma.rn.f32x2 %0, %0, %1, %2;" : "+l"(x[u]) : "l"(a), "l"(b));
  }
  float s = r[0] + r[1] + r[2] + r[3]; for (int u = 0; u < 8; ++u) { float2 t = *(float2*)&x[u]; s += t.x + t.y; }
  if (s == 12345.f) out[0] = s;
}

int main() {
  float* o; cudaMalloc(&o, 4);
  int sm; cudaDeviceGetAttribute(&sm, cudaDevAttrMultiProcessorCount, 0);
  const int blocks = sm * 8, thr = 256, iters = 20000;
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  auto run = [&](const char* name, void (*k)(float*, int), double ops_per_iter_thread) {
    k<<<blocks, thr>>>(o, 100);
    cudaEventRecord(a); k<<<blocks, thr>>>(o, iters); cudaEventRecord(b); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b);
    double ops = ops_per_iter_thread * iters * (double)blocks * thr;
    printf("%-10s %.3f ms  %.3e lane-ops/s  = %.2f per SM per ns\n", name, ms, ops / (ms * 1e-3), ops / (ms * 1e-3) / sm / 1e9);
  };
  run("rsqrt", k_rsq, 8);
  run("ffma", k_ffma, 8);
  run("ffma2", k_ffma2, 8);
  run("mix 1:6", k_mix, 4);   // counted in rsqrt (4 per iter per thread; 24 ffma2)
  return 0;
}
