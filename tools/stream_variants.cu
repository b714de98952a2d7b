// Microbenchmark of STREAM kernel layouts (development tool, not the product).
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>

template <int U, int T, bool TWO, bool CS>
__global__ void __launch_bounds__(T) k_vec(const float4* __restrict__ x, const float4* __restrict__ y,
                                           float4* __restrict__ z, int64_t n4) {
  const int64_t base = (int64_t)blockIdx.x * T * U + threadIdx.x;
  float4 a[U], b[U];
  if (base + (U - 1) * T < n4) {
#pragma unroll
    for (int u = 0; u < U; ++u) {
      a[u] = CS ? __ldcs(x + base + u * T) : x[base + u * T];
      if (TWO) b[u] = CS ? __ldcs(y + base + u * T) : y[base + u * T];
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      float4 o = a[u];
      if (TWO) { o.x += b[u].x; o.y += b[u].y; o.z += b[u].z; o.w += b[u].w; }
      else { o.x *= 3.f; o.y *= 3.f; o.z *= 3.f; o.w *= 3.f; }
      if (CS) __stcs(z + base + u * T, o); else z[base + u * T] = o;
    }
  }
}

template <int U, bool TWO>
__global__ void __launch_bounds__(256) k_persist(const float4* __restrict__ x, const float4* __restrict__ y,
                                                 float4* __restrict__ z, int64_t n4) {
  for (int64_t base = (int64_t)blockIdx.x * 256 * U + threadIdx.x; base < n4; base += (int64_t)gridDim.x * 256 * U) {
    float4 a[U], b[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      a[u] = __ldcs(x + base + u * 256);
      if (TWO) b[u] = __ldcs(y + base + u * 256);
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      float4 o = a[u];
      if (TWO) { o.x += b[u].x; o.y += b[u].y; o.z += b[u].z; o.w += b[u].w; }
      else { o.x *= 3.f; o.y *= 3.f; o.z *= 3.f; o.w *= 3.f; }
      __stcs(z + base + u * 256, o);
    }
  }
}

template <class F>
float timeit(F f, int reps = 20) {
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  for (int i = 0; i < 3; ++i) f();
  cudaEventRecord(a);
  for (int i = 0; i < reps; ++i) f();
  cudaEventRecord(b); cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b);
  return ms / reps;
}

int main() {
  const int64_t n = 1LL << 28, n4 = n / 4;
  float4 *x, *y, *z;
  cudaMalloc(&x, n * 4); cudaMalloc(&y, n * 4); cudaMalloc(&z, n * 4);
  cudaMemset(x, 0, n * 4); cudaMemset(y, 0, n * 4);
#define RUN(NAME, TWO, LAUNCH) { float ms = timeit([&] { LAUNCH; }); \
    printf("%-40s %8.1f us  %7.1f GB/s\n", NAME, ms * 1e3, (TWO ? 12.0 : 8.0) * n / (ms * 1e-3) / 1e9); }
  RUN("copy U4 T256 cs", false, (k_vec<4, 256, false, true><<<n4 / 1024, 256>>>(x, y, z, n4)));
  RUN("copy U8 T256 cs", false, (k_vec<8, 256, false, true><<<n4 / 2048, 256>>>(x, y, z, n4)));
  RUN("copy U2 T256 cs", false, (k_vec<2, 256, false, true><<<n4 / 512, 256>>>(x, y, z, n4)));
  RUN("copy U4 T512 cs", false, (k_vec<4, 512, false, true><<<n4 / 2048, 512>>>(x, y, z, n4)));
  RUN("copy U4 T256 plain", false, (k_vec<4, 256, false, false><<<n4 / 1024, 256>>>(x, y, z, n4)));
  RUN("copy U8 T128 cs", false, (k_vec<8, 128, false, true><<<n4 / 1024, 128>>>(x, y, z, n4)));
  RUN("copy persist U4 x148x8", false, (k_persist<4, false><<<148 * 8, 256>>>(x, y, z, n4)));
  RUN("copy persist U8 x148x4", false, (k_persist<8, false><<<148 * 4, 256>>>(x, y, z, n4)));
  RUN("add U4 T256 cs", true, (k_vec<4, 256, true, true><<<n4 / 1024, 256>>>(x, y, z, n4)));
  RUN("add U8 T256 cs", true, (k_vec<8, 256, true, true><<<n4 / 2048, 256>>>(x, y, z, n4)));
  RUN("add U2 T256 cs", true, (k_vec<2, 256, true, true><<<n4 / 512, 256>>>(x, y, z, n4)));
  RUN("add U4 T256 plain", true, (k_vec<4, 256, true, false><<<n4 / 1024, 256>>>(x, y, z, n4)));
  RUN("add persist U4 x148x8", true, (k_persist<4, true><<<148 * 8, 256>>>(x, y, z, n4)));
  RUN("memcpy D2D", false, (cudaMemcpyAsync(z, x, n * 4, cudaMemcpyDeviceToDevice)));
  return 0;
}
