// Microbenchmark of HotSpot kernel layouts (development tool, not the product).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o /tmp/hv tools/hotspot_variants.cu
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <vector>

struct HotCoef { float sdc, rx1, ry1, rz1, amb; };
__device__ __forceinline__ float cell(float c, float n, float s, float w, float e, float p, const HotCoef& k) {
  const float two = __fadd_rn(c, c);
  const float dv = __fmul_rn(__fsub_rn(__fadd_rn(s, n), two), k.ry1);
  const float dh = __fmul_rn(__fsub_rn(__fadd_rn(e, w), two), k.rx1);
  const float dz = __fmul_rn(__fsub_rn(k.amb, c), k.rz1);
  const float sum = __fadd_rn(__fadd_rn(__fadd_rn(p, dv), dh), dz);
  return __fadd_rn(c, __fmul_rn(k.sdc, sum));
}

// strip kernel: tile = (colblock, strip of H rows); persistent if grid < tiles (in-order sweep)
template <int H, bool PREF>
__global__ void __launch_bounds__(256) strip(const float* __restrict__ tin, const float* __restrict__ pw,
    float* __restrict__ tout, int64_t rows, int64_t cols, HotCoef k, int64_t ncb, int64_t ntiles) {
  const int lane = threadIdx.x & 31;
  for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const int64_t cb = tile % ncb, st = tile / ncb;
    const int64_t x0 = (cb * 256 + threadIdx.x) * 4;
    const int64_t ys = st * H, ye = min(ys + H, rows);
    const bool active = x0 < cols;
    const int64_t xs = active ? x0 : 0;
    auto ld4 = [&](int64_t y) -> float4 { return *reinterpret_cast<const float4*>(tin + y * cols + xs); };
    float4 up = ld4(ys > 0 ? ys - 1 : ys);
    float4 cu = ld4(ys);
    float4 dn = ld4(ys + 1 < rows ? ys + 1 : ys);
    float4 p = __ldcs(reinterpret_cast<const float4*>(pw + ys * cols + xs));
    for (int64_t y = ys; y < ye; ++y) {
      float4 dn2 = dn, pn = p;
      if (PREF && y + 1 < ye) {
        dn2 = ld4(y + 2 < rows ? y + 2 : rows - 1);
        pn = __ldcs(reinterpret_cast<const float4*>(pw + (y + 1) * cols + xs));
      }
      float w = __shfl_up_sync(0xffffffffu, cu.w, 1);
      float e = __shfl_down_sync(0xffffffffu, cu.x, 1);
      if (lane == 0) w = (x0 > 0 && active) ? tin[y * cols + x0 - 1] : cu.x;
      if (lane == 31) e = (x0 + 4 < cols && active) ? tin[y * cols + x0 + 4] : cu.w;
      if (x0 == 0) w = cu.x;
      if (x0 + 4 >= cols) e = cu.w;
      const bool top = y > 0, bot = y + 1 < rows;
      float4 o;
      o.x = cell(cu.x, top ? up.x : cu.x, bot ? dn.x : cu.x, w, cu.y, p.x, k);
      o.y = cell(cu.y, top ? up.y : cu.y, bot ? dn.y : cu.y, cu.x, cu.z, p.y, k);
      o.z = cell(cu.z, top ? up.z : cu.z, bot ? dn.z : cu.z, cu.y, cu.w, p.z, k);
      o.w = cell(cu.w, top ? up.w : cu.w, bot ? dn.w : cu.w, cu.z, e, p.w, k);
      if (active) __stcs(reinterpret_cast<float4*>(tout + y * cols + x0), o);
      up = cu; cu = dn;
      if (PREF) { dn = dn2; p = pn; }
      else if (y + 1 < ye) { dn = ld4(y + 2 < rows ? y + 2 : rows - 1); p = __ldcs(reinterpret_cast<const float4*>(pw + (y + 1) * cols + xs)); }
    }
  }
}

// batch kernel: each thread loads all H+2 T rows and H P rows of its float4
// column first (deep MLP), then computes H rows.
template <int H>
__global__ void __launch_bounds__(256) batch(const float* __restrict__ tin, const float* __restrict__ pw,
    float* __restrict__ tout, int64_t rows, int64_t cols, HotCoef k, int64_t ncb) {
  const int lane = threadIdx.x & 31;
  const int64_t tile = blockIdx.x;
  const int64_t cb = tile % ncb, st = tile / ncb;
  const int64_t x0 = (cb * 256 + threadIdx.x) * 4;
  const int64_t ys = st * H;
  const bool active = x0 < cols;
  const int64_t xs = active ? x0 : 0;
  float4 T[H + 2], P[H];
  float W[H], E[H];
#pragma unroll
  for (int j = 0; j < H + 2; ++j) {
    int64_t y = ys - 1 + j; y = y < 0 ? 0 : (y >= rows ? rows - 1 : y);
    T[j] = *reinterpret_cast<const float4*>(tin + y * cols + xs);
  }
#pragma unroll
  for (int j = 0; j < H; ++j) {
    int64_t y = ys + j; y = y >= rows ? rows - 1 : y;
    P[j] = __ldcs(reinterpret_cast<const float4*>(pw + y * cols + xs));
    W[j] = (lane == 0 && x0 > 0 && active) ? tin[y * cols + x0 - 1] : 0.f;
    E[j] = (lane == 31 && x0 + 4 < cols && active) ? tin[y * cols + x0 + 4] : 0.f;
  }
#pragma unroll
  for (int j = 0; j < H; ++j) {
    const int64_t y = ys + j;
    if (y >= rows) break;
    const float4 up = T[j], cu = T[j + 1], dn = T[j + 2], p = P[j];
    float w = __shfl_up_sync(0xffffffffu, cu.w, 1);
    float e = __shfl_down_sync(0xffffffffu, cu.x, 1);
    if (lane == 0) w = (x0 > 0 && active) ? W[j] : cu.x;
    if (lane == 31) e = (x0 + 4 < cols && active) ? E[j] : cu.w;
    if (x0 == 0) w = cu.x;
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

__global__ void copy3(const float4* a, const float4* b, float4* c, int64_t n4) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n4; i += (int64_t)gridDim.x * blockDim.x) {
    float4 x = __ldcs(a + i), y = __ldcs(b + i);
    __stcs(c + i, make_float4(x.x + y.x, x.y + y.y, x.z + y.z, x.w + y.w));
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

template <int H>
void run_batch(float* t, float* p, float* o, int64_t n) {
  const int64_t ncb = (n / 4 + 255) / 256, ntiles = ncb * ((n + H - 1) / H);
  int occ = 0; cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, batch<H>, 256, 0);
  HotCoef k{1.3653333f, 0.1f, 0.1f, 4.8828125e-5f, 80.f};
  float ms = timeit([&] { batch<H><<<(unsigned)ntiles, 256>>>(t, p, o, n, n, k, ncb); });
  printf("%-28s n=%6lld H=%3d occ=%d grid=%7lld  %8.1f us  %7.1f GB/s\n", "batch", (long long)n, H, occ,
         (long long)ntiles, ms * 1e3, 12.0 * n * n / (ms * 1e-3) / 1e9);
}

template <int H, bool PREF>
void run_strip(const char* name, float* t, float* p, float* o, int64_t n, bool persistent) {
  const int64_t ncb = (n / 4 + 255) / 256, ntiles = ncb * ((n + H - 1) / H);
  int occ = 0; cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, strip<H, PREF>, 256, 0);
  int64_t grid = persistent ? std::min<int64_t>(ntiles, 148LL * occ) : ntiles;
  HotCoef k{1.3653333f, 0.1f, 0.1f, 4.8828125e-5f, 80.f};
  float ms = timeit([&] { strip<H, PREF><<<(unsigned)grid, 256>>>(t, p, o, n, n, k, ncb, ntiles); });
  printf("%-28s n=%6lld H=%3d pref=%d pers=%d occ=%d grid=%7lld  %8.1f us  %7.1f GB/s\n", name, (long long)n, H, PREF,
         persistent, occ, (long long)grid, ms * 1e3, 12.0 * n * n / (ms * 1e-3) / 1e9);
}

int main() {
  for (int64_t n : {8192LL, 16384LL}) {
    float *t, *p, *o;
    cudaMalloc(&t, n * n * 4); cudaMalloc(&p, n * n * 4); cudaMalloc(&o, n * n * 4);
    cudaMemset(t, 0, n * n * 4); cudaMemset(p, 0, n * n * 4);
    float ms = timeit([&] { copy3<<<148 * 8, 256>>>((float4*)t, (float4*)p, (float4*)o, n * n / 4); });
    printf("add-like reference            n=%6lld %8.1f us %7.1f GB/s\n", (long long)n, ms * 1e3, 12.0 * n * n / (ms * 1e-3) / 1e9);
    run_batch<2>(t, p, o, n);
    run_batch<4>(t, p, o, n);
    run_batch<6>(t, p, o, n);
    run_batch<8>(t, p, o, n);
    run_batch<12>(t, p, o, n);
    run_strip<4, true>("strip", t, p, o, n, false);
    run_strip<8, false>("strip", t, p, o, n, false);
    run_strip<16, false>("strip", t, p, o, n, false);
    run_strip<32, false>("strip", t, p, o, n, false);
    run_strip<64, false>("strip", t, p, o, n, false);
    run_strip<8, true>("strip", t, p, o, n, false);
    run_strip<16, true>("strip", t, p, o, n, false);
    run_strip<32, true>("strip", t, p, o, n, false);
    run_strip<16, false>("strip", t, p, o, n, true);
    run_strip<16, true>("strip", t, p, o, n, true);
    run_strip<32, true>("strip", t, p, o, n, true);
    run_strip<8, true>("strip", t, p, o, n, true);
    cudaFree(t); cudaFree(p); cudaFree(o);
  }
  return 0;
}
