// Counter-hash input generator on the device (the
// same recipe as synthgen.py, checked bit for bit by tests/test_gpu_parity.py).
// Holds no arithmetic of the method: it only produces seeded synthetic inputs
// in place on each device (resident mode).
#include "kernels.h"

namespace mm {

namespace {

__device__ __forceinline__ uint64_t splitmix64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

__global__ void fill_u(float* __restrict__ dst, int64_t n, uint64_t key, int64_t start, float lo,
                       float span) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    const uint64_t h = splitmix64((uint64_t)(start + i) ^ key) >> 40;
    const float u = __fmul_rn((float)h, 5.9604644775390625e-08f);  // * 2^-24, exact
    dst[i] = __fadd_rn(lo, __fmul_rn(span, u));
  }
}

__global__ void fill_i(float* __restrict__ dst, int64_t n, uint64_t key, int64_t start, int32_t lo,
                       uint64_t span) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    const uint64_t h = splitmix64((uint64_t)(start + i) ^ key) >> 40;
    dst[i] = (float)(lo + (int64_t)(h % span));
  }
}

unsigned grid_for(int64_t n) {
  int64_t b = (n + 255) / 256;
  if (b > 148 * 64) b = 148 * 64;
  return (unsigned)(b < 1 ? 1 : b);
}

}  // namespace

cudaError_t fill_uniform(float* dst, int64_t n, uint64_t seed, int32_t array_id, int64_t start,
                         float lo, float hi, cudaStream_t s) {
  if (n <= 0) return cudaSuccess;
  const uint64_t key = seed ^ ((uint64_t)(uint32_t)array_id << 48);
  const float span = hi - lo;  // one float32 rounding, as synthgen
  note_launch();
  fill_u<<<grid_for(n), 256, 0, s>>>(dst, n, key, start, lo, span);
  return cudaGetLastError();
}

cudaError_t fill_integers(float* dst, int64_t n, uint64_t seed, int32_t array_id, int64_t start,
                          int32_t lo, int32_t hi, cudaStream_t s) {
  if (n <= 0) return cudaSuccess;
  if (hi < lo) return cudaErrorInvalidValue;
  const uint64_t key = seed ^ ((uint64_t)(uint32_t)array_id << 48);
  note_launch();
  fill_i<<<grid_for(n), 256, 0, s>>>(dst, n, key, start, lo, (uint64_t)(hi - lo + 1));
  return cudaGetLastError();
}

}  // namespace mm

namespace mm {

namespace {

__device__ __forceinline__ uint64_t splitmix64b(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

// Tile-major element e -> (r, c); A[r][c] = (S[r][c] + S[c][r]) * 0.5 + n [r==c]
// in FP64 (both terms are exact 24-bit dyadics), one rounding to FP32.
__global__ void fill_spd(float* __restrict__ dst, int64_t n, int64_t b, uint64_t key) {
  const int64_t T = n / b, bb = b * b, tot = n * n;
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < tot; e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t tile = e / bb, w = e % bb;
    const int64_t r = (tile / T) * b + w / b, c = (tile % T) * b + w % b;
    const double u1 = (double)(splitmix64b((uint64_t)(r * n + c) ^ key) >> 40) * 5.9604644775390625e-08;
    const double u2 = (double)(splitmix64b((uint64_t)(c * n + r) ^ key) >> 40) * 5.9604644775390625e-08;
    double v = (u1 + u2) * 0.5;
    if (r == c) v += (double)n;
    dst[e] = (float)v;
  }
}

}  // namespace

cudaError_t fill_spd_tiles(float* dst, int64_t n, int64_t b, uint64_t seed, int32_t array_id, cudaStream_t s) {
  if (n <= 0 || b <= 0 || n % b) return cudaErrorInvalidValue;
  const uint64_t key = seed ^ ((uint64_t)(uint32_t)array_id << 48);
  int64_t blocks = (n * n + 255) / 256;
  if (blocks > 148 * 64) blocks = 148 * 64;
  note_launch();
  fill_spd<<<(unsigned)blocks, 256, 0, s>>>(dst, n, b, key);
  return cudaGetLastError();
}

}  // namespace mm
