// MatrixMul C = A x B, FP32, row-major, rows [r0, r1) of A and C (P211-215
// Table II, P311: "each task instance receives multiple consecutive rows of A
// and the full B").
//
// variant 1 (FFMA): classic register-blocked SIMT SGEMM — 128x128 CTA tile,
// BK = 8, 256 threads x (8x8) outputs, shared-memory double buffering.  It is
// the FFMA baseline (tensor cores only via 3xTF32 or
// FFMA).  variant 2 (default) is the tcgen05 3xTF32 kernel in kernels_gemm_tc.cu.
#include "kernels.h"

namespace mm {

cudaError_t sgemm_tf32x3_rows(const float* A, const float* B, float* C, int64_t M, int64_t N,
                              int64_t K, int64_t r0, int64_t r1, cudaStream_t s, int sms, Scratch* scr,
                              bool b_readonly);

namespace {

constexpr int BM = 128, BN = 128, BK = 8, TM = 8, TN = 8, NT = 256;

__global__ void __launch_bounds__(NT) sgemm_ffma(const float* __restrict__ A, const float* __restrict__ B,
                                                 float* __restrict__ C, int64_t N, int64_t K,
                                                 int64_t r0, int64_t r1) {
  __shared__ __align__(16) float As[2][BK][BM + 4];
  __shared__ __align__(16) float Bs[2][BK][BN];
  const int tid = threadIdx.x;
  const int64_t m0 = r0 + (int64_t)blockIdx.y * BM;
  const int64_t n0 = (int64_t)blockIdx.x * BN;
  // loader mapping: A tile BM x BK -> thread loads rows (tid/2) cols (tid%2)*4..+3
  const int a_row = tid >> 1, a_col = (tid & 1) * 4;
  // B tile BK x BN -> thread loads row tid/32, cols (tid%32)*4..+3
  const int b_row = tid >> 5, b_col = (tid & 31) * 4;
  const int ty = tid >> 4, tx = tid & 15;  // 16 x 16 threads, 8 x 8 each

  float acc[TM][TN];
#pragma unroll
  for (int i = 0; i < TM; ++i)
#pragma unroll
    for (int j = 0; j < TN; ++j) acc[i][j] = 0.f;

  auto load_a = [&](int64_t k0, float4& v) {
    const int64_t m = m0 + a_row;
    const int64_t k = k0 + a_col;
    v = make_float4(0.f, 0.f, 0.f, 0.f);
    if (m < r1) {
      const float* p = A + m * K + k;
      if (k + 3 < K && ((K & 3) == 0)) v = *reinterpret_cast<const float4*>(p);
      else {
        if (k + 0 < K) v.x = p[0];
        if (k + 1 < K) v.y = p[1];
        if (k + 2 < K) v.z = p[2];
        if (k + 3 < K) v.w = p[3];
      }
    }
  };
  auto load_b = [&](int64_t k0, float4& v) {
    const int64_t k = k0 + b_row;
    const int64_t n = n0 + b_col;
    v = make_float4(0.f, 0.f, 0.f, 0.f);
    if (k < K) {
      const float* p = B + k * N + n;
      if (n + 3 < N && ((N & 3) == 0)) v = *reinterpret_cast<const float4*>(p);
      else {
        if (n + 0 < N) v.x = p[0];
        if (n + 1 < N) v.y = p[1];
        if (n + 2 < N) v.z = p[2];
        if (n + 3 < N) v.w = p[3];
      }
    }
  };
  auto store = [&](int buf, const float4& va, const float4& vb) {
    As[buf][a_col + 0][a_row] = va.x;
    As[buf][a_col + 1][a_row] = va.y;
    As[buf][a_col + 2][a_row] = va.z;
    As[buf][a_col + 3][a_row] = va.w;
    *reinterpret_cast<float4*>(&Bs[buf][b_row][b_col]) = vb;
  };

  float4 va, vb;
  load_a(0, va);
  load_b(0, vb);
  store(0, va, vb);
  __syncthreads();
  const int64_t nk = (K + BK - 1) / BK;
  for (int64_t kt = 0; kt < nk; ++kt) {
    const int cur = kt & 1;
    if (kt + 1 < nk) {
      load_a((kt + 1) * BK, va);
      load_b((kt + 1) * BK, vb);
    }
#pragma unroll
    for (int kk = 0; kk < BK; ++kk) {
      float ra[TM], rb[TN];
      const float4 a0 = *reinterpret_cast<const float4*>(&As[cur][kk][ty * 4]);
      const float4 a1 = *reinterpret_cast<const float4*>(&As[cur][kk][64 + ty * 4]);
      const float4 b0 = *reinterpret_cast<const float4*>(&Bs[cur][kk][tx * 4]);
      const float4 b1 = *reinterpret_cast<const float4*>(&Bs[cur][kk][64 + tx * 4]);
      ra[0] = a0.x; ra[1] = a0.y; ra[2] = a0.z; ra[3] = a0.w;
      ra[4] = a1.x; ra[5] = a1.y; ra[6] = a1.z; ra[7] = a1.w;
      rb[0] = b0.x; rb[1] = b0.y; rb[2] = b0.z; rb[3] = b0.w;
      rb[4] = b1.x; rb[5] = b1.y; rb[6] = b1.z; rb[7] = b1.w;
#pragma unroll
      for (int i = 0; i < TM; ++i)
#pragma unroll
        for (int j = 0; j < TN; ++j) acc[i][j] = fmaf(ra[i], rb[j], acc[i][j]);
    }
    if (kt + 1 < nk) {
      store(cur ^ 1, va, vb);
    }
    __syncthreads();
  }
  // epilogue: rows ty*4+{0..3} and 64+ty*4+{0..3}; cols tx*4.. and 64+tx*4..
#pragma unroll
  for (int i = 0; i < TM; ++i) {
    const int64_t m = m0 + (i < 4 ? ty * 4 + i : 64 + ty * 4 + (i - 4));
    if (m >= r1) continue;
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      const int64_t n = n0 + h * 64 + tx * 4;
      float* p = C + m * N + n;
      const float4 v = make_float4(acc[i][h * 4 + 0], acc[i][h * 4 + 1], acc[i][h * 4 + 2], acc[i][h * 4 + 3]);
      if (n + 3 < N && (N & 3) == 0) *reinterpret_cast<float4*>(p) = v;
      else {
        if (n + 0 < N) p[0] = v.x;
        if (n + 1 < N) p[1] = v.y;
        if (n + 2 < N) p[2] = v.z;
        if (n + 3 < N) p[3] = v.w;
      }
    }
  }
}

}  // namespace

cudaError_t sgemm_rows(const float* A, const float* B, float* C, int64_t M, int64_t N, int64_t K,
                       int64_t r0, int64_t r1, int32_t variant, cudaStream_t s, int sms, Scratch* scr,
                       bool b_readonly) {
  (void)M;
  if (r1 <= r0 || N <= 0) return cudaSuccess;
  if (variant == 2) return sgemm_tf32x3_rows(A, B, C, M, N, K, r0, r1, s, sms, scr, b_readonly);
  dim3 grid((unsigned)((N + BN - 1) / BN), (unsigned)((r1 - r0 + BM - 1) / BM));
  note_launch();
  sgemm_ffma<<<grid, NT, 0, s>>>(A, B, C, N, K, r0, r1);
  return cudaGetLastError();
}

}  // namespace mm
