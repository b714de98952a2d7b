// Issue cost of tcgen05.mma kind::tf32 (development tool): one CTA per SM
// issues R back-to-back MMAs (garbage operands) from one thread, single-CTA
// (cta_group::1) M = 128 with N = 64 / 128 / 256, A from smem (SS) or TMEM
// (TS), and reports clocks per MMA (commit + wait after the last one).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I include \
//        -I paper_conf_icpp_shenvms15_b200/csrc tools/mma_rates.cu -o /tmp/mma_rates
#include <cstdio>
#include <cuda_runtime.h>

#include "tc_ptx.h"

using namespace mm::tcx;

__device__ volatile int g_stop;

template <int N, bool TS, int D = 0>
__global__ void __launch_bounds__(128, 1) k_mma(long long* out, int R) {
  extern __shared__ __align__(1024) uint8_t sm[];
  __shared__ uint64_t bar;
  __shared__ uint32_t tslot;
  uint8_t* base = sm + ((1024u - (saddr(sm) & 1023u)) & 1023u);
  const int warp = threadIdx.x >> 5;
  if (threadIdx.x == 0) {
    mbar_init(&bar, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(saddr(&tslot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = tslot;
  __shared__ int stop;
  if (threadIdx.x == 0) stop = 0;
  __syncthreads();
  if (D != 0 && warp >= 1) {   // disturbance while thread 0 issues
    const int lane = threadIdx.x & 31;
    float v[16];
    for (int c = 0; c < 16; ++c) v[c] = lane * 1.f + c;
    float* sp = reinterpret_cast<float*>(base + 8192 + N * 64);   // scratch smem beyond the operands
    int it = 0;
    while (!*(volatile int*)&stop && it < 200000) {
      if (D == 1) {
        asm volatile(
            "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};" ::"r"(
                tmem + ((uint32_t)((warp & 3) * 32) << 16) + 384u + (uint32_t)((it & 7) * 16)),
            "f"(v[0]), "f"(v[1]), "f"(v[2]), "f"(v[3]), "f"(v[4]), "f"(v[5]), "f"(v[6]), "f"(v[7]), "f"(v[8]), "f"(v[9]),
            "f"(v[10]), "f"(v[11]), "f"(v[12]), "f"(v[13]), "f"(v[14]), "f"(v[15])
            : "memory");
        asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
      } else {
        *reinterpret_cast<float4*>(sp + ((threadIdx.x * 4 + it * 512) & 511)) = make_float4(v[0], v[1], v[2], v[3]);
      }
      ++it;
    }
  }
  if (threadIdx.x == 0) {
    const uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
    const uint64_t a = sdesc(base), b = sdesc(base + 8192);
    long long t0 = clock64();
    for (int i = 0; i < R; ++i) {
      const uint64_t adv = (uint64_t)((i & 1) * 32) >> 4;
      if (TS) {
        asm volatile(
            "{\n .reg .pred p;\n setp.ne.b32 p, %4, 0;\n"
            " tcgen05.mma.cta_group::1.kind::tf32 [%0], [%1], %2, %3, p;\n}\n" ::"r"(tmem),
            "r"(tmem + 256u + (uint32_t)((i & 7) * 8)), "l"(b + adv), "r"(idesc), "r"(1));
      } else {
        mma_tf32(tmem, a + adv, b + adv, idesc, 1u);
      }
    }
    mma_commit(&bar);
    mbar_wait(&bar, 0);
    long long t1 = clock64();
    out[blockIdx.x] = (t1 - t0);
    stop = 1;
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (warp == 0) {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tmem));
  }
}

template <int N, bool TS, int D = 0>
void run(const char* name, int R, long long* d, int grid) {
  const int smem = 8192 + N * 64 + 2048 + 4096;
  cudaFuncSetAttribute(k_mma<N, TS, D>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  k_mma<N, TS, D><<<grid, 128, smem>>>(d, R);
  k_mma<N, TS, D><<<grid, 128, smem>>>(d, R);
  cudaError_t e = cudaDeviceSynchronize();
  long long h[148];
  cudaMemcpy(h, d, grid * 8, cudaMemcpyDeviceToHost);
  double s = 0;
  for (int i = 0; i < grid; ++i) s += h[i];
  const double clk = s / grid / R;
  const double flop = 2.0 * 128 * N * 8;
  printf("%-10s grid %3d: %7.1f clk per MMA, %6.0f flop/clk/SM (%s)\n", name, grid, clk, flop / clk,
         cudaGetErrorString(e));
}

__device__ __forceinline__ void mma_ts2(uint32_t d, uint32_t a, uint64_t b, uint32_t idesc) {
  asm volatile(
      "{\n .reg .pred p;\n setp.ne.b32 p, %4, 0;\n"
      " tcgen05.mma.cta_group::2.kind::tf32 [%0], [%1], %2, %3, p;\n}\n" ::"r"(d),
      "r"(a), "l"(b), "r"(idesc), "r"(1));
}

// cta_group::2 pair: the leader CTA issues M = 256 MMAs; each CTA holds its
// 128 rows of A (smem or TMEM) and half of B
template <int N, bool TS, int C = 0>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(128, 1) k_mma2(long long* out, int R) {
  extern __shared__ __align__(1024) uint8_t sm[];
  __shared__ uint64_t bar, sbar[4];
  __shared__ uint32_t tslot;
  uint8_t* base = sm + ((1024u - (saddr(sm) & 1023u)) & 1023u);
  uint32_t rank;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(rank));
  const int warp = threadIdx.x >> 5;
  if (threadIdx.x == 0) {
    mbar_init(&bar, 1);
    for (int q = 0; q < 4; ++q) mbar_init(&sbar[q], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(saddr(&tslot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  cluster_sync_all();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = tslot;
  __shared__ int stop2;
  if (threadIdx.x == 0) stop2 = 0;
  __syncthreads();
  cluster_sync_all();
  if (C == 6 && warp >= 1) {
    const int lane = threadIdx.x & 31;
    float v[16];
    for (int c = 0; c < 16; ++c) v[c] = lane * 1.f + c;
    int it = 0;
    while (!*(volatile int*)&stop2 && it < 400000) {
      asm volatile(
          "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};" ::"r"(
              tmem + ((uint32_t)((warp & 3) * 32) << 16) + 128u + (uint32_t)((it & 7) * 16)),
          "f"(v[0]), "f"(v[1]), "f"(v[2]), "f"(v[3]), "f"(v[4]), "f"(v[5]), "f"(v[6]), "f"(v[7]), "f"(v[8]), "f"(v[9]),
          "f"(v[10]), "f"(v[11]), "f"(v[12]), "f"(v[13]), "f"(v[14]), "f"(v[15])
          : "memory");
      asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
      ++it;
      if (rank == 1 && (it & 255) == 0) {   // the peer stops when the leader does
        uint32_t v2;
        asm volatile("ld.shared::cluster.u32 %0, [%1];" : "=r"(v2) : "r"(peer_addr(&stop2, 0)) : "memory");
        if (v2) break;
      }
    }
  }
  if (threadIdx.x == 0 && rank == 0) {
    const uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(256 >> 4) << 24);
    const uint64_t a = sdesc(base), b = sdesc(base + 8192);
    long long t0 = clock64();
    for (int i = 0; i < R; ++i) {
      const uint64_t adv = (uint64_t)((i & 1) * 32) >> 4;
      if (C >= 3) {   // fused-kernel pattern: 6 MMAs per k-step, stage = k-step % 8 (C=4: stage 0 only)
        if (i % 6) continue;
        const int st = C != 4 ? (i / 6) % 8 : 0;
        if (C >= 5) asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        const uint64_t bhi = sdesc(base + 8192 + st * 8192), blo = sdesc(base + 8192 + st * 8192 + 4096);
        const uint32_t ahi = tmem + 128u + (uint32_t)(st * 32), alo = ahi + 16u;
#pragma unroll
        for (int kk = 0; kk < 2; ++kk) {
          const uint64_t ad = (uint64_t)(kk * 32) >> 4;
          mma_ts2(tmem, alo + 8u * kk, bhi + ad, idesc);
          mma_ts2(tmem, ahi + 8u * kk, blo + ad, idesc);
          mma_ts2(tmem, ahi + 8u * kk, bhi + ad, idesc);
        }
        if (C >= 5) mma_commit_pair(&sbar[(i / 6) & 3]);
      } else if (TS) {
        asm volatile(
            "{\n .reg .pred p;\n setp.ne.b32 p, %4, 0;\n"
            " tcgen05.mma.cta_group::2.kind::tf32 [%0], [%1], %2, %3, p;\n}\n" ::"r"(tmem),
            "r"(tmem + 256u + (uint32_t)((i & 7) * 8)), "l"(b + adv), "r"(idesc), "r"(1));
      } else {
        mma_tf32_pair(tmem, a + adv, b + adv, idesc, 1u);
      }
      if (C >= 1 && C < 3 && i % 6 == 5) {
        mma_commit_pair(&sbar[(i / 6) & 3]);
        if (C >= 2) {
          asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        }
      }
    }
    mma_commit_pair(&bar);
    mbar_wait(&bar, 0);
    long long t1 = clock64();
    out[blockIdx.x / 2] = (t1 - t0);
    stop2 = 1;
  }
  if (threadIdx.x == 0 && rank == 1) mbar_wait(&bar, 0);
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  cluster_sync_all();
  if (warp == 0) {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, 512;" ::"r"(tmem));
  }
}

template <int N, bool TS, int C = 0>
void run2(const char* name, int R, long long* d, int pairs) {
  const int smem = C >= 3 ? 8192 + 8 * 8192 + 2048 : 8192 + N * 32 + 2048;
  cudaFuncSetAttribute(k_mma2<N, TS, C>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  k_mma2<N, TS, C><<<2 * pairs, 128, smem>>>(d, R);
  k_mma2<N, TS, C><<<2 * pairs, 128, smem>>>(d, R);
  cudaError_t e = cudaDeviceSynchronize();
  long long h[148];
  cudaMemcpy(h, d, pairs * 8, cudaMemcpyDeviceToHost);
  double s = 0;
  for (int i = 0; i < pairs; ++i) s += h[i];
  const double clk = s / pairs / R;
  const double flop = 2.0 * 256 * N * 8 / 2;   // per SM
  printf("%-10s pairs %3d: %7.1f clk per MMA, %6.0f flop/clk/SM (%s)\n", name, pairs, clk, flop / clk,
         cudaGetErrorString(e));
}

int main() {
  long long* d;
  cudaMalloc(&d, 148 * 8);
  for (int grid : {1, 148}) {
    run<64, false>("SS N=64", 4096, d, grid);
    run<128, false>("SS N=128", 4096, d, grid);
    run<256, false>("SS N=256", 4096, d, grid);
    run<64, true>("TS N=64", 4096, d, grid);
    run<128, true>("TS N=128", 4096, d, grid);
    run<256, true>("TS N=256", 4096, d, grid);
  }
  run<128, true, 1>("TS128+tst", 4096, d, 148);
  run<128, true, 2>("TS128+sts", 4096, d, 148);
  run<128, false, 1>("SS128+tst", 4096, d, 148);
  run<128, false, 2>("SS128+sts", 4096, d, 148);
  run2<128, true, 3>("2TS128stm", 4098, d, 74);
  run2<128, true, 4>("2TS128st0", 4098, d, 74);
  run2<128, true, 5>("2TS128fus", 4098, d, 74);
  run2<128, true, 6>("2TS128f+d", 4098, d, 74);
  run2<128, true, 1>("2TS128+cm", 4098, d, 74);
  run2<128, true, 2>("2TS128+cmf", 4098, d, 74);
  for (int pairs : {1, 74}) {
    run2<128, false>("2SS N=128", 4096, d, pairs);
    run2<256, false>("2SS N=256", 4096, d, pairs);
    run2<128, true>("2TS N=128", 4096, d, pairs);
    run2<256, true>("2TS N=256", 4096, d, pairs);
  }
  return 0;
}
