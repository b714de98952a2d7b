// Cholesky TRSM of one step's column in ONE launch (round 2): X_i <- A_ik
// L_kk^{-T} for a batch of tiles i (substitution, no inverse;
// reading R28), replacing the 8 leaf + 7 block-update launches per step of the
// leaf path in kernels_chol.cu.
//
// A CTA owns 128 rows of one tile (grid = (b/128, tasks)); its rows are
// independent of every other CTA's, so there is no cross-CTA traffic.  Left
// looking over the 128-column leaves q = 0 .. b/128-1:
//
//   acc_q  = sum_{j<q} X_j L_qj^T           3xTF32 tcgen05.mma, M = N = 128,
//                                            FP32 accumulator in TMEM
//   leaf q: X_q = (B_q - acc_q) L_qq^{-T}    substitution, thread = row, four
//                                            32-column sub-blocks in registers
//
// Warp roles (320 threads, one CTA per SM):
//   warp 0   TMA producer: operand stages of the j <= q-2 terms (X_j hi/lo
//            from the step's panel slot, written back by this CTA's earlier
//            leaves; L_qj hi/lo from the L_kk slot) and the B half of the
//            j = q-1 term
//   warp 1   TMEM allocator (512 columns: acc A, acc B, X hi, X lo) and the
//            single-thread MMA issuer; the j = q-1 term reads X_{q-1} straight
//            from TMEM (TS form), so the critical hand-off leaf q-1 -> acc_q
//            never goes through global memory
//   warps 2-9 the substitution (TMEM lane = row; warps w and w+4 share a
//            row group, each taking 16 of a sub-block's 32 columns: the first
//            solves its 16 and hands them to the second through TMEM, so the
//            arithmetic and its order are one thread's).  A sub-block: x = B -
//            acc (tcgen05.ld), minus the earlier sub-blocks of the leaf
//            (accumulated first, ascending, as in the leaf kernels), then the
//            32-column forward substitution with div_rcp quotients; the
//            solved x goes to TMEM (fp32 into the consumed acc columns for
//            the later sub-blocks, hi/lo for the MMA) and through a SWIZZLE_128B
//            staging buffer to global memory by TMA stores (X into the tile,
//            hi/lo into the panel slot the step's SYRK/GEMM and this CTA's
//            later leaves read).
// acc_{q+1}'s j <= q-1 terms run on the tensor pipe while leaf q substitutes.
// The leaf's L_qq block arrives transposed with its reciprocal diagonal
// (lkk_prep, one launch per step) by one bulk copy into shared memory.
//
// Exact-factor inputs stay exact (every product and partial sum an integer
// below 2^24, every quotient exact), so the factor is L0 bit for bit; the
// result of a tile does not depend on the batch it runs in.
#include <cuda.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "kernels.h"
#include "tc_ptx.h"

namespace mm {

cudaError_t encode_tmap_2d_f32(CUtensorMap* m, const void* base, uint64_t inner, uint64_t outer,
                               uint64_t row_bytes, uint32_t box_inner, uint32_t box_outer);
size_t chol_potrf_flag_bytes(int64_t b);

namespace {

using namespace tcx;

constexpr int kTcRows = 128, kTcLeaf = 128, kTcBK = 16, kTcStages = 3, kTcThreads = 320;
constexpr int kTcOpBytes = kTcRows * kTcBK * 4;            // 8 KB: one operand box (16 fp32 x 128 rows)
constexpr int kTcStageBytes = 4 * kTcOpBytes;               // A hi, A lo, B hi, B lo
// The leaf's L block, packed as the 32 x 32 blocks the substitution reads
// (all threads read the same address: broadcasts):
//   U[s(s-1)/2 + mb][i][c] = L[c0+32s+c][c0+32mb+i]   s = 1..3, mb < s
//   D[s][c][c2]            = L[c0+32s+c2][c0+32s+c]   s = 0..3
//   rd[m]                  = RN(1 / L[c0+m][c0+m])
constexpr int kLtBytes = kLtFloats * 4;                     // 41472 (layout: kernels.h)
constexpr int kStgBytes = kTcRows * 32 * 4;                 // 16 KB: 128 rows x 32 fp32 (SWIZZLE_128B)
constexpr int kMaxLeaves = 32;                              // b <= 4096
constexpr int kSmRing = 0, kSmStg = kTcStages * kTcStageBytes, kSmBpre = kSmStg + 3 * kStgBytes;
constexpr int kSmLt = kSmBpre + 2 * kStgBytes, kSmBar = kSmLt + kLtBytes;
constexpr int kNBar = 2 * kTcStages + 2 + 7 * kMaxLeaves;  // see trsm_col
constexpr int kTcSmem = kSmBar + 8 * kNBar + 16 + 1024;
constexpr int kStampsPerCta = 64;   // MM_TRSM_STAMPS: globaltimer per CTA (see trsm_col)

struct ColJob {
  int32_t n, k, slot0, nleaf;
  int64_t T, b;
  int32_t ti[kCholBatch];
};

__device__ __forceinline__ bool tw(uint64_t* b, uint32_t parity) {
  uint32_t done;
  asm volatile("{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
               : "=r"(done)
               : "r"(saddr(b)), "r"(parity)
               : "memory");
  return done;
}
// mbarrier wait that traps after ~4 s instead of hanging the GPU
__device__ __forceinline__ void twait(uint64_t* b, uint32_t parity) {
  if (tw(b, parity)) return;
  uint64_t t0, t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  for (;;) {
    if (tw(b, parity)) return;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    if (t - t0 > 4000000000ull) __trap();
  }
}

// rowcnt != NULL (launched as a programmatic dependent of the step's POTRF):
// the rows of leaf q of L_kk, with their split and packed block, are final
// once POTRF counted all 16 q + 10 of their 32 x 32 blocks
__device__ __forceinline__ void wait_rows(const int* rowcnt, int q) {
  if (!rowcnt) return;
  uint64_t t0 = 0;
  for (;;) {
    int v;
    asm volatile("ld.acquire.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(rowcnt + q) : "memory");
    if (v >= 16 * q + 10) break;
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    if (!t0) t0 = t;
    else if (t - t0 > 4000000000ull) __trap();
    __nanosleep(64);
  }
  asm volatile("fence.proxy.async.global;" ::: "memory");   // POTRF's generic stores -> our TMA / bulk loads
}

__device__ __forceinline__ void mma_ts(uint32_t d, uint32_t a_tmem, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n .reg .pred p;\n setp.ne.b32 p, %4, 0;\n"
      " tcgen05.mma.cta_group::1.kind::tf32 [%0], [%1], %2, %3, p;\n}\n" ::"r"(d),
      "r"(a_tmem), "l"(b), "r"(idesc), "r"(acc));
}

__device__ __forceinline__ void tmem_ld32(uint32_t ta, float (&v)[32]) {
  uint32_t* u = reinterpret_cast<uint32_t*>(v);
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
      "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
      : "=r"(u[0]), "=r"(u[1]), "=r"(u[2]), "=r"(u[3]), "=r"(u[4]), "=r"(u[5]), "=r"(u[6]), "=r"(u[7]),
        "=r"(u[8]), "=r"(u[9]), "=r"(u[10]), "=r"(u[11]), "=r"(u[12]), "=r"(u[13]), "=r"(u[14]), "=r"(u[15]),
        "=r"(u[16]), "=r"(u[17]), "=r"(u[18]), "=r"(u[19]), "=r"(u[20]), "=r"(u[21]), "=r"(u[22]), "=r"(u[23]),
        "=r"(u[24]), "=r"(u[25]), "=r"(u[26]), "=r"(u[27]), "=r"(u[28]), "=r"(u[29]), "=r"(u[30]), "=r"(u[31])
      : "r"(ta));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}
__device__ __forceinline__ void tmem_ld16(uint32_t ta, float (&v)[16]) {
  uint32_t* u = reinterpret_cast<uint32_t*>(v);
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
      : "=r"(u[0]), "=r"(u[1]), "=r"(u[2]), "=r"(u[3]), "=r"(u[4]), "=r"(u[5]), "=r"(u[6]), "=r"(u[7]),
        "=r"(u[8]), "=r"(u[9]), "=r"(u[10]), "=r"(u[11]), "=r"(u[12]), "=r"(u[13]), "=r"(u[14]), "=r"(u[15])
      : "r"(ta));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}
__device__ __forceinline__ void tmem_st16(uint32_t ta, const float (&v)[16]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};" ::"r"(
          ta),
      "f"(v[0]), "f"(v[1]), "f"(v[2]), "f"(v[3]), "f"(v[4]), "f"(v[5]), "f"(v[6]), "f"(v[7]), "f"(v[8]), "f"(v[9]),
      "f"(v[10]), "f"(v[11]), "f"(v[12]), "f"(v[13]), "f"(v[14]), "f"(v[15])
      : "memory");
}
__device__ __forceinline__ void tmem_st32(uint32_t ta, const float (&v)[32]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,"
      "%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};" ::"r"(ta),
      "f"(v[0]), "f"(v[1]), "f"(v[2]), "f"(v[3]), "f"(v[4]), "f"(v[5]), "f"(v[6]), "f"(v[7]), "f"(v[8]),
      "f"(v[9]), "f"(v[10]), "f"(v[11]), "f"(v[12]), "f"(v[13]), "f"(v[14]), "f"(v[15]), "f"(v[16]),
      "f"(v[17]), "f"(v[18]), "f"(v[19]), "f"(v[20]), "f"(v[21]), "f"(v[22]), "f"(v[23]), "f"(v[24]),
      "f"(v[25]), "f"(v[26]), "f"(v[27]), "f"(v[28]), "f"(v[29]), "f"(v[30]), "f"(v[31])
      : "memory");
}

__device__ __forceinline__ void tma_store_2d(const CUtensorMap* map, int32_t x, int32_t y, const void* src) {
  asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%1, %2}], [%3];" ::"l"((uint64_t)map),
               "r"(x), "r"(y), "r"(saddr(src))
               : "memory");
}

__device__ __forceinline__ float div_q(float a, float b, float y) {   // = kernels_chol.cu div_rcp
  const float q0 = __fmul_rn(a, y);
  const float r = __fmaf_rn(-b, q0, a);
  return __fmaf_rn(r, y, q0);
}

__global__ void __launch_bounds__(kTcThreads, 1)
    trsm_col(float* __restrict__ A, const float* __restrict__ lt, const __grid_constant__ CUtensorMap tLhi,
             const __grid_constant__ CUtensorMap tLlo, const __grid_constant__ CUtensorMap tSx,
             const __grid_constant__ CUtensorMap tShi, const __grid_constant__ CUtensorMap tSlo,
             const __grid_constant__ ColJob job, const int* __restrict__ rowcnt, uint64_t* __restrict__ stamps) {
  extern __shared__ __align__(16) uint8_t smem_raw[];
  // 1024-B aligned (SWIZZLE_64B / 128B atoms), pointer arithmetic on the
  // shared array so the accesses stay LDS/STS
  uint8_t* base = smem_raw + ((1024u - (saddr(smem_raw) & 1023u)) & 1023u);
  uint8_t* ring = base + kSmRing;
  float* stg = reinterpret_cast<float*>(base + kSmStg);       // [3][128 rows][32] swizzled: x, hi, lo
  float* LsT = reinterpret_cast<float*>(base + kSmLt);        // packed leaf block (kLtU / kLtD / kLtRd)
  uint64_t* full = reinterpret_cast<uint64_t*>(base + kSmBar);
  uint64_t* empty = full + kTcStages;
  uint64_t* tfull = empty + kTcStages;        // [q] acc_q complete (MMA commit)
  uint64_t* xsub = tfull + kMaxLeaves;        // [4q+s] hi/lo of X_q sub-block s in TMEM (128 arrivals)
  uint64_t* xgl = xsub + 4 * kMaxLeaves;      // [q] X_q hi/lo in global (TMA stores complete)
  uint64_t* lsb = xgl + kMaxLeaves;           // [q] L block of leaf q in smem
  uint64_t* bful = lsb + kMaxLeaves;          // [2] B sub-block prefetch buffer loaded (tx)
  uint32_t* tslot = reinterpret_cast<uint32_t*>(bful + 2);
  float* bpre = reinterpret_cast<float*>(base + kSmBpre);    // [2][128 rows][32] swizzled: B sub-blocks
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nleaf = job.nleaf;
  const int64_t b = job.b;
  const int32_t ti = job.ti[blockIdx.y];
  const int32_t r0 = (int32_t)blockIdx.x * kTcRows;                        // rows of the tile
  const int32_t ya = (job.slot0 + ti) * (int32_t)b + r0;                   // panel slot rows (X_i)
  const int32_t yl = (job.slot0 + job.k) * (int32_t)b;                     // L_kk slot rows
  const int32_t yx = (int32_t)(((int64_t)ti * job.T + job.k) * b) + r0;    // rows of A (tile (ti, k))
  const bool issuer = threadIdx.x == 64;                                   // warp 2 lane 0

  if (threadIdx.x == 0) {
    for (int s = 0; s < kTcStages; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], 1);
    }
    for (int q = 0; q < kMaxLeaves; ++q) {
      mbar_init(&tfull[q], 1);
      mbar_init(&xgl[q], 1);
      mbar_init(&lsb[q], 1);
      for (int u = 0; u < 4; ++u) mbar_init(&xsub[4 * q + u], 256);
    }
    mbar_init(&bful[0], 1);
    mbar_init(&bful[1], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tLhi) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tLlo) : "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(saddr(tslot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = *tslot;
  uint64_t* stp = stamps ? stamps + ((int64_t)blockIdx.y * gridDim.x + blockIdx.x) * kStampsPerCta : nullptr;
  auto stamp = [&](int i) {
    if (stp) {
      uint64_t t;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
      stp[i] = t;
    }
  };
  if (threadIdx.x == 0) stamp(0);

  if (warp == 0) {
    if (lane == 0) {   // ===== TMA producer
      int it = 0;
      for (int q = 1; q < nleaf; ++q) {
        const int32_t yb = yl + q * kTcLeaf;
        wait_rows(rowcnt, q);   // L_qj (j < q): row block q of L_kk
        for (int j = 0; j <= q - 1; ++j) {
          const bool ts = j == q - 1;                 // X_{q-1} comes from TMEM
          if (!ts && j == q - 2) twait(&xgl[j], 0);   // X_j of this CTA's leaf j is in global memory
          for (int kb = 0; kb < kTcLeaf / kTcBK; ++kb, ++it) {
            const int s = it % kTcStages;
            if (it >= kTcStages) twait(&empty[s], (uint32_t)(((it / kTcStages) - 1) & 1));
            uint8_t* st = ring + s * kTcStageBytes;
            const int32_t kx = j * kTcLeaf + kb * kTcBK;
            mbar_expect_tx(&full[s], ts ? 2 * kTcOpBytes : kTcStageBytes);
            if (!ts) {
              tma_load_2d(st, &tLhi, kx, ya, &full[s]);
              tma_load_2d(st + kTcOpBytes, &tLlo, kx, ya, &full[s]);
            }
            tma_load_2d(st + 2 * kTcOpBytes, &tLhi, kx, yb, &full[s]);
            tma_load_2d(st + 3 * kTcOpBytes, &tLlo, kx, yb, &full[s]);
          }
        }
      }
    }
    __syncwarp();
  } else if (warp == 1) {
    if (lane == 0) {   // ===== MMA issuer
      const uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(kTcLeaf >> 3) << 17) |
                             ((uint32_t)(kTcRows >> 4) << 24);
      int it = 0;
      for (int q = 1; q < nleaf; ++q) {
        const uint32_t acc = tmem + (uint32_t)((q & 1) * 128);
        if (q >= 2) {   // leaf q-2 no longer reads accumulator q%2 (its last sub-block is stored)
          twait(&xsub[4 * (q - 2) + 3], 0);
          asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        }
        bool first = true;
        if (q < 8) stamp(17 + q);
        for (int j = 0; j <= q - 2; ++j) {   // SS terms: X_j from the panel slot
          for (int kb = 0; kb < kTcLeaf / kTcBK; ++kb, ++it) {
            const int s = it % kTcStages;
            twait(&full[s], (uint32_t)((it / kTcStages) & 1));
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
            uint8_t* st = ring + s * kTcStageBytes;
            const uint64_t ahi = sdesc(st), alo = sdesc(st + kTcOpBytes);
            const uint64_t bhi = sdesc(st + 2 * kTcOpBytes), blo = sdesc(st + 3 * kTcOpBytes);
#pragma unroll
            for (int kk = 0; kk < kTcBK / 8; ++kk) {
              const uint64_t adv = (uint64_t)(kk * 32) >> 4;
              mma_tf32(acc, alo + adv, bhi + adv, idesc, first ? 0u : 1u);
              first = false;
              mma_tf32(acc, ahi + adv, blo + adv, idesc, 1u);
              mma_tf32(acc, ahi + adv, bhi + adv, idesc, 1u);
            }
            mma_commit(&empty[s]);
          }
        }
        // TS term j = q-1, one 32-column sub-block of X_{q-1} at a time as the
        // substitution produces it (TMEM: hi at 256 + 32u, lo at 384 + 32u)
        for (int u = 0; u < 4; ++u) {
          twait(&xsub[4 * (q - 1) + u], 0);
          asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
          if (u == 0 && q < 8) stamp(25 + q);
          const uint32_t xh = tmem + 256u + (uint32_t)(32 * u);
          for (int h = 0; h < 2; ++h, ++it) {
            const int s = it % kTcStages;
            twait(&full[s], (uint32_t)((it / kTcStages) & 1));
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
            uint8_t* st = ring + s * kTcStageBytes;
            const uint64_t bhi = sdesc(st + 2 * kTcOpBytes), blo = sdesc(st + 3 * kTcOpBytes);
#pragma unroll
            for (int kk = 0; kk < kTcBK / 8; ++kk) {
              const uint64_t adv = (uint64_t)(kk * 32) >> 4;
              const uint32_t ahi = xh + (uint32_t)(16 * h + 8 * kk), alo = ahi + 128u;
              mma_ts(acc, alo, bhi + adv, idesc, first ? 0u : 1u);
              first = false;
              mma_ts(acc, ahi, blo + adv, idesc, 1u);
              mma_ts(acc, ahi, bhi + adv, idesc, 1u);
            }
            mma_commit(&empty[s]);
          }
        }
        mma_commit(&tfull[q]);
        if (q < 8) stamp(33 + q);
      }
    }
    __syncwarp();
  } else {   // ===== substitution: warps 2..9, row = TMEM lane, two warps per row group
    // (warps w and w + 4 share TMEM lanes 32 (w % 4) ..: half hf = 0 / 1 takes
    // columns 16 hf .. 16 hf + 15 of every sub-block)
    const int grp = warp & 3, rr = grp * 32 + lane, hf = (warp - 2) >> 2, cb = 16 * hf;
    const uint32_t lane_off = (uint32_t)(grp * 32) << 16;
    const float* brow = A + ((int64_t)yx + rr) * b;   // this row of tile (ti, k): B, then X
    const float* rd = LsT + kLtRd;
    // B sub-blocks (32 columns x 128 rows of the tile) through a double
    // buffer, TMA-loaded one sub-block ahead by the issuer
    auto bload = [&](int idx) {   // idx = 4 q + s
      if (idx >= 4 * nleaf) return;
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      mbar_expect_tx(&bful[idx & 1], kStgBytes);
      tma_load_2d(bpre + (idx & 1) * 4096, &tSx, 32 * idx, yx, &bful[idx & 1]);
    };
    if (issuer) {   // LsT of leaf 0
      wait_rows(rowcnt, 0);
      mbar_expect_tx(&lsb[0], kLtBytes);
      asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                       saddr(LsT)),
                   "l"(lt), "r"(kLtBytes), "r"(saddr(&lsb[0]))
                   : "memory");
    }
    if (issuer) bload(0);
    int pending = -1;   // leaf whose TMA stores the issuer has not waited for yet
#pragma unroll 1
    for (int q = 0; q < nleaf; ++q) {
      const int c0 = q * kTcLeaf;
      const uint32_t accq = tmem + (uint32_t)((q & 1) * 128) + lane_off;
      twait(&lsb[q], 0);
      if (q >= 1) {
        twait(&tfull[q], 0);
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
      }
      if (issuer && q < 8) stamp(1 + q);
#pragma unroll 1
      for (int s = 0; s < 4; ++s) {
        const int idx = 4 * q + s;
        if (issuer) bload(idx + 1);
        twait(&bful[idx & 1], (uint32_t)((idx >> 1) & 1));
        float x[16];
        {
          const float* bp = bpre + (idx & 1) * 4096 + rr * 32;
#pragma unroll
          for (int v = 0; v < 4; ++v) {
            const float4 t = *reinterpret_cast<const float4*>(bp + (((4 * hf + v) ^ (rr & 7)) * 4));
            x[4 * v] = t.x; x[4 * v + 1] = t.y; x[4 * v + 2] = t.z; x[4 * v + 3] = t.w;
          }
        }
        if (q >= 1) {   // x = B - sum_{j<q} X_j L_qj^T
          float a[16];
          tmem_ld16(accq + (uint32_t)(32 * s + cb), a);
#pragma unroll
          for (int c = 0; c < 16; ++c) x[c] -= a[c];
        }
        if (s > 0) {   // earlier sub-blocks of this leaf: accumulate ascending, subtract once
          float acc[16];
#pragma unroll
          for (int c = 0; c < 16; ++c) acc[c] = 0.f;
#pragma unroll 1
          for (int m0 = 0; m0 < 32 * s; m0 += 16) {
            float xm[16];
            tmem_ld16(accq + (uint32_t)m0, xm);
#pragma unroll
            for (int i = 0; i < 16; ++i) {
              const float4* l4 = reinterpret_cast<const float4*>(
                  LsT + kLtU + (s * (s - 1) / 2 + (m0 >> 5)) * 1024 + ((m0 & 31) + i) * 32 + cb);
#pragma unroll
              for (int u = 0; u < 4; ++u) {
                const float4 l = l4[u];
                acc[4 * u + 0] = fmaf(xm[i], l.x, acc[4 * u + 0]);
                acc[4 * u + 1] = fmaf(xm[i], l.y, acc[4 * u + 1]);
                acc[4 * u + 2] = fmaf(xm[i], l.z, acc[4 * u + 2]);
                acc[4 * u + 3] = fmaf(xm[i], l.w, acc[4 * u + 3]);
              }
            }
          }
#pragma unroll
          for (int c = 0; c < 16; ++c) x[c] -= acc[c];
        }
        // the 32-column substitution: half 0 solves columns 0..15 and hands
        // them over through TMEM (fp32, the consumed accumulator columns);
        // half 1 applies them, then solves 16..31 — the operations and their
        // order are those of one thread doing all 32
        const float* Ds = LsT + kLtD + s * 1024;   // Ds[c * 32 + c2] = L[c0+32s+c2][c0+32s+c]
        if (hf == 0) {
#pragma unroll
          for (int c = 0; c < 16; ++c) {
            x[c] = div_q(x[c], Ds[c * 32 + c], rd[32 * s + c]);
#pragma unroll
            for (int c2 = c + 1; c2 < 16; ++c2) x[c2] -= x[c] * Ds[c * 32 + c2];
          }
          tmem_st16(accq + (uint32_t)(32 * s), x);
          asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
          asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
        }
        // the row group's two warps meet at ONE barrier instruction (per-warp
        // aligned barriers reached from two code sites count as divergent)
        asm volatile("bar.sync %0, 64;" ::"r"(2 + grp) : "memory");
        if (hf == 1) {
          asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
          float x0[16];
          tmem_ld16(accq + (uint32_t)(32 * s), x0);
#pragma unroll
          for (int i = 0; i < 16; ++i)
#pragma unroll
            for (int c = 0; c < 16; ++c) x[c] -= x0[i] * Ds[i * 32 + 16 + c];
#pragma unroll
          for (int c = 0; c < 16; ++c) {
            x[c] = div_q(x[c], Ds[(16 + c) * 32 + 16 + c], rd[32 * s + 16 + c]);
#pragma unroll
            for (int c2 = c + 1; c2 < 16; ++c2) x[c2] -= x[c] * Ds[(16 + c) * 32 + 16 + c2];
          }
          tmem_st16(accq + (uint32_t)(32 * s + 16), x);
        }
        // hi/lo to TMEM columns 256 / 384 + 32 s (their previous contents, X_{q-1},
        // were read by acc_q's MMAs, complete before tfull[q])
        const uint32_t xslot = tmem + 256u + lane_off + (uint32_t)(32 * s);
        // staging (SWIZZLE_128B: 16-B chunk u of row r at chunk u ^ (r & 7)) -> TMA stores
        if (issuer) {
          if (pending >= 0) {   // the previous leaf's stores: complete, so the producer may load them
            asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
            asm volatile("fence.proxy.async.global;" ::: "memory");
            mbar_arrive(&xgl[pending]);
            pending = -1;
          } else {
            asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
          }
        }
        asm volatile("bar.sync 1, 256;" ::: "memory");
        {
          float h[16], l[16];
#pragma unroll
          for (int c = 0; c < 16; ++c) {
            h[c] = tf32_rn(x[c]);
            l[c] = tf32_rn(x[c] - h[c]);
          }
          tmem_st16(xslot + (uint32_t)cb, h);
          tmem_st16(xslot + 128u + (uint32_t)cb, l);
#pragma unroll
          for (int v = 0; v < 4; ++v) {
            const int u = 4 * hf + v, off = rr * 32 + ((u ^ (rr & 7)) * 4);
            *reinterpret_cast<float4*>(stg + off) = make_float4(x[4 * v], x[4 * v + 1], x[4 * v + 2], x[4 * v + 3]);
            *reinterpret_cast<float4*>(stg + 4096 + off) = make_float4(h[4 * v], h[4 * v + 1], h[4 * v + 2], h[4 * v + 3]);
            *reinterpret_cast<float4*>(stg + 8192 + off) = make_float4(l[4 * v], l[4 * v + 1], l[4 * v + 2], l[4 * v + 3]);
          }
        }
        asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
        asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
        mbar_arrive(&xsub[4 * q + s]);   // acc_{q+1}'s MMAs may read this sub-block
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        asm volatile("bar.sync 1, 256;" ::: "memory");
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");   // the other half's x columns
        if (issuer) {
          const int32_t xc = c0 + 32 * s;
          tma_store_2d(&tSx, xc, yx, stg);
          tma_store_2d(&tShi, xc, ya, stg + 4096);
          tma_store_2d(&tSlo, xc, ya, stg + 8192);
          asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        }
      }
      // leaf q done: LsT free, accumulator q%3 free after the x reads above
      if (issuer && q < 8) stamp(9 + q);
      asm volatile("bar.sync 1, 256;" ::: "memory");
      if (issuer) {
        pending = q;
        if (q + 1 < nleaf) {
          wait_rows(rowcnt, q + 1);
          asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
          mbar_expect_tx(&lsb[q + 1], kLtBytes);
          asm volatile(
              "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                  saddr(LsT)),
              "l"(lt + (int64_t)(q + 1) * kLtFloats), "r"(kLtBytes), "r"(saddr(&lsb[q + 1]))
              : "memory");
        }
      }
    }
    if (issuer) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    if (issuer) stamp(41);
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (warp == 1) {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tmem));
  }
}

// Per step: L_kk split into its panel slot (hi/lo, = split_tiles) and, per
// leaf q, LsT_q[m][c] = L[c0+c][c0+m] (c0 = 128 q) followed by RN(1/L[c0+m][c0+m]).
__global__ void __launch_bounds__(256) lkk_prep(const float* __restrict__ L, float* __restrict__ hi,
                                                float* __restrict__ lo, float* __restrict__ lt, int b, int nsplit) {
  __shared__ float t[32][33];
  if ((int)blockIdx.x < nsplit) {
    const int64_t n4 = (int64_t)b * b / 4;
    for (int64_t e = (int64_t)blockIdx.x * 256 + threadIdx.x; e < n4; e += (int64_t)nsplit * 256) {
      const float4 x = reinterpret_cast<const float4*>(L)[e];
      float4 h, l;
      split2(x.x, h.x, l.x);
      split2(x.y, h.y, l.y);
      split2(x.z, h.z, l.z);
      split2(x.w, h.w, l.w);
      reinterpret_cast<float4*>(hi)[e] = h;
      reinterpret_cast<float4*>(lo)[e] = l;
    }
    return;
  }
  const int idx = (int)blockIdx.x - nsplit, q = idx / 16, mi = (idx % 16) / 4, ci = idx % 4;
  if (mi > ci) return;   // blocks above L's diagonal are never read
  const int c0 = q * kTcLeaf, tx = threadIdx.x & 31, ty = threadIdx.x >> 5;
  float* dst = lt + (int64_t)q * kLtFloats + (mi < ci ? kLtU + (ci * (ci - 1) / 2 + mi) * 1024 : kLtD + ci * 1024);
#pragma unroll
  for (int j = ty; j < 32; j += 8)   // t[c][m] = L[c0 + 32ci + c][c0 + 32mi + m]
    t[j][tx] = L[(int64_t)(c0 + 32 * ci + j) * b + c0 + 32 * mi + tx];
  __syncthreads();
#pragma unroll
  for (int j = ty; j < 32; j += 8)   // [j][tx] = L[c0 + 32ci + tx][c0 + 32mi + j]
    dst[j * 32 + tx] = t[tx][j];
  if (mi == ci && threadIdx.x < 32)
    lt[(int64_t)q * kLtFloats + kLtRd + 32 * mi + tx] = __frcp_rn(t[tx][tx]);
}

}  // namespace

// MM_TRSM_STAMPS=<file> (diagnostics; eager launches only): every launch
// appends one line per CTA: k, cta, then the globaltimer stamps relative to
// the CTA's start: leaf q start (1..8), leaf q end (9..16), acc_q MMA start
// (17..24), TS term start (25..32), commit (33..40), CTA end (41).
static uint64_t* trsm_stamps_buffer(cudaStream_t s, size_t n) {
  static const char* path = getenv("MM_TRSM_STAMPS");
  if (!path) return nullptr;
  cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
  cudaStreamIsCapturing(s, &cs);
  if (cs != cudaStreamCaptureStatusNone) return nullptr;
  static uint64_t* buf = nullptr;
  static size_t cap = 0;
  if (n > cap) {
    if (buf) cudaFree(buf);
    if (cudaMalloc(&buf, n * 8) != cudaSuccess) return nullptr;
    cap = n;
  }
  cudaMemsetAsync(buf, 0, n * 8, s);
  return buf;
}
static void trsm_stamps_dump(cudaStream_t s, const uint64_t* d, int gx, int gy, int k) {
  const size_t n = (size_t)gx * gy * kStampsPerCta;
  std::vector<uint64_t> h(n);
  cudaStreamSynchronize(s);
  cudaMemcpy(h.data(), d, n * 8, cudaMemcpyDeviceToHost);
  FILE* f = fopen(getenv("MM_TRSM_STAMPS"), "a");
  if (!f) return;
  for (int c = 0; c < gx * gy; ++c) {
    const uint64_t* r = h.data() + (size_t)c * kStampsPerCta;
    fprintf(f, "%d,%d", k, c);
    for (int i = 1; i <= 41; ++i) fprintf(f, ",%.3f", r[i] ? (double)(int64_t)(r[i] - r[0]) * 1e-3 : -1.0);
    fprintf(f, "\n");
  }
  fclose(f);
}

size_t chol_trsm_lt_bytes(int64_t b) { return (size_t)(b / kTcLeaf) * kLtBytes; }

bool chol_trsm_overlap_enabled() {
  static const int env = getenv("MM_TRSM_OVERLAP") ? atoi(getenv("MM_TRSM_OVERLAP")) : 1;
  return env != 0;
}

bool chol_trsm_col_enabled() {
  static const int env = getenv("MM_TRSM_COL") ? atoi(getenv("MM_TRSM_COL")) : 1;
  return env != 0;
}

// One launch per batch; the step's L_kk preparation once per step and device
// (split tag of slot k, as chol_trsm_prepare).
cudaError_t chol_trsm_col(float* A, int64_t T, int64_t b, int32_t k, const int32_t* ti, int32_t n, cudaStream_t s,
                          Scratch* scr) {
  if (n <= 0) return cudaSuccess;
  if (b % kTcLeaf != 0 || b / kTcLeaf > kMaxLeaves || b < 2 * kTcLeaf) return cudaErrorNotSupported;
  if (!scr || !scr->ptr || scr->bytes < chol_scratch_bytes(T, b)) return cudaErrorNotSupported;
  float* hi = static_cast<float*>(scr->ptr);
  float* lo = hi + 2 * T * b * b;
  float* lt = reinterpret_cast<float*>(static_cast<char*>(scr->ptr) + chol_tc_scratch(T, b) +
                                       chol_potrf_flag_bytes(b));
  const int32_t slot0 = (k & 1) * (int32_t)T;
  static std::atomic<uint64_t> attr{0};
  cudaError_t e = once_per_device(attr, [] {
    return cudaFuncSetAttribute(trsm_col, cudaFuncAttributeMaxDynamicSharedMemorySize, kTcSmem);
  });
  if (e != cudaSuccess) return e;
  if (scr->panel.size() != (size_t)(2 * T)) scr->panel.assign(2 * T, 0);
  const uint64_t tag = (scr->epoch << 20) | (uint64_t)(k + 1);   // = kernels_gemm_tc.cu split_tag
  // the step's POTRF ran right before on this stream and wrote L_kk's split
  // and packed leaves itself: overlap it (PDL launch, per-leaf row counts)
  const bool overlap = chol_trsm_overlap_enabled() && scr->potrf_k == k && scr->potrf_stream == (const void*)s &&
                       scr->potrf_epoch == scr->epoch;
  const int* rowcnt = overlap ? chol_potrf_rowcnt(scr, T, b) : nullptr;
  if (overlap) scr->panel[slot0 + k] = tag;
  if (scr->panel[slot0 + k] != tag) {
    scr->panel[slot0 + k] = tag;
    const int nsplit = 64;
    note_launch();
    lkk_prep<<<(unsigned)(nsplit + (b / kTcLeaf) * 16), 256, 0, s>>>(A + ((int64_t)k * T + k) * b * b,
                                                                     hi + (slot0 + k) * b * b,
                                                                     lo + (slot0 + k) * b * b, lt, (int)b, nsplit);
    if ((e = cudaGetLastError()) != cudaSuccess) return e;
  }
  CUtensorMap mLhi, mLlo, mSx, mShi, mSlo;
  if ((e = encode_tmap_2d_f32(&mLhi, hi, b, 2 * T * b, b * 4, kTcBK, kTcRows)) != cudaSuccess) return e;
  if ((e = encode_tmap_2d_f32(&mLlo, lo, b, 2 * T * b, b * 4, kTcBK, kTcRows)) != cudaSuccess) return e;
  if ((e = encode_tmap_2d_f32(&mSx, A, b, T * T * b, b * 4, 32, kTcRows)) != cudaSuccess) return e;
  if ((e = encode_tmap_2d_f32(&mShi, hi, b, 2 * T * b, b * 4, 32, kTcRows)) != cudaSuccess) return e;
  if ((e = encode_tmap_2d_f32(&mSlo, lo, b, 2 * T * b, b * 4, 32, kTcRows)) != cudaSuccess) return e;
  ColJob job;
  job.k = k;
  job.slot0 = slot0;
  job.nleaf = (int32_t)(b / kTcLeaf);
  job.T = T;
  job.b = b;
  for (int32_t q0 = 0; q0 < n; q0 += kCholBatch) {
    job.n = std::min<int32_t>(kCholBatch, n - q0);
    for (int32_t q = 0; q < job.n; ++q) job.ti[q] = ti[q0 + q];
    uint64_t* stamps = trsm_stamps_buffer(s, (size_t)(b / kTcRows) * job.n * kStampsPerCta);
    note_launch();
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)(b / kTcRows), (unsigned)job.n);
    cfg.blockDim = dim3(kTcThreads);
    cfg.dynamicSmemBytes = kTcSmem;
    cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = rowcnt ? 1 : 0;
    if ((e = cudaLaunchKernelEx(&cfg, trsm_col, A, (const float*)lt, mLhi, mLlo, mSx, mShi, mSlo, job, rowcnt,
                                stamps)) != cudaSuccess)
      return e;
    if (stamps) trsm_stamps_dump(s, stamps, (int)(b / kTcRows), job.n, k);
  }
  for (int32_t q = 0; q < n; ++q) scr->panel[slot0 + ti[q]] = tag;
  return cudaSuccess;
}

}  // namespace mm
