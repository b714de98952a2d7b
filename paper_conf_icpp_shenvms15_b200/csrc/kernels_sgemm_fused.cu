// Small-SGEMM path of MatrixMul (BASELINE configs[0], 1024^2; P311 C = A x B,
// row-wise split): fused kernels with no reduction pass.  Three variants
// (MM_SGEMM_FUSED = 1 / 2 / 3, default 3):
//  3  split_bT (kernels_gemm_tc.cu) writes B_hi^T / B_lo^T once, then
//     sgemm_fused2: single-SM 128 x 256 tiles (tcgen05 M = 128, N = 256), S = 4
//     K splits per cluster; TMA brings raw A and the split B, the converter
//     warps only split A into TMEM.  1024^2: split_bT 4.9 us + sgemm_fused2
//     19.0 us (ncu, serialised; PDL overlaps them in the stream), bench step
//     30.2 us.  globaltimer: main loop 7.6 us for 16 k-steps (~82 % of the
//     MMA time), TMEM -> smem 1.5 us, cluster barrier 0.8 us, DSMEM reduction
//     of 4 partials 3.9 us.
//  2  sgemm_fused1: the same tiles with B transposed and split in-kernel by
//     the converter warps (25.4 us: the B transposition keeps the main loop
//     at ~15 us).
//  1  the pair design below (25.3 us).
// Variant 1, the original fused kernel, in ONE launch: no operand-split pass.
//
// A cluster of 2 S CTAs computes one 256 x 128 output tile pair over S K
// splits (S in 2..4, the largest whose clusters are all resident at once):
// CTA rank r = 2 z + h is half h (128 rows) of the 2-SM pair (tcgen05
// cta_group::2) of K split z (k-blocks [z nkb / S, (z+1) nkb / S)).
//  warp 0      TMA producer: RAW fp32 tiles straight from A (row-major,
//              K-major: box 16 x 128 rows, SWIZZLE_64B) and B (row-major: two
//              boxes of 32 columns x 16 k-rows, SWIZZLE_128B) into a 12-stage
//              raw ring (L2/HBM latency).
//  warps 2-9   two groups of four converter warps, alternating k-steps:
//              x -> hi = tf32_rn(x), lo = tf32_rn(x - hi) (the split of the
//              two-pass path); A rows (thread = TMEM lane) straight into 32
//              TMEM columns per stage (tcgen05.st), B transposed into the
//              K-major SWIZZLE_64B layout of the two-pass path's B^T in a
//              4-stage smem ring (an MN-major B descriptor read zeros on this
//              B200); one arrival per warp on the leader CTA's barrier.
//  warp 1      (leader CTA) tcgen05.mma.cta_group::2.kind::tf32 with A from
//              TMEM, B from smem: 3 MMAs per k-step (lo.hi + hi.lo + hi.hi)
//              into a 128-column TMEM accumulator; commits free the stages.
//  epilogue    the converter warps: TMEM -> registers -> this CTA's smem
//              (padded rows); cluster barrier; CTA z sums float4 columns
//              [z 32 / S, (z+1) 32 / S) of its 128 rows over the S partials
//              in split order ((p0 + p1) + p2) + p3 by distributed-shared-
//              memory loads from its cluster peers and stores C; cluster
//              barrier before exit.
// 1024^2 (S = 2, 128 CTAs in clusters of 4): 23.5 us (ncu, cold) against 33 us
// for the split -> GEMM -> reduce chain.  globaltimer stamps: set-up 0.8 us,
// first MMA at 1.9 us, ~490 ns per k-step (the converters of both CTAs run
// 2-3 steps ahead), reduction ~4 us (DSMEM moves ~20 B/clk per SM).  The 6
// MMAs of a k-step need 384 clk at the measured full rate (tools/mma_rates.cu:
// 64 clk per 256 x 128 x 8 pair MMA, TS or SS, also with streamed operand
// stages); the rest of the ~940 clk per k-step is per-step overhead that
// neither an 8-stage split ring, 4 converter groups, two stages per
// wait/commit round, the MMA warp as the highest warp id of its
// sub-partition nor issuing without waiting for split_full removed (all
// measured unchanged; doubling the MMAs of a step added exactly their 64 clk
// each).  Issuing all 192 MMAs without any wait still takes 14.5 us (~148 clk
// per MMA) here, while the microbenchmark of the same issue pattern (pair, TS,
// streamed stages, fence + multicast commit per step) runs at 79 clk and at
// 96 clk with three warps per CTA storing to TMEM beside it.
// Tried and dropped: 256-wide pairs with S = 3 (24.9 us, both operands in
// smem: 26 us), a cp.async.bulk push of the partial slices and a reduction
// through L2 (both slower than the DSMEM pull).
#include <cuda.h>

#include <algorithm>
#include <atomic>
#include <cstdlib>

#include "kernels.h"
#include "tc_ptx.h"

namespace mm {

cudaError_t encode_tmap_2d_f32(CUtensorMap* m, const void* base, uint64_t inner, uint64_t outer,
                               uint64_t row_bytes, uint32_t box_inner, uint32_t box_outer);

namespace {

using namespace tcx;

constexpr int FBM = 128, FBK = 16, FHALF = 64;                 // rows per CTA, k per stage, B columns per CTA
constexpr int FBN = 2 * FHALF;                                 // output columns of a tile pair (MMA N)
// warps: 0 producer, 1 MMA issuer, 2.. kConvGroups groups of 4 converter warps
// (group g converts the stages i with i % kConvGroups == g: a converter's
// per-stage chain — smem loads, split, TMEM stores + wait, arrive — is
// latency-bound, so two groups alternate)
constexpr int kConvGroups = 2;
// The raw ring is deep: its TMA loads come from L2/HBM (~1 us), and a 4-stage
// ring bounded a k-step to latency / 4 (measured 470 ns per k-step).
constexpr int kRawStages = 12, kSplitStages = 4, kFThreads = 64 + 128 * kConvGroups;
constexpr int RAW_A = FBM * FBK * 4, RAW_B = FHALF * FBK * 4;  // 8 KB + 4 KB
constexpr int RAW_BYTES = RAW_A + RAW_B;
constexpr int SPLIT_BYTES = 2 * RAW_B;                         // B_hi, B_lo (A_hi, A_lo go to TMEM)
constexpr int kRingBytes = kRawStages * RAW_BYTES + kSplitStages * SPLIT_BYTES;   // 192 KB
constexpr int RED_LD = FBN + 4;        // padded fp32 row of the partial (reuses the drained rings)
constexpr int kTmemCols = 256;         // FBN accumulator columns + kSplitStages x 32 A columns
static_assert(FBN + kSplitStages * 32 <= kTmemCols, "TMEM columns");
constexpr int kFusedSmem = kRingBytes + 1024 + 256;
static_assert(FBM * RED_LD * 4 <= kRingBytes, "partial buffer");

// arrive on the barrier of cluster peer `rank` (default .release.cta
// semantics, as CUTLASS's ClusterBarrier::arrive(cta_id): a .cluster-scope
// release compiles to a GPU-wide MEMBAR per arrival)
__device__ __forceinline__ void arrive_remote(uint64_t* bar, uint32_t rank) {
  asm volatile("mbarrier.arrive.shared::cluster.b64 _, [%0];" ::"r"(peer_addr(bar, rank)) : "memory");
}

__device__ __forceinline__ void cluster_arrive_relaxed_wait() {
  asm volatile("barrier.cluster.arrive.relaxed.aligned;\n barrier.cluster.wait.aligned;" ::: "memory");
}

// tcgen05.commit of the pair's MMAs: arrive on `bar` in both CTAs of the pair
// (cluster ranks pair0, pair0 + 1)
__device__ __forceinline__ void commit_pair_at(uint64_t* bar, uint32_t pair0) {
  asm volatile(
      "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
          saddr(bar)),
      "h"((uint16_t)(0x3u << pair0))
      : "memory");
}

// mbarrier wait that fails (trap -> launch error) instead of hanging if a
// phase never completes (a lost arrival would otherwise wedge the GPU)
template <bool CLUSTER = false>
__device__ __forceinline__ uint32_t try_wait(uint64_t* b, uint32_t parity) {
  uint32_t done;
  if (CLUSTER)
    asm volatile(
        "{\n .reg .pred p;\n mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 p, [%1], %2;\n"
        " selp.u32 %0, 1, 0, p;\n}\n"
        : "=r"(done)
        : "r"(saddr(b)), "r"(parity)
        : "memory");
  else
    asm volatile(
        "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
        : "=r"(done)
        : "r"(saddr(b)), "r"(parity)
        : "memory");
  return done;
}

template <bool CLUSTER = false>
__device__ __forceinline__ void fwait(uint64_t* b, uint32_t parity) {
  if (try_wait<CLUSTER>(b, parity)) return;
  uint64_t t0;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  for (;;) {
    if (try_wait<CLUSTER>(b, parity)) return;
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    if (t - t0 > 4000000000ull) __trap();
  }
}

// 3xTF32 pair MMA with A read from tensor memory (TS form), B from smem
__device__ __forceinline__ void mma_tf32_pair_ts(uint32_t tmem_d, uint32_t tmem_a, uint64_t b, uint32_t idesc,
                                                 uint32_t acc) {
  asm volatile(
      "{\n .reg .pred p;\n setp.ne.b32 p, %4, 0;\n"
      " tcgen05.mma.cta_group::2.kind::tf32 [%0], [%1], %2, %3, p;\n}\n" ::"r"(tmem_d),
      "r"(tmem_a), "l"(b), "r"(idesc), "r"(acc));
}

// 16 consecutive 32-bit TMEM columns of this thread's lane
__device__ __forceinline__ void tmem_st16(uint32_t taddr, const float (&v)[16]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};" ::"r"(
          taddr),
      "f"(v[0]), "f"(v[1]), "f"(v[2]), "f"(v[3]), "f"(v[4]), "f"(v[5]), "f"(v[6]), "f"(v[7]), "f"(v[8]), "f"(v[9]),
      "f"(v[10]), "f"(v[11]), "f"(v[12]), "f"(v[13]), "f"(v[14]), "f"(v[15])
      : "memory");
}

__device__ __forceinline__ float4 ld_dsmem_f4(uint32_t addr) {
  float4 v;
  asm volatile("ld.shared::cluster.v4.f32 {%0, %1, %2, %3}, [%4];"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w)
               : "r"(addr)
               : "memory");
  return v;
}

// One 256 x 256 tile pair, K split z of S (k-blocks [z nkb / S, (z+1) nkb / S));
// cluster = 2 S CTAs.
__global__ void __launch_bounds__(kFThreads, 1)
    sgemm_fused(const __grid_constant__ CUtensorMap tA, const __grid_constant__ CUtensorMap tB, float* __restrict__ C,
                int64_t N, int64_t row0, int64_t mrows, int nblk, int S, int nkb_all) {
  uint32_t rank;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(rank));
  const uint32_t h = rank & 1u, z = rank >> 1;
  const bool leader = h == 0;
  const int cl = (int)(blockIdx.x / (2 * S));
  const int mp = cl / nblk, nb = cl % nblk;
  const int m_blk = 2 * mp + (int)h;
  const int kb0 = (int)z * nkb_all / S, nkb = ((int)z + 1) * nkb_all / S - kb0;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* base = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* raw = base;
  uint8_t* spl = base + kRawStages * RAW_BYTES;
  uint64_t* raw_full = reinterpret_cast<uint64_t*>(base + kRingBytes);
  uint64_t* raw_empty = raw_full + kRawStages;
  uint64_t* split_full = raw_empty + kRawStages;   // leader: the 4 converter warps of both CTAs
  uint64_t* split_empty = split_full + kSplitStages;
  uint64_t* tfull = split_empty + kSplitStages;
  uint32_t* tslot = reinterpret_cast<uint32_t*>(tfull + 1);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

  if (warp == 0 && lane == 0) {
    for (int s = 0; s < kRawStages; ++s) {
      mbar_init(&raw_full[s], 1);
      mbar_init(&raw_empty[s], 4);          // the 4 converter warps of this CTA
    }
    for (int s = 0; s < kSplitStages; ++s) {
      mbar_init(&split_full[s], 8);
      mbar_init(&split_empty[s], 1);        // the leader's commit, multicast
    }
    mbar_init(tfull, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tA) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tB) : "memory");
  }
  if (warp == 1) {
    // FBN accumulator columns + per split stage 32 columns of A (hi 16, lo 16)
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(saddr(tslot)), "n"(kTmemCols));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  cluster_arrive_relaxed_wait();   // peers' barriers initialised (fence.mbarrier_init above)
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = *tslot;
  asm volatile("griddepcontrol.wait;" ::: "memory");

  if (warp == 0) {
    if (lane == 0) {   // ===== producer: raw tiles of this CTA (own barrier)
      const int32_t ya = m_blk * FBM;
      const int32_t xb = nb * FBN + (int32_t)h * FHALF;
      for (int i = 0; i < nkb; ++i) {
        const int s = i % kRawStages;
        if (i >= kRawStages) fwait(&raw_empty[s], (uint32_t)(((i / kRawStages) - 1) & 1));
        uint8_t* st = raw + s * RAW_BYTES;
        const int32_t kx = (kb0 + i) * FBK;
        mbar_expect_tx(&raw_full[s], RAW_BYTES);
        tma_load_2d(st, &tA, kx, ya, &raw_full[s]);
#pragma unroll
        for (int j = 0; j < FHALF / 32; ++j) tma_load_2d(st + RAW_A + j * 2048, &tB, xb + 32 * j, kx, &raw_full[s]);
      }
    }
    __syncwarp();
  } else if (warp == 1) {
    if (lane == 0 && leader) {   // ===== MMA issuer
      const uint32_t idesc = (1u << 4)                 // D: fp32
                             | (2u << 7) | (2u << 10)  // A, B: tf32
                             | ((uint32_t)(FBN >> 3) << 17) | ((uint32_t)(256 >> 4) << 24);
      for (int i = 0; i < nkb; ++i) {
        const int s = i % kSplitStages;
        fwait(&split_full[s], (uint32_t)((i / kSplitStages) & 1));
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        uint8_t* st = spl + s * SPLIT_BYTES;
        const uint64_t bhi = sdesc(st), blo = sdesc(st + RAW_B);
        const uint32_t ahi = tmem + (uint32_t)FBN + (uint32_t)(s * 32), alo = ahi + 16u;   // A in TMEM columns
#pragma unroll
        for (int kk = 0; kk < FBK / 8; ++kk) {
          const uint64_t adv = (uint64_t)(kk * 32) >> 4;     // 8 fp32 along K inside B's 64-B row
          mma_tf32_pair_ts(tmem, alo + 8u * kk, bhi + adv, idesc, (i | kk) != 0);
          mma_tf32_pair_ts(tmem, ahi + 8u * kk, blo + adv, idesc, 1u);
          mma_tf32_pair_ts(tmem, ahi + 8u * kk, bhi + adv, idesc, 1u);
        }
        commit_pair_at(&split_empty[s], rank);
      }
      commit_pair_at(tfull, rank);
    }
    __syncwarp();
  } else {   // ===== converters, then the epilogue (warps 2..5)
    const int cg = (warp - 2) / 4;                // converter group
    const int ct = (threadIdx.x - 64) & 127;      // 0..127 within the group
    for (int i = cg; i < nkb; i += kConvGroups) {
      const int s = i % kRawStages, q = i % kSplitStages;
      fwait(&raw_full[s], (uint32_t)((i / kRawStages) & 1));
      if (i >= kSplitStages) fwait(&split_empty[q], (uint32_t)(((i / kSplitStages) - 1) & 1));
      const uint8_t* rs = raw + s * RAW_BYTES;
      uint8_t* dst = spl + q * SPLIT_BYTES;
      // A: row r = this thread's TMEM lane (warp w owns lanes 32 (w % 4) ..):
      // its 16 k of the raw K-major SWIZZLE_64B tile (chunk c of row r at
      // chunk c ^ ((r >> 1) & 3)), split, written to TMEM columns of slot q
      const int ar = (warp & 3) * 32 + lane;
      float4 v[4];
#pragma unroll
      for (int c = 0; c < 4; ++c)
        v[c] = *reinterpret_cast<const float4*>(rs + ar * 64 + ((c ^ ((ar >> 1) & 3)) << 4));
      // B: the raw tile is MN-major (4 boxes of 16 k-rows x 32 columns,
      // SWIZZLE_128B: 16-B chunk c of row k stored at chunk c ^ (k & 7)); it is
      // transposed into the K-major SWIZZLE_64B layout the MMA reads (row n =
      // 64 B of 16 k, chunk c stored at c ^ ((n >> 1) & 3)).  Output float4 o:
      // n = o & 127, k = 4 (o >> 7) .. +3; a warp reads 32 consecutive columns
      // of one raw row per load (conflict-free).
      constexpr int NB4 = FHALF * 4 / 128;   // B output float4 per converter thread
      float4 w[NB4];
#pragma unroll
      for (int j = 0; j < NB4; ++j) {
        const int o = ct + 128 * j, n = o % FHALF, k0 = 4 * (o / FHALF);
        const uint8_t* box = rs + RAW_A + (n >> 5) * 2048 + (n & 3) * 4;
        const int c16 = (n & 31) >> 2;
        float t[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const int k = k0 + u;
          t[u] = *reinterpret_cast<const float*>(box + k * 128 + ((c16 ^ (k & 7)) << 4));
        }
        w[j] = make_float4(t[0], t[1], t[2], t[3]);
      }
      {
        float ah[16], al[16];
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          split2(v[c].x, ah[4 * c], al[4 * c]);
          split2(v[c].y, ah[4 * c + 1], al[4 * c + 1]);
          split2(v[c].z, ah[4 * c + 2], al[4 * c + 2]);
          split2(v[c].w, ah[4 * c + 3], al[4 * c + 3]);
        }
        const uint32_t ta = tmem + ((uint32_t)((warp & 3) * 32) << 16) + (uint32_t)FBN + (uint32_t)(q * 32);
        tmem_st16(ta, ah);
        tmem_st16(ta + 16u, al);
      }
#pragma unroll
      for (int j = 0; j < NB4; ++j) {
        float4 hi, lo;
        const int o = ct + 128 * j, n = o % FHALF, kc4 = o / FHALF;
        const int boff = n * 64 + ((kc4 ^ ((n >> 1) & 3)) << 4);
        split2(w[j].x, hi.x, lo.x);
        split2(w[j].y, hi.y, lo.y);
        split2(w[j].z, hi.z, lo.z);
        split2(w[j].w, hi.w, lo.w);
        *reinterpret_cast<float4*>(dst + boff) = hi;
        *reinterpret_cast<float4*>(dst + RAW_B + boff) = lo;
      }
      asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");   // A in TMEM
      asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // B: generic writes -> tensor-core reads
      __syncwarp();
      if (lane == 0) {
        mbar_arrive(&raw_empty[s]);
        if (leader) mbar_arrive(&split_full[q]);
        else arrive_remote(&split_full[q], rank ^ 1u);
      }
    }
    // ---- epilogue: accumulator (TMEM lanes 32 grp .. +32 = this warp's rows)
    const int grp = warp & 3;
    fwait(tfull, 0);
    // the partial reuses the rings: every converter's raw-ring reads happened
    // before its stage arrival and so before the last MMA's commit (tfull);
    // the named barrier states it in a form compute-sanitizer's racecheck
    // follows (it does not model the tcgen05.commit arrival)
    asm volatile("bar.sync 1, %0;" ::"n"(128 * kConvGroups) : "memory");
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const int r = grp * 32 + lane;                       // row within the CTA's 128
    const int64_t grow = (int64_t)m_blk * FBM + r;       // row within [row0, row0 + mrows)
    float* red = reinterpret_cast<float*>(base);         // all rings drained: reuse for the partial
    for (int c = cg * (FBN / kConvGroups); c < (cg + 1) * (FBN / kConvGroups); c += 16) {
      uint32_t v[16];
      const uint32_t ta = tmem + ((uint32_t)(grp * 32) << 16) + (uint32_t)c;
      asm volatile(
          "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
          : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
            "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15])
          : "r"(ta));
      asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
      if (S > 1) {
#pragma unroll
        for (int q = 0; q < 4; ++q)
          *reinterpret_cast<float4*>(red + r * RED_LD + c + 4 * q) =
              make_float4(__uint_as_float(v[4 * q]), __uint_as_float(v[4 * q + 1]), __uint_as_float(v[4 * q + 2]),
                          __uint_as_float(v[4 * q + 3]));
      } else if (grow < mrows) {
        const int64_t n0 = (int64_t)nb * FBN + c;
        float* crow = C + (row0 + grow) * N;
#pragma unroll
        for (int q = 0; q < 4; ++q)
          if (n0 + 4 * q < N)
            *reinterpret_cast<float4*>(crow + n0 + 4 * q) =
                make_float4(__uint_as_float(v[4 * q]), __uint_as_float(v[4 * q + 1]),
                            __uint_as_float(v[4 * q + 2]), __uint_as_float(v[4 * q + 3]));
      }
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  }
  __syncthreads();
  if (S > 1) {
    cluster_sync_all();   // every partial of the cluster is in shared memory
    // CTA z reduces float4 columns [z FBN/4 / S, (z+1) FBN/4 / S) of its 128 rows:
    // the S partial loads of an element issued before the adds, summed in
    // split order ((p0 + p1) + p2) + p3; all 192 threads take part
    const int c4a = (int)z * (FBN / 4) / S, c4n = ((int)z + 1) * (FBN / 4) / S - c4a;
    const float* red = reinterpret_cast<const float*>(base);
    uint32_t peer[4];
#pragma unroll
    for (int zz = 0; zz < 4; ++zz) peer[zz] = peer_addr(red, (uint32_t)(2 * (zz < S ? zz : 0)) + h);
    for (int e = threadIdx.x; e < FBM * c4n; e += kFThreads) {
      const int rr = e / c4n, cc = 4 * (c4a + e % c4n);
      const uint32_t off = (uint32_t)((rr * RED_LD + cc) * 4);
      float4 p[4];
#pragma unroll
      for (int zz = 0; zz < 4; ++zz)
        if (zz < S) p[zz] = ld_dsmem_f4(peer[zz] + off);
      float4 a = p[0];
#pragma unroll
      for (int zz = 1; zz < 4; ++zz)
        if (zz < S) {
          a.x += p[zz].x; a.y += p[zz].y; a.z += p[zz].z; a.w += p[zz].w;
        }
      const int64_t grow = (int64_t)m_blk * FBM + rr, n0 = (int64_t)nb * FBN + cc;
      if (grow < mrows && n0 < N) *reinterpret_cast<float4*>(C + (row0 + grow) * N + n0) = a;
    }
    cluster_arrive_relaxed_wait();   // no CTA exits while a peer still reads its shared memory
  } else {
    cluster_sync_all();
  }
  if (warp == 1) {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem), "n"(kTmemCols));
  }
}

// ---------------------------------------------------------------------------
// Single-SM variant (round 2): one CTA = 128 rows x 256 columns (M = 128,
// N = 256 tcgen05.mma.cta_group::1, twice the work per instruction of the
// pair's 256 x 128), S K splits in a cluster of S CTAs reduced through DSMEM.
// Same stage pipeline: raw TMA ring -> converter warps (A to TMEM, B
// transposed into the K-major SWIZZLE_64B smem layout) -> MMA thread.
constexpr int G1N = 256;                                       // output columns per CTA (MMA N)
constexpr int RAW1_A = FBM * FBK * 4, RAW1_B = G1N * FBK * 4;  // 8 KB + 16 KB
constexpr int RAW1_BYTES = RAW1_A + RAW1_B;
constexpr int kRaw1 = 6, kSplit1 = 2;
constexpr int SPLIT1_BYTES = 2 * RAW1_B;                       // B_hi, B_lo
constexpr int kRing1 = kRaw1 * RAW1_BYTES + kSplit1 * SPLIT1_BYTES;   // 208 KB
constexpr int RED1_LD = G1N + 4;
constexpr int kTmem1 = 512;                                    // 256 accumulator + kSplit1 x 32 A columns
static_assert(G1N + kSplit1 * 32 <= kTmem1, "TMEM columns");
static_assert(FBM * RED1_LD * 4 <= kRing1, "partial buffer");
constexpr int kFused1Smem = kRing1 + 1024 + 256;

__device__ __forceinline__ void mma_tf32_ts1(uint32_t tmem_d, uint32_t tmem_a, uint64_t b, uint32_t idesc,
                                             uint32_t acc) {
  asm volatile(
      "{\n .reg .pred p;\n setp.ne.b32 p, %4, 0;\n"
      " tcgen05.mma.cta_group::1.kind::tf32 [%0], [%1], %2, %3, p;\n}\n" ::"r"(tmem_d),
      "r"(tmem_a), "l"(b), "r"(idesc), "r"(acc));
}

__global__ void __launch_bounds__(kFThreads, 1)
    sgemm_fused1(const __grid_constant__ CUtensorMap tA, const __grid_constant__ CUtensorMap tB, float* __restrict__ C,
                 int64_t N, int64_t row0, int64_t mrows, int nblk, int S, int nkb_all) {
  uint32_t z;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(z));
  const int cl = (int)(blockIdx.x / S);
  const int m_blk = cl / nblk, nb = cl % nblk;
  const int kb0 = (int)z * nkb_all / S, nkb = ((int)z + 1) * nkb_all / S - kb0;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* base = smem_raw + ((1024u - (saddr(smem_raw) & 1023u)) & 1023u);
  uint8_t* raw = base;
  uint8_t* spl = base + kRaw1 * RAW1_BYTES;
  uint64_t* raw_full = reinterpret_cast<uint64_t*>(base + kRing1);
  uint64_t* raw_empty = raw_full + kRaw1;
  uint64_t* split_full = raw_empty + kRaw1;    // this CTA's 4 converter warps of the stage's group
  uint64_t* split_empty = split_full + kSplit1;
  uint64_t* tfull = split_empty + kSplit1;
  uint32_t* tslot = reinterpret_cast<uint32_t*>(tfull + 1);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

  if (warp == 0 && lane == 0) {
    for (int q = 0; q < kRaw1; ++q) {
      mbar_init(&raw_full[q], 1);
      mbar_init(&raw_empty[q], 4);
    }
    for (int q = 0; q < kSplit1; ++q) {
      mbar_init(&split_full[q], 4);
      mbar_init(&split_empty[q], 1);
    }
    mbar_init(tfull, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tA) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tB) : "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(saddr(tslot)), "n"(kTmem1));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = *tslot;
  asm volatile("griddepcontrol.wait;" ::: "memory");

  if (warp == 0) {
    if (lane == 0) {   // ===== producer: raw A (16 k x 128 rows) and B (16 k-rows x 256 columns)
      const int32_t ya = m_blk * FBM, xb = nb * G1N;
      for (int i = 0; i < nkb; ++i) {
        const int q = i % kRaw1;
        if (i >= kRaw1) fwait(&raw_empty[q], (uint32_t)(((i / kRaw1) - 1) & 1));
        uint8_t* st = raw + q * RAW1_BYTES;
        const int32_t kx = (kb0 + i) * FBK;
        mbar_expect_tx(&raw_full[q], RAW1_BYTES);
        tma_load_2d(st, &tA, kx, ya, &raw_full[q]);
#pragma unroll
        for (int j = 0; j < G1N / 32; ++j) tma_load_2d(st + RAW1_A + j * 2048, &tB, xb + 32 * j, kx, &raw_full[q]);
      }
    }
    __syncwarp();
  } else if (warp == 1) {
    if (lane == 0) {   // ===== MMA issuer (every CTA is its own issuer)
      const uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(G1N >> 3) << 17) |
                             ((uint32_t)(FBM >> 4) << 24);
      for (int i = 0; i < nkb; ++i) {
        const int q = i % kSplit1;
        fwait(&split_full[q], (uint32_t)((i / kSplit1) & 1));
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        uint8_t* st = spl + q * SPLIT1_BYTES;
        const uint64_t bhi = sdesc(st), blo = sdesc(st + RAW1_B);
        const uint32_t ahi = tmem + (uint32_t)G1N + (uint32_t)(q * 32), alo = ahi + 16u;
#pragma unroll
        for (int kk = 0; kk < FBK / 8; ++kk) {
          const uint64_t adv = (uint64_t)(kk * 32) >> 4;
          mma_tf32_ts1(tmem, alo + 8u * kk, bhi + adv, idesc, (i | kk) != 0);
          mma_tf32_ts1(tmem, ahi + 8u * kk, blo + adv, idesc, 1u);
          mma_tf32_ts1(tmem, ahi + 8u * kk, bhi + adv, idesc, 1u);
        }
        mma_commit(&split_empty[q]);
      }
      mma_commit(tfull);
    }
    __syncwarp();
  } else {   // ===== converters (warps 2..9, two groups alternating k-steps), then the epilogue
    const int cg = (warp - 2) / 4;
    const int ct = (threadIdx.x - 64) & 127;
    for (int i = cg; i < nkb; i += kConvGroups) {
      const int q = i % kRaw1, p = i % kSplit1;
      fwait(&raw_full[q], (uint32_t)((i / kRaw1) & 1));
      if (i >= kSplit1) fwait(&split_empty[p], (uint32_t)(((i / kSplit1) - 1) & 1));
      const uint8_t* rs = raw + q * RAW1_BYTES;
      uint8_t* dst = spl + p * SPLIT1_BYTES;
      const int ar = (warp & 3) * 32 + lane;
      float4 v[4];
#pragma unroll
      for (int c = 0; c < 4; ++c)
        v[c] = *reinterpret_cast<const float4*>(rs + ar * 64 + ((c ^ ((ar >> 1) & 3)) << 4));
      constexpr int NB4 = G1N * 4 / 128;   // 8 B output float4 per converter thread
#pragma unroll 2
      for (int j0 = 0; j0 < NB4; j0 += 2) {
        float4 w[2];
#pragma unroll
        for (int j = 0; j < 2; ++j) {
          const int o = ct + 128 * (j0 + j), n = o % G1N, k0 = 4 * (o / G1N);
          const uint8_t* box = rs + RAW1_A + (n >> 5) * 2048 + (n & 3) * 4;
          const int c16 = (n & 31) >> 2;
          float t[4];
#pragma unroll
          for (int u = 0; u < 4; ++u) {
            const int k = k0 + u;
            t[u] = *reinterpret_cast<const float*>(box + k * 128 + ((c16 ^ (k & 7)) << 4));
          }
          w[j] = make_float4(t[0], t[1], t[2], t[3]);
        }
#pragma unroll
        for (int j = 0; j < 2; ++j) {
          float4 hi, lo;
          const int o = ct + 128 * (j0 + j), n = o % G1N, kc4 = o / G1N;
          const int boff = n * 64 + ((kc4 ^ ((n >> 1) & 3)) << 4);
          split2(w[j].x, hi.x, lo.x);
          split2(w[j].y, hi.y, lo.y);
          split2(w[j].z, hi.z, lo.z);
          split2(w[j].w, hi.w, lo.w);
          *reinterpret_cast<float4*>(dst + boff) = hi;
          *reinterpret_cast<float4*>(dst + RAW1_B + boff) = lo;
        }
      }
      {
        float ah[16], al[16];
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          split2(v[c].x, ah[4 * c], al[4 * c]);
          split2(v[c].y, ah[4 * c + 1], al[4 * c + 1]);
          split2(v[c].z, ah[4 * c + 2], al[4 * c + 2]);
          split2(v[c].w, ah[4 * c + 3], al[4 * c + 3]);
        }
        const uint32_t ta = tmem + ((uint32_t)((warp & 3) * 32) << 16) + (uint32_t)G1N + (uint32_t)(p * 32);
        tmem_st16(ta, ah);
        tmem_st16(ta + 16u, al);
      }
      asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
      asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      __syncwarp();
      if (lane == 0) {
        mbar_arrive(&raw_empty[q]);
        mbar_arrive(&split_full[p]);
      }
    }
    // ---- epilogue: accumulator -> this CTA's smem partial (or C when S = 1)
    const int grp = warp & 3;
    fwait(tfull, 0);
    asm volatile("bar.sync 1, %0;" ::"n"(128 * kConvGroups) : "memory");
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const int r = grp * 32 + lane;
    const int64_t grow = (int64_t)m_blk * FBM + r;
    float* red = reinterpret_cast<float*>(base);
    for (int c = cg * (G1N / kConvGroups); c < (cg + 1) * (G1N / kConvGroups); c += 16) {
      uint32_t v[16];
      const uint32_t ta = tmem + ((uint32_t)(grp * 32) << 16) + (uint32_t)c;
      asm volatile(
          "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
          : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
            "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15])
          : "r"(ta));
      asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
      if (S > 1) {
#pragma unroll
        for (int u = 0; u < 4; ++u)
          *reinterpret_cast<float4*>(red + r * RED1_LD + c + 4 * u) =
              make_float4(__uint_as_float(v[4 * u]), __uint_as_float(v[4 * u + 1]), __uint_as_float(v[4 * u + 2]),
                          __uint_as_float(v[4 * u + 3]));
      } else if (grow < mrows) {
        const int64_t n0 = (int64_t)nb * G1N + c;
        float* crow = C + (row0 + grow) * N;
#pragma unroll
        for (int u = 0; u < 4; ++u)
          if (n0 + 4 * u < N)
            *reinterpret_cast<float4*>(crow + n0 + 4 * u) =
                make_float4(__uint_as_float(v[4 * u]), __uint_as_float(v[4 * u + 1]),
                            __uint_as_float(v[4 * u + 2]), __uint_as_float(v[4 * u + 3]));
      }
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  }
  __syncthreads();
  if (S > 1) {
    cluster_sync_all();   // every partial of the cluster is in shared memory
    // CTA z reduces float4 columns [z G1N/4 / S, (z+1) G1N/4 / S) of the 128
    // rows over the S partials in split order ((p0 + p1) + p2) + p3
    const int c4a = (int)z * (G1N / 4) / S, c4n = ((int)z + 1) * (G1N / 4) / S - c4a;
    const float* red = reinterpret_cast<const float*>(base);
    uint32_t peer[4];
#pragma unroll
    for (int zz = 0; zz < 4; ++zz) peer[zz] = peer_addr(red, (uint32_t)(zz < S ? zz : 0));
    for (int e = threadIdx.x; e < FBM * c4n; e += kFThreads) {
      const int rr = e / c4n, cc = 4 * (c4a + e % c4n);
      const uint32_t off = (uint32_t)((rr * RED1_LD + cc) * 4);
      float4 pp[4];
#pragma unroll
      for (int zz = 0; zz < 4; ++zz)
        if (zz < S) pp[zz] = ld_dsmem_f4(peer[zz] + off);
      float4 a = pp[0];
#pragma unroll
      for (int zz = 1; zz < 4; ++zz)
        if (zz < S) {
          a.x += pp[zz].x; a.y += pp[zz].y; a.z += pp[zz].z; a.w += pp[zz].w;
        }
      const int64_t grow = (int64_t)m_blk * FBM + rr, n0 = (int64_t)nb * G1N + cc;
      if (grow < mrows && n0 < N) *reinterpret_cast<float4*>(C + (row0 + grow) * N + n0) = a;
    }
    cluster_arrive_relaxed_wait();
  }
  if (warp == 1) {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "n"(kTmem1));
  }
}

// ---------------------------------------------------------------------------
// Pre-split-B variant: as the single-SM variant, but B arrives already split
// and K-major (split_ab, one launch before, PDL) by TMA, so the converter
// warps only split A into TMEM (the B transposition was the converters' main
// load).  Single-SM variant (round 2): one CTA = 128 rows x 256 columns (M = 128,
// N = 256 tcgen05.mma.cta_group::1, twice the work per instruction of the
// pair's 256 x 128), S K splits in a cluster of S CTAs reduced through DSMEM.
// Same stage pipeline: raw TMA ring -> converter warps (A to TMEM, B
// transposed into the K-major SWIZZLE_64B smem layout) -> MMA thread.
constexpr int G2N = 256;                                       // output columns per CTA (MMA N)
constexpr int RAW2_A = FBM * FBK * 4, RAW2_B = G2N * FBK * 4;  // 8 KB + 16 KB (x2: hi, lo)
constexpr int RAW2_BYTES = RAW2_A + 2 * RAW2_B;
constexpr int kRaw2 = 5, kSplit2 = 8;                          // raw stages; A stages in TMEM
constexpr int kRing2 = kRaw2 * RAW2_BYTES;                     // 200 KB
constexpr int RED2_LD = G2N + 4;
constexpr int kTmem2 = 512;                                    // 256 accumulator + kSplit2 x 32 A columns
static_assert(G2N + kSplit2 * 32 <= kTmem2, "TMEM columns");
static_assert(FBM * RED2_LD * 4 <= kRing2, "partial buffer");
constexpr int kFused2Smem = kRing2 + 1024 + 256;

__global__ void __launch_bounds__(kFThreads, 1)
    sgemm_fused2(const __grid_constant__ CUtensorMap tA, const __grid_constant__ CUtensorMap tBh,
                 const __grid_constant__ CUtensorMap tBl, float* __restrict__ C,
                 int64_t N, int64_t row0, int64_t mrows, int nblk, int S, int nkb_all) {
  uint32_t z;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(z));
  const int cl = (int)(blockIdx.x / S);
  const int m_blk = cl / nblk, nb = cl % nblk;
  const int kb0 = (int)z * nkb_all / S, nkb = ((int)z + 1) * nkb_all / S - kb0;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* base = smem_raw + ((1024u - (saddr(smem_raw) & 1023u)) & 1023u);
  uint8_t* raw = base;
  uint64_t* raw_full = reinterpret_cast<uint64_t*>(base + kRing2);
  uint64_t* raw_empty = raw_full + kRaw2;
  uint64_t* split_full = raw_empty + kRaw2;    // this CTA's 4 converter warps of the stage's group
  uint64_t* split_empty = split_full + kSplit2;
  uint64_t* tfull = split_empty + kSplit2;
  uint32_t* tslot = reinterpret_cast<uint32_t*>(tfull + 1);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

  if (warp == 0 && lane == 0) {
    for (int q = 0; q < kRaw2; ++q) {
      mbar_init(&raw_full[q], 1);
      mbar_init(&raw_empty[q], 1);          // the MMA commit (B is read by the MMAs in place)
    }
    for (int q = 0; q < kSplit2; ++q) {
      mbar_init(&split_full[q], 4);
      mbar_init(&split_empty[q], 1);
    }
    mbar_init(tfull, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tA) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tBh) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tBl) : "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(saddr(tslot)), "n"(kTmem2));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = *tslot;
  asm volatile("griddepcontrol.wait;" ::: "memory");

  if (warp == 0) {
    if (lane == 0) {   // ===== producer: raw A (16 k x 128 rows) and B (16 k-rows x 256 columns)
      const int32_t ya = m_blk * FBM, xb = nb * G2N;
      for (int i = 0; i < nkb; ++i) {
        const int q = i % kRaw2;
        if (i >= kRaw2) fwait(&raw_empty[q], (uint32_t)(((i / kRaw2) - 1) & 1));
        uint8_t* st = raw + q * RAW2_BYTES;
        const int32_t kx = (kb0 + i) * FBK;
        mbar_expect_tx(&raw_full[q], RAW2_BYTES);
        tma_load_2d(st, &tA, kx, ya, &raw_full[q]);
        tma_load_2d(st + RAW2_A, &tBh, kx, xb, &raw_full[q]);            // B_hi^T rows n, 16 k (K-major)
        tma_load_2d(st + RAW2_A + RAW2_B, &tBl, kx, xb, &raw_full[q]);
      }
    }
    __syncwarp();
  } else if (warp == 1) {
    if (lane == 0) {   // ===== MMA issuer (every CTA is its own issuer)
      const uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(G2N >> 3) << 17) |
                             ((uint32_t)(FBM >> 4) << 24);
      for (int i = 0; i < nkb; ++i) {
        const int q = i % kRaw2, p = i % kSplit2;
        fwait(&raw_full[q], (uint32_t)((i / kRaw2) & 1));      // B of this k-step
        fwait(&split_full[p], (uint32_t)((i / kSplit2) & 1));  // A of this k-step in TMEM
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        uint8_t* st = raw + q * RAW2_BYTES;
        const uint64_t bhi = sdesc(st + RAW2_A), blo = sdesc(st + RAW2_A + RAW2_B);
        const uint32_t ahi = tmem + (uint32_t)G2N + (uint32_t)(p * 32), alo = ahi + 16u;
#pragma unroll
        for (int kk = 0; kk < FBK / 8; ++kk) {
          const uint64_t adv = (uint64_t)(kk * 32) >> 4;
          mma_tf32_ts1(tmem, alo + 8u * kk, bhi + adv, idesc, (i | kk) != 0);
          mma_tf32_ts1(tmem, ahi + 8u * kk, blo + adv, idesc, 1u);
          mma_tf32_ts1(tmem, ahi + 8u * kk, bhi + adv, idesc, 1u);
        }
        mma_commit(&raw_empty[q]);     // the converters finished reading this stage's A before split_full
        mma_commit(&split_empty[p]);
      }
      mma_commit(tfull);
    }
    __syncwarp();
  } else {   // ===== converters (warps 2..9, two groups alternating k-steps), then the epilogue
    const int cg = (warp - 2) / 4;
    const int ct = (threadIdx.x - 64) & 127;
    (void)ct;
    for (int i = cg; i < nkb; i += kConvGroups) {
      const int q = i % kRaw2, p = i % kSplit2;
      fwait(&raw_full[q], (uint32_t)((i / kRaw2) & 1));
      if (i >= kSplit2) fwait(&split_empty[p], (uint32_t)(((i / kSplit2) - 1) & 1));
      const uint8_t* rs = raw + q * RAW2_BYTES;
      const int ar = (warp & 3) * 32 + lane;
      float4 v[4];
#pragma unroll
      for (int c = 0; c < 4; ++c)
        v[c] = *reinterpret_cast<const float4*>(rs + ar * 64 + ((c ^ ((ar >> 1) & 3)) << 4));
      float ah[16], al[16];
#pragma unroll
      for (int c = 0; c < 4; ++c) {
        split2(v[c].x, ah[4 * c], al[4 * c]);
        split2(v[c].y, ah[4 * c + 1], al[4 * c + 1]);
        split2(v[c].z, ah[4 * c + 2], al[4 * c + 2]);
        split2(v[c].w, ah[4 * c + 3], al[4 * c + 3]);
      }
      const uint32_t ta = tmem + ((uint32_t)((warp & 3) * 32) << 16) + (uint32_t)G2N + (uint32_t)(p * 32);
      tmem_st16(ta, ah);
      tmem_st16(ta + 16u, al);
      asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
      asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
      __syncwarp();
      if (lane == 0) mbar_arrive(&split_full[p]);
    }
    // ---- epilogue: accumulator -> this CTA's smem partial (or C when S = 1)
    const int grp = warp & 3;
    fwait(tfull, 0);
    asm volatile("bar.sync 1, %0;" ::"n"(128 * kConvGroups) : "memory");
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const int r = grp * 32 + lane;
    const int64_t grow = (int64_t)m_blk * FBM + r;
    float* red = reinterpret_cast<float*>(base);
    for (int c = cg * (G2N / kConvGroups); c < (cg + 1) * (G2N / kConvGroups); c += 16) {
      uint32_t v[16];
      const uint32_t ta = tmem + ((uint32_t)(grp * 32) << 16) + (uint32_t)c;
      asm volatile(
          "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
          : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
            "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15])
          : "r"(ta));
      asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
      if (S > 1) {
#pragma unroll
        for (int u = 0; u < 4; ++u)
          *reinterpret_cast<float4*>(red + r * RED2_LD + c + 4 * u) =
              make_float4(__uint_as_float(v[4 * u]), __uint_as_float(v[4 * u + 1]), __uint_as_float(v[4 * u + 2]),
                          __uint_as_float(v[4 * u + 3]));
      } else if (grow < mrows) {
        const int64_t n0 = (int64_t)nb * G2N + c;
        float* crow = C + (row0 + grow) * N;
#pragma unroll
        for (int u = 0; u < 4; ++u)
          if (n0 + 4 * u < N)
            *reinterpret_cast<float4*>(crow + n0 + 4 * u) =
                make_float4(__uint_as_float(v[4 * u]), __uint_as_float(v[4 * u + 1]),
                            __uint_as_float(v[4 * u + 2]), __uint_as_float(v[4 * u + 3]));
      }
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  }
  __syncthreads();
  if (S > 1) {
    cluster_sync_all();   // every partial of the cluster is in shared memory
    // CTA z reduces float4 columns [z G2N/4 / S, (z+1) G2N/4 / S) of the 128
    // rows over the S partials in split order ((p0 + p1) + p2) + p3
    const int c4a = (int)z * (G2N / 4) / S, c4n = ((int)z + 1) * (G2N / 4) / S - c4a;
    const float* red = reinterpret_cast<const float*>(base);
    uint32_t peer[4];
#pragma unroll
    for (int zz = 0; zz < 4; ++zz) peer[zz] = peer_addr(red, (uint32_t)(zz < S ? zz : 0));
    for (int e = threadIdx.x; e < FBM * c4n; e += kFThreads) {
      const int rr = e / c4n, cc = 4 * (c4a + e % c4n);
      const uint32_t off = (uint32_t)((rr * RED2_LD + cc) * 4);
      float4 pp[4];
#pragma unroll
      for (int zz = 0; zz < 4; ++zz)
        if (zz < S) pp[zz] = ld_dsmem_f4(peer[zz] + off);
      float4 a = pp[0];
#pragma unroll
      for (int zz = 1; zz < 4; ++zz)
        if (zz < S) {
          a.x += pp[zz].x; a.y += pp[zz].y; a.z += pp[zz].z; a.w += pp[zz].w;
        }
      const int64_t grow = (int64_t)m_blk * FBM + rr, n0 = (int64_t)nb * G2N + cc;
      if (grow < mrows && n0 < N) *reinterpret_cast<float4*>(C + (row0 + grow) * N + n0) = a;
    }
    cluster_arrive_relaxed_wait();
  }
  if (warp == 1) {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "n"(kTmem2));
  }
}

}  // namespace

int max_active_clusters(int csize);

// K splits of the fused path for a row range: the largest S <= 4 with at
// least 8 k-blocks per split whose clusters of 2 S CTAs all fit on the GPU at
// once (one wave: cudaOccupancyMaxActiveClusters), 0 = use the two-pass path
// (the tile pairs alone fill the GPU, or the operands are not 16-B aligned).
static int fused_variant() {   // 1: 2-SM pairs (256 x 128), 2: single-SM 128 x 256 tiles, 3: 2 + pre-split B
  static const int env = getenv("MM_SGEMM_FUSED") ? atoi(getenv("MM_SGEMM_FUSED")) : 3;
  return env;
}
bool sgemm_fused_presplit_b() { return fused_variant() == 3; }
int max_active_clusters1(int csize);

int sgemm_fused_splits(const float* A, const float* B, float* C, int64_t mrows, int64_t N, int64_t K, int64_t r0) {
  const int env = fused_variant();
  if (!env || (K & 3) || (N & 3)) return 0;
  if (env >= 2) {
    if ((reinterpret_cast<uintptr_t>(A + r0 * K) | reinterpret_cast<uintptr_t>(B) | reinterpret_cast<uintptr_t>(C)) &
        15)
      return 0;
    const int64_t tiles = (mrows + FBM - 1) / FBM * ((N + G1N - 1) / G1N);
    const int64_t nkb = (K + FBK - 1) / FBK;
    if (tiles > 148 / 2) return 0;
    for (int S = 4; S >= 2; --S)
      if (nkb / S >= 8 && max_active_clusters1(S) >= tiles) return S;
    return 0;
  }
  if ((reinterpret_cast<uintptr_t>(A + r0 * K) | reinterpret_cast<uintptr_t>(B) | reinterpret_cast<uintptr_t>(C)) & 15)
    return 0;
  const int64_t pairs = ((mrows + FBM - 1) / FBM + 1) / 2 * ((N + FBN - 1) / FBN);
  const int64_t nkb = (K + FBK - 1) / FBK;
  if (pairs * 2 > 148 / 2) return 0;   // at least half the GPU in tile pairs already: no K split
  for (int S = 4; S >= 2; --S)
    if (nkb / S >= 8 && max_active_clusters(2 * S) >= pairs) return S;
  return 0;
}

int max_active_clusters(int csize) {
  static int cache[9] = {-1, -1, -1, -1, -1, -1, -1, -1, -1};
  if (csize < 1 || csize > 8) return 0;
  if (cache[csize] >= 0) return cache[csize];
  if (cudaFuncSetAttribute(sgemm_fused, cudaFuncAttributeMaxDynamicSharedMemorySize, kFusedSmem) != cudaSuccess ||
      cudaFuncSetAttribute(sgemm_fused, cudaFuncAttributeNonPortableClusterSizeAllowed, 1) != cudaSuccess)
    return 0;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)(csize * 16));
  cfg.blockDim = dim3(kFThreads);
  cfg.dynamicSmemBytes = kFusedSmem;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = (unsigned)csize;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  int n = 0;
  if (cudaOccupancyMaxActiveClusters(&n, (void*)sgemm_fused, &cfg) != cudaSuccess) n = 0;
  cache[csize] = n;
  return n;
}

int max_active_clusters1(int csize) {
  static int cache[9] = {-1, -1, -1, -1, -1, -1, -1, -1, -1};
  if (csize < 1 || csize > 8) return 0;
  if (cache[csize] >= 0) return cache[csize];
  if (cudaFuncSetAttribute(sgemm_fused1, cudaFuncAttributeMaxDynamicSharedMemorySize, kFused1Smem) != cudaSuccess)
    return 0;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)(csize * 16));
  cfg.blockDim = dim3(kFThreads);
  cfg.dynamicSmemBytes = kFused1Smem;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = (unsigned)csize;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  int n = 0;
  if (cudaOccupancyMaxActiveClusters(&n, (void*)sgemm_fused1, &cfg) != cudaSuccess) n = 0;
  cache[csize] = n;
  return n;
}

static cudaError_t sgemm_fused1_rows(const float* A, const float* B, float* C, int64_t N, int64_t K, int64_t r0,
                                     int64_t mrows, int S, cudaStream_t s) {
  CUtensorMap tA, tB;
  cudaError_t e;
  if ((e = encode_tmap_2d_f32(&tA, A + r0 * K, K, mrows, K * 4, FBK, FBM)) != cudaSuccess) return e;
  if ((e = encode_tmap_2d_f32(&tB, B, N, K, N * 4, 32, FBK)) != cudaSuccess) return e;
  static std::atomic<uint64_t> attr{0};
  e = once_per_device(attr, [] {
    return cudaFuncSetAttribute(sgemm_fused1, cudaFuncAttributeMaxDynamicSharedMemorySize, kFused1Smem);
  });
  if (e != cudaSuccess) return e;
  const int mblk = (int)((mrows + FBM - 1) / FBM);
  const int nblk = (int)((N + G1N - 1) / G1N);
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)(mblk * nblk * S));
  cfg.blockDim = dim3(kFThreads);
  cfg.dynamicSmemBytes = kFused1Smem;
  cfg.stream = s;
  cudaLaunchAttribute at[2];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = (unsigned)S;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  at[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = 2;
  note_launch();
  return cudaLaunchKernelEx(&cfg, sgemm_fused1, tA, tB, C, N, r0, mrows, nblk, S, (int)((K + FBK - 1) / FBK));
}

// B already split and K-major (bhi / blo: N x Kp, written by the previous
// launch on the stream); PDL lets the set-up overlap that launch.
cudaError_t sgemm_fused_presplit_rows(const float* A, const float* bhi, const float* blo, int64_t Kp, float* C,
                                      int64_t N, int64_t K, int64_t r0, int64_t mrows, int S, cudaStream_t s) {
  CUtensorMap tA, tBh, tBl;
  cudaError_t e;
  if ((e = encode_tmap_2d_f32(&tA, A + r0 * K, K, mrows, K * 4, FBK, FBM)) != cudaSuccess) return e;
  if ((e = encode_tmap_2d_f32(&tBh, bhi, Kp, N, Kp * 4, FBK, G2N)) != cudaSuccess) return e;
  if ((e = encode_tmap_2d_f32(&tBl, blo, Kp, N, Kp * 4, FBK, G2N)) != cudaSuccess) return e;
  static std::atomic<uint64_t> attr{0};
  e = once_per_device(attr, [] {
    return cudaFuncSetAttribute(sgemm_fused2, cudaFuncAttributeMaxDynamicSharedMemorySize, kFused2Smem);
  });
  if (e != cudaSuccess) return e;
  const int mblk = (int)((mrows + FBM - 1) / FBM);
  const int nblk = (int)((N + G2N - 1) / G2N);
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)(mblk * nblk * S));
  cfg.blockDim = dim3(kFThreads);
  cfg.dynamicSmemBytes = kFused2Smem;
  cfg.stream = s;
  cudaLaunchAttribute at[2];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = (unsigned)S;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  at[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = 2;
  note_launch();
  return cudaLaunchKernelEx(&cfg, sgemm_fused2, tA, tBh, tBl, C, N, r0, mrows, nblk, S, (int)((K + FBK - 1) / FBK));
}

cudaError_t sgemm_fused_rows(const float* A, const float* B, float* C, int64_t N, int64_t K, int64_t r0,
                             int64_t mrows, int S, cudaStream_t s) {
  if (fused_variant() >= 2) return sgemm_fused1_rows(A, B, C, N, K, r0, mrows, S, s);
  CUtensorMap tA, tB;
  cudaError_t e;
  if ((e = encode_tmap_2d_f32(&tA, A + r0 * K, K, mrows, K * 4, FBK, FBM)) != cudaSuccess) return e;
  if ((e = encode_tmap_2d_f32(&tB, B, N, K, N * 4, 32, FBK)) != cudaSuccess) return e;
  static std::atomic<uint64_t> attr{0};
  e = once_per_device(attr, [] {
    cudaError_t r = cudaFuncSetAttribute(sgemm_fused, cudaFuncAttributeMaxDynamicSharedMemorySize, kFusedSmem);
    if (r != cudaSuccess) return r;
    return cudaFuncSetAttribute(sgemm_fused, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
  });
  if (e != cudaSuccess) return e;
  const int mblk = (int)((mrows + FBM - 1) / FBM);
  const int mpairs = (mblk + 1) / 2;
  const int nblk = (int)((N + FBN - 1) / FBN);
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)(mpairs * nblk * 2 * S));
  cfg.blockDim = dim3(kFThreads);
  cfg.dynamicSmemBytes = kFusedSmem;
  cfg.stream = s;
  cudaLaunchAttribute at[2];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = (unsigned)(2 * S);
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  // programmatic dependent launch: barrier/TMEM set-up overlaps the previous
  // kernel's tail; the first global access follows griddepcontrol.wait
  at[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = 2;
  note_launch();
  return cudaLaunchKernelEx(&cfg, sgemm_fused, tA, tB, C, N, r0, mrows, nblk, S, (int)((K + FBK - 1) / FBK));
}

}  // namespace mm
