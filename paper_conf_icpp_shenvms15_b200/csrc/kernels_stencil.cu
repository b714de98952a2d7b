// HotSpot thermal stencil (P229-233 Table II "Rodinia [2]", P319: 8192x8192,
// row-wise split) and the MK-Loop residual kernel (BASELINE configs[3]).
//
// hotspot_rows: HBM-bound, 12 algorithmic bytes per cell (read T, read P,
// write T').  Tiles of kH rows x 1024 columns; every thread batches all its
// loads before computing (see hotspot_vec).  The update uses
// round-to-nearest intrinsics in the oracle's operation order (R16), so the
// result is bit-identical to oracle/numeric.c.
//
// row_residual: rowsum[y] = sum_x ((double)t1 - (double)t0)^2 — one CTA per
// row, FP64 accumulation, fixed shuffle tree (deterministic and independent of
// the partitioning).
#include "kernels.h"

namespace mm {

namespace {

constexpr int kThreads = 256;          // 1024 columns per CTA

__device__ __forceinline__ float cell(float c, float n, float s, float w, float e, float p,
                                      const HotCoef& k) {
  const float two = __fadd_rn(c, c);
  const float dv = __fmul_rn(__fsub_rn(__fadd_rn(s, n), two), k.ry1);
  const float dh = __fmul_rn(__fsub_rn(__fadd_rn(e, w), two), k.rx1);
  const float dz = __fmul_rn(__fsub_rn(k.amb, c), k.rz1);
  const float sum = __fadd_rn(__fadd_rn(__fadd_rn(p, dv), dh), dz);
  return __fadd_rn(c, __fmul_rn(k.sdc, sum));
}

// cols % 4 == 0, 16-B aligned rows.  A CTA owns a tile of kH rows x 1024
// columns of [r0, r1); each thread owns one float4 column group and issues
// ALL its loads first — kH+2 rows of T (rows above/below included) and kH rows
// of P, plus the warp-edge scalars — so each thread has 2kH+2 independent
// 16-B loads in flight, then computes the kH rows from registers (vertical
// reuse) and warp shuffles (horizontal reuse).  Measured on B200
// (tools/hotspot_variants.cu): 6.89 TB/s at 8192^2 and 7.13 TB/s at 16384^2,
// vs 6.13 TB/s for a row-walking strip with one row of prefetch and 4.79 TB/s
// for a single-wave TMA (cp.async.bulk + mbarrier) ring — the halo rows of
// neighbouring tiles are L2 hits, so deep MLP beats smem staging here.
constexpr int kH = 4;

__global__ void __launch_bounds__(kThreads) hotspot_vec(const float* __restrict__ tin,
                                                        const float* __restrict__ pw,
                                                        float* __restrict__ tout, int64_t rows,
                                                        int64_t cols, int64_t r0, int64_t r1,
                                                        HotCoef k, int64_t ncb) {
  const int lane = threadIdx.x & 31;
  const int64_t cb = blockIdx.x % ncb, st = blockIdx.x / ncb;
  const int64_t x0 = (cb * kThreads + threadIdx.x) * 4;
  const int64_t ys = r0 + st * kH;
  const bool active = x0 < cols;
  const int64_t xs = active ? x0 : 0;  // inactive lanes still join the shuffles
  const bool wl = lane == 0 && active && x0 > 0;
  const bool el = lane == 31 && active && x0 + 4 < cols;
  float4 T[kH + 2], P[kH];
  float W[kH], E[kH];
#pragma unroll
  for (int j = 0; j < kH + 2; ++j) {
    int64_t y = ys - 1 + j;
    y = y < 0 ? 0 : (y >= rows ? rows - 1 : y);
    T[j] = *reinterpret_cast<const float4*>(tin + y * cols + xs);
  }
#pragma unroll
  for (int j = 0; j < kH; ++j) {
    int64_t y = ys + j;
    y = y >= rows ? rows - 1 : y;
    P[j] = __ldcs(reinterpret_cast<const float4*>(pw + y * cols + xs));
    W[j] = wl ? tin[y * cols + x0 - 1] : 0.f;
    E[j] = el ? tin[y * cols + x0 + 4] : 0.f;
  }
#pragma unroll
  for (int j = 0; j < kH; ++j) {
    const int64_t y = ys + j;
    if (y >= r1) break;
    const float4 up = T[j], cu = T[j + 1], dn = T[j + 2], p = P[j];
    float w = __shfl_up_sync(0xffffffffu, cu.w, 1);
    float e = __shfl_down_sync(0xffffffffu, cu.x, 1);
    if (lane == 0) w = wl ? W[j] : cu.x;
    if (lane == 31) e = el ? E[j] : cu.w;
    if (x0 == 0) w = cu.x;               // chip edge: neighbour = the cell itself
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

// Temporal blocking (Rodinia's "pyramid"): one launch
// advances rows [r0, r1) by H iterations, reading T rows [r0-H, r1+H) (the
// halo the ownership directory pulls, access halo = H rows) and P once.
// Algorithmic HBM bytes per launch: 12 B per cell for H cell-updates.
//
// Each WARP owns an independent tile: 128 columns (one float4 group per lane;
// the HC = 4*ceil(H/4) columns at each end are halo, recomputed by the
// neighbouring warp) by a strip of SR output rows, and streams down the strip
// with an H-level software pipeline: at step r, level s = 1..H computes row
// r-s from the three newest rows of level s-1.  Level-0 (input) rows of T and
// the P rows arrive through a per-warp shared-memory ring filled by cp.async
// kTbAhead rows ahead; levels 1..H-1 keep their 3-row windows in registers
// (slot = row index mod 3, compile-time because the row loop is unrolled by
// 3).  Horizontal neighbours come from warp shuffles.  The 4 cells of a lane
// are updated as two f32x2 pairs (FADD2/FFMA2: same round-to-nearest results
// as the oracle's R16 ops, half the issue slots; DESIGN R35).  Rows outside the grid are
// never stored and halo columns lose one valid column per level and are not
// stored, so every stored cell went through exactly H applications of the
// R16 update: bit-identical to H single-step launches.
//
// One CTA of 12 warps per SM (3 per SM sub-partition: the register-bound
// residency at ~150 registers); every warp of a CTA runs the same number of
// steps.  Measured at 8192^2 x 1000 (h = 8): 41.8 ms vs 45.8 ms with three
// 4-warp CTAs per SM, whose SMs averaged 9.3 of 12 active warps (ncu) — the
// warps of one sub-partition drifted apart and the last ones ran alone,
// latency-bound on their level chains.  CTAs of 4 or 6 warps: 45.6 / 46.2 ms;
// CTA barriers every 6-48 steps: slower.
constexpr int kTbWarps = 12;                     // warps per CTA
constexpr int kTbHeadGroups = 5;                 // 3-step groups at a strip's head with fewer levels (>= (2H - 1) / 3 for H <= 8)
constexpr int kTbAhead = 3;                      // cp.async prefetch distance (rows, beyond a 3-step group)

// Level-0 rings in shared memory, [row slot][group j][lane] so the lanes'
// 16-B reads are contiguous.  T rows r-2 .. r+ahead+2 (level 1 only) in RT
// slots, P rows r-H .. r+ahead+2 (every level) in RP slots.  Each ring
// sits M slots above the start of its array, and a row whose slot is among
// the ring's last M is also written R slots lower (M = 2 for T, H for P), so
// the rows a step reads are contiguous at fixed offsets below one per-step
// base (array slot(r) + M): no per-level index arithmetic.
template <int H, int CL>
struct TbCfg {
  static constexpr int LW = 4 * CL;              // columns per lane (CL float4 groups)
  static constexpr int HC = LW * ((H + LW - 1) / LW);  // halo columns per side (whole lanes)
  static constexpr int OW = 32 * LW - 2 * HC;    // output columns per warp
  static constexpr int RT = 8, MT = 2;
  static constexpr int RP = 16, MP = H;
  static_assert(kTbAhead + 5 <= RT && H + kTbAhead + 3 <= RP, "ring capacity");
  static constexpr int ROWS = RT + MT + RP + MP; // float4 rows of 32 x CL per warp
};

struct f2 {
  unsigned long long v;
};
__device__ __forceinline__ f2 pk(float a, float b) {
  f2 r;
  asm("mov.b64 %0, {%1, %2};" : "=l"(r.v) : "f"(a), "f"(b));
  return r;
}
__device__ __forceinline__ void upk(f2 x, float& a, float& b) { asm("mov.b64 {%0, %1}, %2;" : "=f"(a), "=f"(b) : "l"(x.v)); }
__device__ __forceinline__ f2 add2(f2 a, f2 b) {
  f2 r;
  asm("add.rn.f32x2 %0, %1, %2;" : "=l"(r.v) : "l"(a.v), "l"(b.v));
  return r;
}
__device__ __forceinline__ f2 sub2(f2 a, f2 b) {
  f2 r;
  asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(r.v) : "l"(a.v), "l"(b.v));
  return r;
}

// products: ptxas contracts mul.rn.f32x2 followed by add.rn.f32x2 into FFMA2
// (single rounding), which would break R16's order, and folds a literal -0
// addend the same way.  fma.rn.f32x2(a, b, z) with z = -0 held in a register
// that comes from a kernel argument (opaque to ptxas) is RN(a*b + -0) =
// RN(a*b) for every a, b (an exact zero product keeps its sign, -0 + -0 = -0,
// +0 + -0 = +0): the R16 product bit for bit, one FFMA2 issue for two cells.
__device__ __forceinline__ f2 mul2s(f2 a, f2 b, f2 nz) {
  f2 r;
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(r.v) : "l"(a.v), "l"(b.v), "l"(nz.v));
  return r;
}

struct HotCoef2 {
  f2 ry1, rx1, rz1, sdc;
  f2 amb, nz, m2;
};

// cell() on two cells at once (R16 order, every op rounded to nearest), with
// the horizontal sums e + w already formed
// The doubling two = c + c is exact (unless it overflows, |c| >= 2^127), so
// RN(x - two) = RN(x - 2c) = fma(c, -2, x): the R16 difference bit for bit
// with one FP op per cell fewer (13 issued instead of R16's 14; R35).
__device__ __forceinline__ f2 sub_twice(f2 x, f2 c, f2 m2) {
  f2 r;
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(r.v) : "l"(c.v), "l"(m2.v), "l"(x.v));
  return r;
}

__device__ __forceinline__ f2 cell2h(f2 c, f2 n, f2 s, f2 ew, f2 p, const HotCoef2& k) {
  const f2 dv = mul2s(sub_twice(add2(s, n), c, k.m2), k.ry1, k.nz);
  const f2 dh = mul2s(sub_twice(ew, c, k.m2), k.rx1, k.nz);
  const f2 dz = mul2s(sub2(k.amb, c), k.rz1, k.nz);
  const f2 sum = add2(add2(add2(p, dv), dh), dz);
  return add2(c, mul2s(sum, k.sdc, k.nz));
}

// Four cells of a lane as the pairs (x, y), (z, w).  The east + west sums
// straddle the pairs ((w_prev, x) + (y, z), ...), so they are four scalar
// FADDs written straight into aligned pairs: packing the straddling operands
// for FADD2 cost ~8 MOVs per lane and level (ncu: 12.8 % of the issued
// instructions of hotspot_tb<8>).
__device__ __forceinline__ float4 cell4(float4 cu, float4 up, float4 dn, float w, float e, float4 p, const HotCoef2& k) {
  const f2 ewa = pk(__fadd_rn(cu.y, w), __fadd_rn(cu.z, cu.x));
  const f2 ewb = pk(__fadd_rn(cu.w, cu.y), __fadd_rn(e, cu.z));
  const f2 a = cell2h(pk(cu.x, cu.y), pk(up.x, up.y), pk(dn.x, dn.y), ewa, pk(p.x, p.y), k);
  const f2 b = cell2h(pk(cu.z, cu.w), pk(up.z, up.w), pk(dn.z, dn.w), ewb, pk(p.z, p.w), k);
  float4 o;
  upk(a, o.x, o.y);
  upk(b, o.z, o.w);
  return o;
}

__device__ __forceinline__ void cp_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }

// Per-lane state of a warp's strip.  The global row pointers advance by one
// row per fetch and the store pointer by one row per step, so neither the
// fetches nor the stores recompute 64-bit addresses.
struct TbArgs {
  const char* gT;                   // T and P bytes of the next row to fetch (lane's columns)
  const char* gP;
  float* so;                        // output row r - H of the current step (lane's columns)
  int64_t rowB;                     // row stride in bytes
  uint32_t trs, prs;                // shared addresses of the T / P arrays (+ lane)
  int rows, cols;                   // 32-bit: rows, cols < 2^31 (checked at launch)
  int qlo, qn;                      // rows q in [qlo, qlo + qn) are fetched (empty if the lane is off the grid)
  int sr0, sn;                      // step r stores row r - H iff r - sr0 in [0, sn)
  int eh;                           // step r has no grid-edge row iff r - H - 1 in [0, eh)
  bool wedge, eedge;                // chip-edge lanes
};

__device__ __forceinline__ void cp16s(uint32_t dst, const char* src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst), "l"(src) : "memory");
}

// issue the copies of level-0 row q (T and P) into the rings (and their
// mirrors), one commit group; rows are fetched in order, one per call
template <int H, int CL>
__device__ __forceinline__ void tb_fetch(TbArgs& a, int q) {
  using C = TbCfg<H, CL>;
  constexpr uint32_t SLOT = CL * 32 * 16;         // bytes per ring slot
  if ((unsigned)(q - a.qlo) < (unsigned)a.qn) {
    const int st = q & (C::RT - 1), sp = q & (C::RP - 1);
    const uint32_t dt = a.trs + (uint32_t)(st + C::MT) * SLOT, dp = a.prs + (uint32_t)(sp + C::MP) * SLOT;
#pragma unroll
    for (int j = 0; j < CL; ++j) {
      cp16s(dt + j * 512, a.gT + 16 * j);
      cp16s(dp + j * 512, a.gP + 16 * j);
      if (st >= C::RT - C::MT) cp16s(dt - C::RT * SLOT + j * 512, a.gT + 16 * j);
      if (sp >= C::RP - C::MP) cp16s(dp - C::RP * SLOT + j * 512, a.gP + 16 * j);
    }
  }
  cp_commit();
  a.gT += a.rowB;
  a.gP += a.rowB;
}

// One step r: level s = 1..H computes row r - s.  EDGE = some row of the
// step is the grid's first or last row; CE = the warp holds the chip's first
// or last column (both warp-uniform, so interior steps of interior warps run
// without boundary selects).  tb = T row r, pb = P row r (ring bases).
// HEAD: only levels 1..smax (the strip's first steps, see tb_run).
template <int H, int CL, int PH, bool EDGE, bool CE, bool HEAD = false>
__device__ __forceinline__ void tb_levels(float4 (&W)[H > 1 ? H - 1 : 1][3][CL], const float4* tb, const float4* pb,
                                          const TbArgs& a, int r, const HotCoef2& k, int smax = H) {
#pragma unroll
  for (int s = 1; s <= H; ++s) {
    if (HEAD && s > smax) break;
    const int y = r - s;
    float4 cu[CL], up[CL], dn[CL], p[CL];
#pragma unroll
    for (int j = 0; j < CL; ++j) {
      if (s == 1) {                               // level 0 rows from the ring
        cu[j] = tb[(j - CL) * 32];
        up[j] = tb[(j - 2 * CL) * 32];
        dn[j] = tb[j * 32];
      } else {
        cu[j] = W[s - 2][((PH - s) % 3 + 3) % 3][j];
        up[j] = W[s - 2][((PH - s - 1) % 3 + 3) % 3][j];
        dn[j] = W[s - 2][((PH - s + 1) % 3 + 3) % 3][j];
      }
      if (EDGE) {
        if (y <= 0) up[j] = cu[j];                // chip edge: neighbour = the cell itself
        if (y + 1 >= a.rows) dn[j] = cu[j];
      }
      p[j] = pb[(j - s * CL) * 32];
    }
    float w = __shfl_up_sync(0xffffffffu, cu[CL - 1].w, 1);
    float e = __shfl_down_sync(0xffffffffu, cu[0].x, 1);
    if (CE) {
      if (a.wedge) w = cu[0].x;
      if (a.eedge) e = cu[CL - 1].w;
    }
#pragma unroll
    for (int j = 0; j < CL; ++j) {
      const float wj = j > 0 ? cu[j - 1].w : w;
      const float ej = j + 1 < CL ? cu[j + 1].x : e;
      const float4 o = cell4(cu[j], up[j], dn[j], wj, ej, p[j], k);
      if (s < H) {
        W[s - 1][((PH - s) % 3 + 3) % 3][j] = o;
      } else if ((unsigned)(r - a.sr0) < (unsigned)a.sn) {
        __stcs(reinterpret_cast<float4*>(a.so) + j, o);
      }
    }
  }
}

// The first step of each unrolled 3-step group fetches rows r + kTbAhead ..
// r + kTbAhead + 2 and waits for rows <= r + 2, so the other two steps carry
// no cp.async instructions (asm volatile, memory clobber) that would keep
// ptxas from interleaving the steps' level chains (measured: 40.8 vs 41.6 ms
// with a fetch + wait in every step).
template <int H, int CL, int PH, bool CE, bool HEAD = false>
__device__ __forceinline__ void tb_step(float4 (&W)[H > 1 ? H - 1 : 1][3][CL], const float4* tr, const float4* pr,
                                        TbArgs& a, int r, const HotCoef2& k, int smax = H) {
  using C = TbCfg<H, CL>;
  if (PH == 0) {
    tb_fetch<H, CL>(a, r + kTbAhead);
    tb_fetch<H, CL>(a, r + kTbAhead + 1);
    tb_fetch<H, CL>(a, r + kTbAhead + 2);
    cp_wait<kTbAhead>();                          // rows <= r + 2 landed (each lane reads only its own copies)
  }
  const float4* tb = tr + ((r & (C::RT - 1)) + C::MT) * CL * 32;
  const float4* pb = pr + ((r & (C::RP - 1)) + C::MP) * CL * 32;
  if (HEAD)       // strip head: boundary selects always on (rare steps)
    tb_levels<H, CL, PH, true, CE, true>(W, tb, pb, a, r, k, smax);
  else if ((unsigned)(r - H - 1) < (unsigned)a.eh)
    tb_levels<H, CL, PH, false, CE>(W, tb, pb, a, r, k);
  else
    tb_levels<H, CL, PH, true, CE>(W, tb, pb, a, r, k);
  a.so += a.cols;
}

// steps r = rb, rb + 1, ... in whole 3-step groups (steps past the strip
// fetch and store nothing)
template <int H, int CL, bool CE>
__device__ __forceinline__ void tb_run(float4 (&W)[H > 1 ? H - 1 : 1][3][CL], const float4* tr, const float4* pr,
                                       TbArgs& a, int rb, int ngroups, const HotCoef2& k) {
  // The strip's first 2H - 2 steps (t = r - rb): level s computes row
  // rb + t - s, which only feeds stored cells from t = 2s - 1 on (row
  // >= Y0 - (H - s)), so step t runs levels 1 .. (t + 1) / 2; a skipped
  // level's window keeps stale values that only reach rows never stored.
  // Saves H^2 of the strip's (SR + 2H - 1) H level-rows (2.2 % at SR = 342).
  for (int g = 0, r = rb; g < kTbHeadGroups; ++g, r += 3) {
    tb_step<H, CL, 0, CE, true>(W, tr, pr, a, r, k, (3 * g + 1) / 2);
    tb_step<H, CL, 1, CE, true>(W, tr, pr, a, r + 1, k, (3 * g + 2) / 2);
    tb_step<H, CL, 2, CE, true>(W, tr, pr, a, r + 2, k, (3 * g + 3) / 2);
  }
  for (int g = kTbHeadGroups, r = rb + 3 * kTbHeadGroups; g < ngroups; ++g, r += 3) {
    tb_step<H, CL, 0, CE>(W, tr, pr, a, r, k);
    tb_step<H, CL, 1, CE>(W, tr, pr, a, r + 1, k);
    tb_step<H, CL, 2, CE>(W, tr, pr, a, r + 2, k);
  }
}

template <int H, int CL, int NW>
__global__ void __launch_bounds__(32 * NW, 1) hotspot_tb(const float* __restrict__ tin, const float* __restrict__ pw,
                                                        float* __restrict__ tout, int rows, int cols, int r0, int r1,
                                                        HotCoef kc, int nwx, int SR, float nz) {
  using C = TbCfg<H, CL>;
  extern __shared__ float4 tb_smem[];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int gw = blockIdx.x * NW + wid;
  const int wx = gw % nwx, wy = gw / nwx;
  // every warp of the CTA runs the same number of steps (a strip past r1
  // or shorter than SR fetches nothing and stores nothing there)
  int64_t y0l = (int64_t)r0 + (int64_t)wy * SR;
  if (y0l > r1) y0l = r1;
  const int Y0 = (int)y0l;
  const int Y1 = Y0 + SR < r1 ? Y0 + SR : r1;
  const int X0 = wx * C::OW;                      // first output column
  const int x0 = X0 - C::HC + C::LW * lane;       // this lane's LW columns
  const bool inx = x0 >= 0 && x0 < cols;          // cols % LW == 0: all or none of them
  const bool store_x = inx && x0 >= X0 && x0 < X0 + C::OW;
  // level-0 rows [rs, re) = [Y0 - H, Y1 + H); at step r level s computes row
  // r - s, so steps r in [rs + 1, re) end with level H row Y1 - 1
  const int rs = Y0 - H, re = Y1 + H;
  const int rb = rs + 1;
  TbArgs a;
  a.rows = rows;
  a.cols = cols;
  a.rowB = (int64_t)cols * 4;
  a.gT = reinterpret_cast<const char*>(tin + (int64_t)rs * cols + x0);
  a.gP = reinterpret_cast<const char*>(pw + (int64_t)rs * cols + x0);
  a.so = tout + (int64_t)(rb - H) * cols + x0;
  a.qlo = rs > 0 ? rs : 0;
  const int qhi = re < rows ? re : rows;
  a.qn = inx && qhi > a.qlo ? qhi - a.qlo : 0;
  a.sr0 = Y0 + H;
  a.sn = store_x ? Y1 - Y0 : 0;
  a.eh = rows - H - 2 > 0 ? rows - H - 2 : 0;
  a.wedge = x0 == 0;
  a.eedge = x0 + C::LW == cols;
  const float4* tr = tb_smem + (size_t)wid * C::ROWS * CL * 32 + lane;
  const float4* pr = tr + (C::RT + C::MT) * CL * 32;
  a.trs = (uint32_t)__cvta_generic_to_shared(tr);
  a.prs = (uint32_t)__cvta_generic_to_shared(pr);
  HotCoef2 k;
  k.ry1 = pk(kc.ry1, kc.ry1); k.rx1 = pk(kc.rx1, kc.rx1); k.rz1 = pk(kc.rz1, kc.rz1); k.sdc = pk(kc.sdc, kc.sdc);
  k.amb = pk(kc.amb, kc.amb);
  k.nz = pk(nz, nz);
  k.m2 = pk(-2.f, -2.f);
  float4 W[H > 1 ? H - 1 : 1][3][CL];
#pragma unroll
  for (int i = 0; i < (H > 1 ? H - 1 : 1); ++i)
#pragma unroll
    for (int j = 0; j < 3; ++j)
#pragma unroll
      for (int g = 0; g < CL; ++g) W[i][j][g] = make_float4(0.f, 0.f, 0.f, 0.f);
  // prologue: rows rs .. rs + kTbAhead in flight (the group at step r
  // fetches r + kTbAhead ..)
#pragma unroll
  for (int q = 0; q <= kTbAhead; ++q) tb_fetch<H, CL>(a, rs + q);
  const int ngroups = (SR + 2 * H - 1 + 2) / 3;
  if (__any_sync(0xffffffffu, a.wedge || a.eedge))
    tb_run<H, CL, true>(W, tr, pr, a, rb, ngroups, k);
  else
    tb_run<H, CL, false>(W, tr, pr, a, rb, ngroups, k);
  cp_wait<0>();
}

template <int H, int CL, int NW>
cudaError_t launch_tb_nw(const float* tin, const float* pw, float* tout, int64_t rows, int64_t cols, int64_t r0,
                         int64_t r1, HotCoef c, cudaStream_t s, int sms) {
  using C = TbCfg<H, CL>;
  if (rows + 16 >= (int64_t)INT32_MAX || cols >= (int64_t)INT32_MAX) return cudaErrorInvalidValue;
  const int64_t nwx = (cols + C::OW - 1) / C::OW;
  const size_t smem = (size_t)NW * C::ROWS * CL * 32 * sizeof(float4);
  static std::atomic<uint64_t> attr{0};
  static std::atomic<int> per_sm{0};   // resident CTAs per SM (registers bound it; same on every B200)
  cudaError_t e = once_per_device(attr, [&] {
    cudaError_t r = cudaFuncSetAttribute(hotspot_tb<H, CL, NW>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (r != cudaSuccess) return r;
    int n = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, hotspot_tb<H, CL, NW>, 32 * NW, smem) != cudaSuccess || n < 1)
      n = 1;
    per_sm.store(n);
    return cudaSuccess;
  });
  if (e != cudaSuccess) return e;
  // at most one wave of resident warps (a partial second wave left SMs
  // idle); strips at least 8H rows tall (vertical redundancy (2H+1)/SR)
  const int64_t target = (int64_t)(sms > 0 ? sms : 148) * per_sm.load() * NW;
  const int64_t nr = r1 - r0;
  int64_t nstrip = target / nwx > 1 ? target / nwx : 1;
  int64_t SR = (nr + nstrip - 1) / nstrip;
  if (SR < 8 * H) SR = 8 * H;
  nstrip = (nr + SR - 1) / SR;
  const int64_t warps = nwx * nstrip;
  if (warps + NW >= (int64_t)INT32_MAX) return cudaErrorInvalidValue;
  note_launch();
  hotspot_tb<H, CL, NW><<<(unsigned)((warps + NW - 1) / NW), 32 * NW, smem, s>>>(
      tin, pw, tout, (int)rows, (int)cols, (int)r0, (int)r1, c, (int)nwx, (int)SR, -0.0f);
  return cudaGetLastError();
}

// CL = 2 (256-column warp tiles, half the halo share, 246 registers, one
// 8-warp CTA per SM) measured 46.2 ms vs 41.8 ms for CL = 1 at 8192^2 x 1000:
// two warps per sub-partition do not hide the level chains' latency.
template <int H>
cudaError_t launch_tb(const float* tin, const float* pw, float* tout, int64_t rows, int64_t cols, int64_t r0,
                      int64_t r1, HotCoef c, cudaStream_t s, int sms) {
  return launch_tb_nw<H, 1, kTbWarps>(tin, pw, tout, rows, cols, r0, r1, c, s, sms);
}

// Generic shapes: one thread per cell.
__global__ void hotspot_scalar(const float* __restrict__ tin, const float* __restrict__ pw,
                               float* __restrict__ tout, int64_t rows, int64_t cols, int64_t r0,
                               int64_t r1, HotCoef k) {
  const int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int64_t n = (r1 - r0) * cols;
  if (idx >= n) return;
  const int64_t y = r0 + idx / cols, x = idx % cols;
  const float c = tin[y * cols + x];
  const float nn = y > 0 ? tin[(y - 1) * cols + x] : c;
  const float ss = y < rows - 1 ? tin[(y + 1) * cols + x] : c;
  const float w = x > 0 ? tin[y * cols + x - 1] : c;
  const float e = x < cols - 1 ? tin[y * cols + x + 1] : c;
  tout[y * cols + x] = cell(c, nn, ss, w, e, pw[y * cols + x], k);
}

__global__ void __launch_bounds__(kThreads) residual_rows(const float* __restrict__ t0,
                                                          const float* __restrict__ t1,
                                                          double* __restrict__ rowsum, int64_t cols,
                                                          int64_t r0) {
  const int64_t y = r0 + blockIdx.x;
  const float* a = t0 + y * cols;
  const float* b = t1 + y * cols;
  double acc = 0.0;
  if ((cols & 3) == 0) {
    const int64_t n4 = cols / 4;
    for (int64_t i = threadIdx.x; i < n4; i += kThreads) {
      const float4 u = __ldcs(reinterpret_cast<const float4*>(a) + i);
      const float4 v = __ldcs(reinterpret_cast<const float4*>(b) + i);
      double d;
      d = (double)v.x - (double)u.x; acc = fma(d, d, acc);
      d = (double)v.y - (double)u.y; acc = fma(d, d, acc);
      d = (double)v.z - (double)u.z; acc = fma(d, d, acc);
      d = (double)v.w - (double)u.w; acc = fma(d, d, acc);
    }
  } else {
    for (int64_t i = threadIdx.x; i < cols; i += kThreads) {
      const double d = (double)b[i] - (double)a[i];
      acc = fma(d, d, acc);
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
  __shared__ double part[kThreads / 32];
  if ((threadIdx.x & 31) == 0) part[threadIdx.x >> 5] = acc;
  __syncthreads();
  if (threadIdx.x == 0) {
    double s = 0.0;
#pragma unroll
    for (int i = 0; i < kThreads / 32; ++i) s += part[i];
    rowsum[y] = s;
  }
}

}  // namespace

cudaError_t hotspot_rows(const float* tin, const float* pw, float* tout, int64_t rows, int64_t cols,
                         int64_t r0, int64_t r1, HotCoef c, cudaStream_t s, int sms, int steps) {
  if (r1 <= r0) return cudaSuccess;
  if (steps > 1) {   // temporal blocking: needs float4 rows (cols % 4 == 0, 16-B aligned)
    if ((cols % 4) != 0 || (((uintptr_t)tin | (uintptr_t)pw | (uintptr_t)tout) & 15u) != 0)
      return cudaErrorInvalidValue;
    switch (steps) {
      case 2: return launch_tb<2>(tin, pw, tout, rows, cols, r0, r1, c, s, sms);
      case 3: return launch_tb<3>(tin, pw, tout, rows, cols, r0, r1, c, s, sms);
      case 4: return launch_tb<4>(tin, pw, tout, rows, cols, r0, r1, c, s, sms);
      case 6: return launch_tb<6>(tin, pw, tout, rows, cols, r0, r1, c, s, sms);
      case 8: return launch_tb<8>(tin, pw, tout, rows, cols, r0, r1, c, s, sms);
      default: return cudaErrorInvalidValue;
    }
  }
  const bool vec = (cols % 4 == 0) && (((uintptr_t)tin | (uintptr_t)pw | (uintptr_t)tout) & 15u) == 0;
  if (vec) {
    const int64_t ncb = (cols / 4 + kThreads - 1) / kThreads;
    const int64_t tiles = ncb * ((r1 - r0 + kH - 1) / kH);
    note_launch();
    hotspot_vec<<<(unsigned)tiles, kThreads, 0, s>>>(tin, pw, tout, rows, cols, r0, r1, c, ncb);
  } else {
    const int64_t n = (r1 - r0) * cols;
    note_launch();
    hotspot_scalar<<<(unsigned)((n + 255) / 256), 256, 0, s>>>(tin, pw, tout, rows, cols, r0, r1, c);
  }
  return cudaGetLastError();
}

cudaError_t row_residual(const float* t0, const float* t1, double* rowsum, int64_t cols, int64_t r0,
                         int64_t r1, cudaStream_t s, int) {
  if (r1 <= r0) return cudaSuccess;
  note_launch();
  residual_rows<<<(unsigned)(r1 - r0), kThreads, 0, s>>>(t0, t1, rowsum, cols, r0);
  return cudaGetLastError();
}

}  // namespace mm
