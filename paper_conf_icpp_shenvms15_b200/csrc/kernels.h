// Launch interface of the sm_100a kernels (one per paper application kernel).
#pragma once

#include <cuda_runtime.h>
#include <atomic>
#include <cstdint>
#include <utility>
#include <vector>

namespace mm {

// Kernel attributes (cudaFuncSetAttribute) are per CUDA device: run `set`
// once for each device this process launches on (a context may span several
// GPUs), thread-safe; `done` is a per-call-site bitmask of device ordinals.
template <class F>
cudaError_t once_per_device(std::atomic<uint64_t>& done, F&& set) {
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  const uint64_t bit = 1ull << (dev & 63);
  if (done.load(std::memory_order_acquire) & bit) return cudaSuccess;
  e = set();
  if (e == cudaSuccess) done.fetch_or(bit, std::memory_order_acq_rel);
  return e;
}

// Kernels launched by this process (mm_kernel_launch_count): every launch
// site calls note_launch; a run's mm_run_stats.n_launches is the delta over
// its issue (CUDA-graph replays add the kernels the graph holds).
extern std::atomic<int64_t> g_kernel_launches;
inline void note_launch(int64_t n = 1) { g_kernel_launches.fetch_add(n, std::memory_order_relaxed); }

// Launch with programmatic stream serialization (PDL): the kernel may start
// while the previous kernel on the stream finishes; it orders itself with
// griddepcontrol.wait.
template <typename... P, typename... A>
cudaError_t launch_pdl(void (*kern)(P...), dim3 grid, dim3 block, size_t smem, cudaStream_t s, A&&... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  note_launch();
  return cudaLaunchKernelEx(&cfg, kern, std::forward<A>(args)...);
}

struct Kernel;
struct Task;

// Library-owned device scratch of one logical device, with the cache of the
// whole-operand split of a 3xTF32 GEMM (B is split once per run and device;
// `epoch` is bumped by the runtime at every run and every profile launch).
struct Scratch {
  void* ptr = nullptr;
  size_t bytes = 0;
  const void* b_src = nullptr;
  int64_t b_K = 0, b_N = 0;
  uint64_t b_epoch = 0;
  uint64_t epoch = 1;
  std::vector<uint64_t> panel;   // Cholesky: split tag (epoch, step) per panel slot
  // Cholesky: the last POTRF launched on this scratch (step, stream, epoch):
  // it also wrote L_kk's split and packed leaves and counts finished blocks
  // per 128-row block, so a TRSM of that step on that stream may start early
  int64_t potrf_k = -1;
  const void* potrf_stream = nullptr;
  uint64_t potrf_epoch = 0;
};

// Packed 128 x 128 leaf blocks of L_kk for the column TRSM (per leaf q, floats):
//   U[s(s-1)/2 + mb][i][c] = L[c0+32s+c][c0+32mb+i]   s = 1..3, mb < s   at kLtU
//   D[s][c][c2]            = L[c0+32s+c2][c0+32s+c]   s = 0..3           at kLtD
//   rd[m]                  = RN(1 / L[c0+m][c0+m])                       at kLtRd
constexpr int kLtU = 0, kLtD = 6 * 1024, kLtRd = 10 * 1024, kLtFloats = kLtRd + 128;

struct Launch {
  const Kernel* k;          // kernel descriptor (op, params)
  const Task* t;            // task: item range [t->b, t->e) / DAG params
  void* const* opnd;        // device pointers, one per access (this device's copy)
  cudaStream_t stream;
  int32_t sms;              // SMs available to this logical device
  Scratch* scr;             // this logical device's scratch
  uint32_t ro_mask;         // bit i: operand i is never written by the app (cacheable)
};

// Device scratch a builtin kernel needs for this task (0 if none).
size_t builtin_scratch_bytes(const Kernel& k, const Task& t);

// Returns cudaSuccess, cudaErrorNotSupported for an unimplemented op, or the
// launch error.  Empty ranges launch nothing.
cudaError_t launch_builtin(const Launch& L);

// STREAM (kernels_stream.cu)
cudaError_t stream_copy(const float* a, float* c, int64_t lo, int64_t hi, cudaStream_t s, int sms);
cudaError_t stream_scale(const float* c, float* b, float q, int64_t lo, int64_t hi, cudaStream_t s, int sms);
cudaError_t stream_add(const float* a, const float* b, float* c, int64_t lo, int64_t hi, cudaStream_t s, int sms);
cudaError_t stream_triad(const float* b, const float* c, float* a, float q, int64_t lo, int64_t hi, cudaStream_t s, int sms);

// HotSpot + residual (kernels_stencil.cu)
struct HotCoef { float sdc, rx1, ry1, rz1, amb; };
cudaError_t hotspot_rows(const float* tin, const float* pw, float* tout, int64_t rows, int64_t cols,
                         int64_t r0, int64_t r1, HotCoef c, cudaStream_t s, int sms, int steps = 1);
cudaError_t row_residual(const float* t0, const float* t1, double* rowsum, int64_t cols,
                         int64_t r0, int64_t r1, cudaStream_t s, int sms);

// BlackScholes (kernels_bs.cu)
cudaError_t blackscholes(const float* S, const float* X, const float* T, float* call, float* put,
                         float R, float V, int64_t lo, int64_t hi, cudaStream_t s, int sms);

// SGEMM rows [r0,r1) of C = A B (kernels_gemm.cu)
cudaError_t sgemm_rows(const float* A, const float* B, float* C, int64_t M, int64_t N, int64_t K,
                       int64_t r0, int64_t r1, int32_t variant, cudaStream_t s, int sms, Scratch* scr,
                       bool b_readonly);
size_t sgemm_tf32x3_scratch(int64_t N, int64_t K, int64_t mrows);

// Cholesky tiles (kernels_chol.cu); A tile-major, T x T tiles of b x b.
constexpr int kCholBatch = 512;   // tasks per batched launch (a whole MK-DAG step at T = 32)
// Device scratch of every Cholesky op: 3xTF32 panel split + POTRF flags.
size_t chol_scratch_bytes(int64_t T, int64_t b);
// n independent tasks of one kernel (ijk = n triples) in one launch.
cudaError_t chol_batch(int32_t op, float* A, int64_t T, int64_t b, const int32_t* ijk, int32_t n,
                       cudaStream_t s, int sms, Scratch* scr);
// 3xTF32 tcgen05 trailing update (kernels_gemm_tc.cu); b % 256 == 0
size_t chol_tc_scratch(int64_t T, int64_t b);
cudaError_t chol_update_tc(float* A, int64_t T, int64_t b, const int32_t* ijk, int32_t n, cudaStream_t s,
                           Scratch* scr);

// TRSM on the split panel slots (kernels_gemm_tc.cu): L_kk split into its
// slot; slots marked split; block update columns [n0, b) -= X[:, kx0:kx0+K] L^T.
cudaError_t chol_trsm_prepare(float* A, int64_t T, int64_t b, int32_t k, cudaStream_t s, Scratch* scr,
                              float** hi, float** lo, int32_t* slot0);
void chol_mark_split(Scratch* scr, int64_t T, int32_t k, const int32_t* tiles, int32_t n);
// TRSM of a batch of step-k tiles in one launch (kernels_chol_trsm.cu; b % 128
// == 0, 256 <= b <= 4096, else cudaErrorNotSupported); MM_TRSM_COL=0 selects
// the leaf path.  Its transposed L_kk leaves live after the POTRF flags.
bool chol_trsm_col_enabled();
// MM_TRSM_OVERLAP=0: no POTRF -> column TRSM overlap (the TRSM then waits for
// the whole POTRF and splits L_kk itself)
bool chol_trsm_overlap_enabled();
// per-128-row-block finished-block counts of the last POTRF on this scratch
int* chol_potrf_rowcnt(Scratch* scr, int64_t T, int64_t b);
size_t chol_trsm_lt_bytes(int64_t b);
cudaError_t chol_trsm_col(float* A, int64_t T, int64_t b, int32_t k, const int32_t* ti, int32_t n, cudaStream_t s,
                          Scratch* scr);
cudaError_t chol_trsm_update_tc(float* A, int64_t T, int64_t b, int32_t k, const int32_t* ti, int32_t n,
                                int32_t kx0, int32_t K, int32_t n0, cudaStream_t s, Scratch* scr,
                                bool pdl = false);   // pdl: launched as a programmatic dependent of a leaf

// Nbody step for bodies [r0, r1) (kernels_nbody.cu); float4 bodies.
cudaError_t nbody_rows_launch(const float* pin, const float* vin, float* pout, float* vout, int64_t n, int64_t r0,
                              int64_t r1, float dt, float eps2, cudaStream_t s);

// Counter-hash generators (kernels_fill.cu) = synthgen.uniform / integers.
cudaError_t fill_uniform(float* dst, int64_t n, uint64_t seed, int32_t array_id, int64_t start,
                         float lo, float hi, cudaStream_t s);
cudaError_t fill_integers(float* dst, int64_t n, uint64_t seed, int32_t array_id, int64_t start,
                          int32_t lo, int32_t hi, cudaStream_t s);
cudaError_t fill_spd_tiles(float* dst, int64_t n, int64_t b, uint64_t seed, int32_t array_id, cudaStream_t s);

}  // namespace mm
