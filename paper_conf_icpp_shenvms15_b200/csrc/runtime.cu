// Runtime of the matchmaking library: logical devices (streams, optional
// green-context SM budgets), the op-program executor (in-process streams and
// events, or NCCL send/recv across processes), CUDA-graph replay, Glinda-style
// profiling (P49) with the DP-Perf warm-up (P311), and result collection.
#include <cuda.h>
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <nccl.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <deque>
#include <memory>
#include <new>
#include <map>
#include <random>
#include <vector>

#include "ipc.h"
#include "kernels.h"
#include "mm_internal.h"
#include "segmap.h"

using namespace mm;

namespace mm {
std::atomic<int64_t> g_kernel_launches{0};
}

struct DevRt {
  int32_t phys = 0, budget = 0, sms = 0, rank = 0;
  Scratch scr;               // device scratch for builtin kernels (e.g. 3xTF32 operand split)
  cudaStream_t stream = nullptr;      // compute stream (kernels, device<->device pulls)
  cudaStream_t h2d = nullptr;         // host->device copies (staged inputs)
  cudaStream_t d2h = nullptr;         // device->host copies (flushes)
  cudaStream_t lane1 = nullptr;       // second compute stream (lane-1 kernels)
  CUgreenCtx gctx = nullptr;
  CUcontext gcu = nullptr;   // CUcontext view of the green context
  bool mine = false;
};

// Driver-API entry points, resolved at run time through the runtime
// (cudaGetDriverEntryPoint) so the library has no link-time dependency on
// libcuda.so (it must load on hosts without a driver).
struct Drv {
  decltype(&cuInit) Init = nullptr;
  decltype(&cuDeviceGet) DeviceGet = nullptr;
  decltype(&cuDeviceGetDevResource) DeviceGetDevResource = nullptr;
  decltype(&cuDevSmResourceSplitByCount) DevSmResourceSplitByCount = nullptr;
  decltype(&cuDevResourceGenerateDesc) DevResourceGenerateDesc = nullptr;
  decltype(&cuGreenCtxCreate) GreenCtxCreate = nullptr;
  decltype(&cuGreenCtxStreamCreate) GreenCtxStreamCreate = nullptr;
  decltype(&cuGreenCtxDestroy) GreenCtxDestroy = nullptr;
  decltype(&cuCtxFromGreenCtx) CtxFromGreenCtx = nullptr;
  decltype(&cuCtxSetCurrent) CtxSetCurrent = nullptr;
  decltype(&cuStreamDestroy) StreamDestroy = nullptr;
  decltype(&cuGetErrorString) GetErrorString = nullptr;
  decltype(&cuTensorMapEncodeTiled) TensorMapEncodeTiled = nullptr;
  bool ok = false;
};

static Drv& drv() {
  static Drv d;
  static bool tried = false;
  if (!tried) {
    tried = true;
    bool ok = true;
    auto get = [&](const char* name, void** fp) {
      cudaDriverEntryPointQueryResult q;
      if (cudaGetDriverEntryPoint(name, fp, cudaEnableDefault, &q) != cudaSuccess ||
          q != cudaDriverEntryPointSuccess || !*fp)
        ok = false;
    };
    get("cuInit", (void**)&d.Init);
    get("cuDeviceGet", (void**)&d.DeviceGet);
    get("cuDeviceGetDevResource", (void**)&d.DeviceGetDevResource);
    get("cuDevSmResourceSplitByCount", (void**)&d.DevSmResourceSplitByCount);
    get("cuDevResourceGenerateDesc", (void**)&d.DevResourceGenerateDesc);
    get("cuGreenCtxCreate", (void**)&d.GreenCtxCreate);
    get("cuGreenCtxStreamCreate", (void**)&d.GreenCtxStreamCreate);
    get("cuGreenCtxDestroy", (void**)&d.GreenCtxDestroy);
    get("cuCtxFromGreenCtx", (void**)&d.CtxFromGreenCtx);
    get("cuCtxSetCurrent", (void**)&d.CtxSetCurrent);
    get("cuStreamDestroy", (void**)&d.StreamDestroy);
    get("cuGetErrorString", (void**)&d.GetErrorString);
    d.ok = ok;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&d.TensorMapEncodeTiled, cudaEnableDefault,
                                &q) != cudaSuccess || q != cudaDriverEntryPointSuccess)
      d.TensorMapEncodeTiled = nullptr;
  }
  return d;
}

// NCCL entry points, resolved with dlopen when a multi-process context is
// created: the library does not link libnccl, so it never pins a second NCCL
// build into a process that also loads torch's (torch's is reused when present).
struct Nccl {
  decltype(&ncclGetUniqueId) GetUniqueId = nullptr;
  decltype(&ncclCommInitRank) CommInitRank = nullptr;
  decltype(&ncclCommDestroy) CommDestroy = nullptr;
  decltype(&ncclGroupStart) GroupStart = nullptr;
  decltype(&ncclGroupEnd) GroupEnd = nullptr;
  decltype(&ncclSend) Send = nullptr;
  decltype(&ncclRecv) Recv = nullptr;
  decltype(&ncclAllReduce) AllReduce = nullptr;
  decltype(&ncclAllGather) AllGather = nullptr;
  decltype(&ncclGetErrorString) GetErrorString = nullptr;
  bool ok = false;
};

static Nccl& nccl() {
  static Nccl n;
  static bool tried = false;
  if (!tried) {
    tried = true;
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);  // already loaded (torch)?
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_LOCAL);
    if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_LOCAL);
    if (!h) return n;
    bool ok = true;
    auto get = [&](const char* name, void** fp) {
      *fp = dlsym(h, name);
      if (!*fp) ok = false;
    };
    get("ncclGetUniqueId", (void**)&n.GetUniqueId);
    get("ncclCommInitRank", (void**)&n.CommInitRank);
    get("ncclCommDestroy", (void**)&n.CommDestroy);
    get("ncclGroupStart", (void**)&n.GroupStart);
    get("ncclGroupEnd", (void**)&n.GroupEnd);
    get("ncclSend", (void**)&n.Send);
    get("ncclRecv", (void**)&n.Recv);
    get("ncclAllReduce", (void**)&n.AllReduce);
    get("ncclAllGather", (void**)&n.AllGather);
    get("ncclGetErrorString", (void**)&n.GetErrorString);
    n.ok = ok;
  }
  return n;
}

struct mm_ctx {
  std::vector<DevRt> dev;
  int32_t G = 0, my_rank = 0, world = 1;
  ncclComm_t comm = nullptr;
  bool poisoned = false;
  float* bar_buf = nullptr;        // NCCL barrier scratch (1 float)
  std::vector<void*> flush_scratch;  // per buffer slot, pinned (lazily)
  std::vector<size_t> flush_scratch_bytes;
  // mm_buffer_register: caller-owned per-device pointers, slot = registration order
  std::vector<std::vector<void*>> reg;
  std::vector<std::pair<int32_t, int64_t>> reg_shape;
  // mm_ctx_set_stream: caller streams the runs of a device are ordered with
  std::vector<cudaStream_t> ext;
  std::vector<cudaEvent_t> ext_ev;    // created in the caller stream's (primary) context
  std::vector<cudaEvent_t> lib_ev;    // created in the device's own (possibly green) context
  // world > 1: IPC transport (default) or NCCL (MM_TRANSPORT=nccl)
  IpcChannel* ipc = nullptr;
  std::vector<char*> ipc_bufs;        // [slot * world + rank]: pointers valid in this process
};

namespace {

#define CU_OK(expr)                                                              \
  do {                                                                           \
    cudaError_t e_ = (expr);                                                     \
    if (e_ != cudaSuccess) {                                                     \
      if (ctx) ctx->poisoned = true;                                             \
      MM_FAIL(MM_ECUDA, "%s failed: %s (%s:%d)", #expr, cudaGetErrorString(e_), __FILE__, __LINE__); \
    }                                                                            \
  } while (0)

#define DRV_OK(expr)                                                             \
  do {                                                                           \
    CUresult r_ = (expr);                                                        \
    if (r_ != CUDA_SUCCESS) {                                                    \
      const char* s_ = nullptr;                                                  \
      if (drv().GetErrorString) drv().GetErrorString(r_, &s_);                   \
      MM_FAIL(MM_ECUDA, "%s failed: %s", #expr, s_ ? s_ : "?");                  \
    }                                                                            \
  } while (0)

#define NCCL_OK(expr)                                                            \
  do {                                                                           \
    ncclResult_t r_ = (expr);                                                    \
    if (r_ != ncclSuccess) {                                                     \
      if (ctx) ctx->poisoned = true;                                             \
      MM_FAIL(MM_ENCCL, "%s failed: %s", #expr, nccl().GetErrorString(r_));      \
    }                                                                            \
  } while (0)

constexpr int kKinds = 4;   // streams per logical device (see sid_stream)

// Adaptive DP-Perf state of a plan: the op program built incrementally at run
// time (its ownership directory persists across runs), one end event per op,
// a begin event per kernel op, and the decision log of the last run.
struct AdaptiveState {
  Plan ap;
  IncPlanner* inc = nullptr;
  std::vector<mm_decision> decisions;
  std::vector<cudaEvent_t> ev_end, ev_beg;
  std::vector<int32_t> ev_dev;
  cudaEvent_t t0 = nullptr;
  ~AdaptiveState() {
    for (auto e : ev_end)
      if (e) cudaEventDestroy(e);
    for (auto e : ev_beg)
      if (e) cudaEventDestroy(e);
    if (t0) cudaEventDestroy(t0);
    if (inc) inc_planner_destroy(inc);
  }
};

struct PlanRt {
  mm_ctx* ctx = nullptr;
  AdaptiveState* ad = nullptr;
  bool last_adaptive = false;
  std::vector<cudaEvent_t> ev;           // per op that another stream waits on
  std::vector<cudaEvent_t> bar_ev;       // per device
  std::vector<cudaEvent_t> join_ev;      // per device
  cudaEvent_t fork = nullptr;
  cudaEvent_t t_start = nullptr, t_stop = nullptr;
  std::vector<cudaEvent_t> kev;          // 2 per kernel op (timing)
  cudaGraphExec_t gexec = nullptr;
  cudaGraph_t graph = nullptr;
  std::vector<void*> graph_bufs;
  int64_t graph_launches = 0;
  int64_t graph_xfer = 0, graph_h2d = 0, graph_d2h = 0;
  // DAG task batching: members[head] = kernel ops launched together with head
  std::vector<int64_t> batch_head;               // -1: not a member of another op's batch
  std::vector<std::vector<int64_t>> members;
  // IPC transport: op i is waited on by another rank's stream (signal its flag)
  std::vector<uint8_t> remote_sig;
};

bool is_batchable_op(int32_t op) {
  return op == MM_OP_CHOL_TRSM || op == MM_OP_CHOL_SYRK || op == MM_OP_CHOL_GEMM;
}
bool is_chol_update(int32_t op) { return op == MM_OP_CHOL_SYRK || op == MM_OP_CHOL_GEMM; }

// Group consecutive independent kernel ops of one device and one kernel into
// one launch (MK-DAG steps: all TRSMs / SYRKs / GEMMs of a step on a device).
// A member joins only if no other op of that device lies between, all of its
// cross-stream waits point before the head, and it neither reads nor writes
// what an earlier member writes (nor writes what an earlier member reads).
// Batch key: tasks of one batch must share it.  Cholesky lookahead: the GEMM
// updates of column k+1 and SYRK(k+1, k) run as their own launches, so step
// k+1's POTRF / TRSM (lane 1) wait only for the updates they read; the rest
// of step k's SYRKs and GEMMs is one launch (no per-column waves of partial
// occupancy; the task order puts them next to each other, R34).
int64_t batch_key(const Kernel& k, const Task& t) {
  static const int merge = getenv("MM_CHOL_MERGE_SYRK") ? atoi(getenv("MM_CHOL_MERGE_SYRK")) : 1;
  if (k.op == MM_OP_CHOL_GEMM) return t.ip[2] * 4 + (t.ip[1] == t.ip[2] + 1 ? 1 : 0);
  if (k.op == MM_OP_CHOL_SYRK) return t.ip[2] * 4 + (t.ip[0] == t.ip[2] + 1 ? 1 : (merge ? 0 : 2));
  return t.ip[2];
}

void compute_batches(const Plan& plan, PlanRt* rt) {
  const size_t n = plan.ops.size();
  rt->batch_head.assign(n, -1);
  rt->members.assign(n, {});
  if (!plan.app.is_dag) return;
  std::vector<int64_t> open(kKinds * plan.G, -1);   // open batch head per stream
  auto overlap = [](const TaskAcc& a, const TaskAcc& b) {
    return a.buffer == b.buffer && a.lo < b.hi && b.lo < a.hi;
  };
  for (size_t i = 0; i < n; ++i) {
    const mm_op_rec& op = plan.ops[i];
    if (op.kind == MM_OPK_BARRIER) {
      std::fill(open.begin(), open.end(), -1);
      continue;
    }
    const int32_t sid = plan.op_stream[i];
    if (op.kind != MM_OPK_KERNEL || !is_batchable_op(plan.app.kernels[op.kernel].op)) {
      open[sid] = -1;   // any other op on the stream ends its batch
      continue;
    }
    const Task& t = plan.tasks[op.task];
    const Kernel& kern = plan.app.kernels[op.kernel];
    int64_t h = open[sid];
    const Kernel& hk = plan.app.kernels[h >= 0 ? plan.ops[h].kernel : op.kernel];
    const bool same = h >= 0 && (plan.ops[h].kernel == op.kernel || (is_chol_update(hk.op) && is_chol_update(kern.op)));
    bool ok = same && (int64_t)rt->members[h].size() + 1 < kCholBatch &&
              batch_key(hk, plan.tasks[plan.ops[h].task]) == batch_key(kern, t);
    if (ok)
      for (auto& w : plan.waits[i])
        if (w.op >= h) ok = false;
    if (ok) {
      std::vector<int64_t> grp = rt->members[h];
      grp.push_back(h);
      for (int64_t m : grp) {
        const Task& u = plan.tasks[plan.ops[m].task];
        for (auto& a : t.acc)
          for (auto& c : u.acc)
            if (overlap(a, c) && ((a.mode & MM_WRITE) || (c.mode & MM_WRITE))) ok = false;
      }
    }
    if (ok) {
      rt->members[h].push_back((int64_t)i);
      rt->batch_head[i] = h;
    } else {
      open[sid] = (int64_t)i;
    }
  }
}

cudaError_t set_dev(mm_ctx* ctx, int32_t d) {
  const DevRt& r = ctx->dev[d];
  if (r.gcu) return drv().CtxSetCurrent(r.gcu) == CUDA_SUCCESS ? cudaSuccess : cudaErrorDeviceUninitialized;
  return cudaSetDevice(r.phys);
}

void destroy_rt(PlanRt* rt) {
  if (!rt) return;
  for (auto e : rt->ev)
    if (e) cudaEventDestroy(e);
  for (auto e : rt->bar_ev)
    if (e) cudaEventDestroy(e);
  for (auto e : rt->join_ev)
    if (e) cudaEventDestroy(e);
  for (auto e : rt->kev)
    if (e) cudaEventDestroy(e);
  if (rt->fork) cudaEventDestroy(rt->fork);
  if (rt->t_start) cudaEventDestroy(rt->t_start);
  if (rt->t_stop) cudaEventDestroy(rt->t_stop);
  if (rt->gexec) cudaGraphExecDestroy(rt->gexec);
  if (rt->graph) cudaGraphDestroy(rt->graph);
  delete rt->ad;
  delete rt;
}

int32_t first_owned(const mm_ctx* ctx) {
  for (int32_t d = 0; d < ctx->G; ++d)
    if (ctx->dev[d].mine) return d;
  return -1;
}

// Op stream ids of the planner: sid = kind * G + d (kind 0 compute lane 0,
// 1 H2D, 2 D2H, 3 compute lane 1); kKinds is defined with PlanRt.
inline int32_t sid_dev(const mm_ctx* ctx, int32_t sid) { return sid % ctx->G; }
inline cudaStream_t sid_stream(const mm_ctx* ctx, int32_t sid) {
  const DevRt& r = ctx->dev[sid % ctx->G];
  const int32_t kind = sid / ctx->G;
  return kind == 0 ? r.stream : (kind == 1 ? r.h2d : (kind == 2 ? r.d2h : r.lane1));
}

}  // namespace

namespace mm {

// 2-D fp32 tensor map; the swizzle span equals the box row (box_inner * 4 =
// 128, 64 or 32 bytes -> SWIZZLE_128B / 64B / 32B).
cudaError_t encode_tmap_2d_f32(CUtensorMap* m, const void* base, uint64_t inner, uint64_t outer,
                               uint64_t row_bytes, uint32_t box_inner, uint32_t box_outer) {
  Drv& D = drv();
  if (!D.TensorMapEncodeTiled) return cudaErrorNotSupported;
  const cuuint64_t dims[2] = {inner, outer};
  const cuuint64_t strides[1] = {row_bytes};
  const cuuint32_t box[2] = {box_inner, box_outer};
  const cuuint32_t estr[2] = {1, 1};
  CUresult r = D.TensorMapEncodeTiled(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<void*>(base), dims, strides,
                                      box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                                      box_inner * 4 == 128 ? CU_TENSOR_MAP_SWIZZLE_128B
                                      : box_inner * 4 == 64 ? CU_TENSOR_MAP_SWIZZLE_64B
                                                            : CU_TENSOR_MAP_SWIZZLE_32B,
                                      CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS ? cudaSuccess : cudaErrorInvalidValue;
}

size_t builtin_scratch_bytes(const Kernel& k, const Task& t) {
  if (k.op == MM_OP_SGEMM && (k.ip[3] == 0 || k.ip[3] == 2))
    return sgemm_tf32x3_scratch(k.ip[1], k.ip[2], t.e - t.b);
  if (k.op == MM_OP_CHOL_POTRF || k.op == MM_OP_CHOL_TRSM || k.op == MM_OP_CHOL_SYRK || k.op == MM_OP_CHOL_GEMM)
    return chol_scratch_bytes(k.ip[0], k.ip[1]);
  return 0;
}

void plan_runtime_free(Plan* plan) {
  destroy_rt(static_cast<PlanRt*>(plan->rt));
  plan->rt = nullptr;
}

cudaError_t launch_builtin(const Launch& L) {
  const Kernel& k = *L.k;
  const Task& t = *L.t;
  const int64_t b = t.b, e = t.e;
  float* const* f = reinterpret_cast<float* const*>(L.opnd);
  switch (k.op) {
    case MM_OP_STREAM_COPY: return stream_copy(f[0], f[1], b, e, L.stream, L.sms);
    case MM_OP_STREAM_SCALE: return stream_scale(f[0], f[1], (float)k.fp[0], b, e, L.stream, L.sms);
    case MM_OP_STREAM_ADD: return stream_add(f[0], f[1], f[2], b, e, L.stream, L.sms);
    case MM_OP_STREAM_TRIAD: return stream_triad(f[0], f[1], f[2], (float)k.fp[0], b, e, L.stream, L.sms);
    case MM_OP_HOTSPOT: {
      HotCoef c{(float)k.fp[0], (float)k.fp[1], (float)k.fp[2], (float)k.fp[3], (float)k.fp[4]};
      return hotspot_rows(f[0], f[1], f[2], k.ip[0], k.ip[1], b, e, c, L.stream, L.sms,
                          k.ip[2] > 1 ? (int)k.ip[2] : 1);
    }
    case MM_OP_ROW_RESIDUAL:
      return row_residual(f[0], f[1], reinterpret_cast<double*>(L.opnd[2]), k.ip[1], b, e, L.stream, L.sms);
    case MM_OP_BLACKSCHOLES:
      return blackscholes(f[0], f[1], f[2], f[3], f[4], (float)k.fp[0], (float)k.fp[1], b, e, L.stream, L.sms);
    case MM_OP_SGEMM: {
      const int32_t variant = k.ip[3] == 0 ? 2 : (int32_t)k.ip[3];
      return sgemm_rows(f[0], f[1], f[2], k.ip[0], k.ip[1], k.ip[2], b, e, variant, L.stream, L.sms, L.scr,
                        (L.ro_mask >> 1) & 1u);
    }
    case MM_OP_NBODY:
      return nbody_rows_launch(f[0], f[1], f[2], f[3], k.ip[0], b, e, (float)k.fp[0], (float)k.fp[1], L.stream);
    case MM_OP_CHOL_POTRF:
    case MM_OP_CHOL_TRSM:
    case MM_OP_CHOL_SYRK:
    case MM_OP_CHOL_GEMM: {
      const int32_t ijk[3] = {(int32_t)t.ip[0], (int32_t)t.ip[1], (int32_t)t.ip[2]};
      return chol_batch(k.op, f[0], k.ip[0], k.ip[1], ijk, 1, L.stream, L.sms, L.scr);
    }
  }
  return cudaErrorNotSupported;
}

}  // namespace mm

namespace {

// Launch the task's kernel on logical device d.
uint32_t readonly_mask(const App& app, const Task& t) {
  uint32_t m = 0;
  for (size_t i = 0; i < t.acc.size() && i < 32; ++i) {
    bool written = false;
    for (auto& k : app.kernels)
      for (auto& a : k.acc)
        if ((a.mode & MM_WRITE) && (a.buffer == t.acc[i].buffer ||
                                    phys_buffer(app, a.buffer, 1) == t.acc[i].buffer))
          written = true;
    for (auto& dt : app.dag)
      for (auto& a : dt.acc)
        if ((a.mode & MM_WRITE) && a.buffer == t.acc[i].buffer) written = true;
    if (!written) m |= 1u << i;
  }
  return m;
}

mm_status launch_task(mm_ctx* ctx, const App& app, const Task& t, int32_t d, void* const* buffers,
                      cudaStream_t s) {
  const Kernel& k = app.kernels[t.kernel];
  void* opnd[MM_MAX_ACCESS];
  const int32_t G = ctx->G;
  for (size_t i = 0; i < t.acc.size() && i < MM_MAX_ACCESS; ++i) {
    opnd[i] = buffers[(size_t)t.acc[i].buffer * G + d];
    if (!opnd[i]) MM_FAIL(MM_EINVAL, "run: buffer slot %d has no pointer on device %d", t.acc[i].buffer, d);
  }
  cudaError_t e;
  if (k.op == MM_OP_CUSTOM) {
    e = (cudaError_t)k.launch(k.user, d, mm_range{t.b, t.e}, opnd, (void*)s);
  } else {
    DevRt& dv = ctx->dev[d];
    const size_t need = builtin_scratch_bytes(k, t);
    if (need > dv.scr.bytes) {
      cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
      cudaStreamIsCapturing(s, &cs);
      if (cs != cudaStreamCaptureStatusNone) MM_FAIL(MM_ESTATE, "scratch not reserved before graph capture");
      if (dv.scr.ptr) {
        cudaStreamSynchronize(s);
        cudaFree(dv.scr.ptr);
      }
      dv.scr = Scratch{nullptr, 0, nullptr, 0, 0, 0, dv.scr.epoch + 1, {}};
      if (cudaMalloc(&dv.scr.ptr, need) != cudaSuccess) MM_FAIL(MM_ENOMEM, "device scratch of %zu bytes", need);
      dv.scr.bytes = need;
    }
    Launch L{&k, &t, opnd, s, dv.sms, &dv.scr, readonly_mask(app, t)};
    e = launch_builtin(L);
  }
  if (e == cudaErrorNotSupported) MM_FAIL(MM_ENOTSUP, "kernel %s (op %d) has no sm_100a implementation yet", k.name.c_str(), k.op);
  if (e != cudaSuccess) {
    ctx->poisoned = true;
    MM_FAIL(MM_ECUDA, "kernel %s launch failed: %s", k.name.c_str(), cudaGetErrorString(e));
  }
  return MM_OK;
}

// Launch independent DAG tasks of one kernel as one batched kernel.
mm_status launch_task_batch(mm_ctx* ctx, const App& app, const std::vector<const Task*>& ts, int32_t d,
                            void* const* buffers, cudaStream_t s) {
  const Task& t0 = *ts[0];
  const Kernel& k = app.kernels[t0.kernel];
  std::vector<int32_t> ijk;
  for (const Task* t : ts) {
    ijk.push_back((int32_t)t->ip[0]);
    ijk.push_back((int32_t)t->ip[1]);
    ijk.push_back((int32_t)t->ip[2]);
  }
  float* A = static_cast<float*>(buffers[(size_t)t0.acc[0].buffer * ctx->G + d]);
  if (!A) MM_FAIL(MM_EINVAL, "run: buffer slot %d has no pointer on device %d", t0.acc[0].buffer, d);
  DevRt& dv = ctx->dev[d];
  const size_t need = builtin_scratch_bytes(k, t0);
  if (need > dv.scr.bytes) {  // reserved by ensure_rt; only profile paths get here
    cudaStreamSynchronize(s);
    if (dv.scr.ptr) cudaFree(dv.scr.ptr);
    dv.scr = Scratch{nullptr, 0, nullptr, 0, 0, 0, dv.scr.epoch + 1, {}};
    if (cudaMalloc(&dv.scr.ptr, need) != cudaSuccess) MM_FAIL(MM_ENOMEM, "device scratch of %zu bytes", need);
    dv.scr.bytes = need;
  }
  cudaError_t e = chol_batch(k.op, A, k.ip[0], k.ip[1], ijk.data(), (int32_t)(ijk.size() / 3), s, dv.sms, &dv.scr);
  if (e != cudaSuccess) {
    ctx->poisoned = true;
    MM_FAIL(MM_ECUDA, "batched %s launch failed: %s", k.name.c_str(), cudaGetErrorString(e));
  }
  return MM_OK;
}

// Launch a batch head together with its members (one batched kernel).
mm_status launch_batch(mm_ctx* ctx, const Plan& plan, const PlanRt* rt, int64_t head, int32_t d,
                       void* const* buffers, cudaStream_t s) {
  std::vector<const Task*> ts{&plan.tasks[plan.ops[head].task]};
  for (int64_t m : rt->members[head]) ts.push_back(&plan.tasks[plan.ops[m].task]);
  return launch_task_batch(ctx, plan.app, ts, d, buffers, s);
}

mm_status ensure_rt(mm_ctx* ctx, Plan& plan, bool timing) {
  PlanRt* rt = static_cast<PlanRt*>(plan.rt);
  if (rt && rt->ctx != ctx) {
    destroy_rt(rt);
    rt = nullptr;
    plan.rt = nullptr;
  }
  if (!rt) {
    rt = new PlanRt();
    rt->ctx = ctx;
    plan.rt = rt;
    const int32_t G = ctx->G;
    rt->ev.assign(plan.ops.size(), nullptr);
    for (size_t i = 0; i < plan.ops.size(); ++i)
      if (plan.needs_event[i] && plan.op_stream[i] >= 0 && ctx->dev[sid_dev(ctx, plan.op_stream[i])].mine) {
        CU_OK(set_dev(ctx, sid_dev(ctx, plan.op_stream[i])));
        CU_OK(cudaEventCreateWithFlags(&rt->ev[i], cudaEventDisableTiming));
      }
    rt->bar_ev.assign(kKinds * G, nullptr);
    rt->join_ev.assign(kKinds * G, nullptr);
    for (int32_t sid = 0; sid < kKinds * G; ++sid) {
      if (!ctx->dev[sid % G].mine) continue;
      CU_OK(set_dev(ctx, sid % G));
      CU_OK(cudaEventCreateWithFlags(&rt->bar_ev[sid], cudaEventDisableTiming));
      CU_OK(cudaEventCreateWithFlags(&rt->join_ev[sid], cudaEventDisableTiming));
    }
    const int32_t root = first_owned(ctx);
    CU_OK(set_dev(ctx, root));
    CU_OK(cudaEventCreateWithFlags(&rt->fork, cudaEventDisableTiming));
    CU_OK(cudaEventCreate(&rt->t_start));
    CU_OK(cudaEventCreate(&rt->t_stop));
    compute_batches(plan, rt);
    rt->remote_sig.assign(plan.ops.size(), 0);
    if (ctx->ipc)
      for (size_t j = 0; j < plan.ops.size(); ++j) {
        if (plan.op_stream[j] < 0) continue;
        const int32_t rj = ctx->dev[sid_dev(ctx, plan.op_stream[j])].rank;
        for (auto& w : plan.waits[j])
          if (ctx->dev[sid_dev(ctx, w.dev)].rank != rj) rt->remote_sig[w.op] = 1;
      }
  }
  // reserve device scratch for every kernel op before any graph capture
  for (size_t i = 0; i < plan.ops.size(); ++i) {
    const mm_op_rec& op = plan.ops[i];
    if (op.kind != MM_OPK_KERNEL || !ctx->dev[op.device].mine) continue;
    const Task& t = plan.tasks[op.task];
    DevRt& dv = ctx->dev[op.device];
    const size_t need = builtin_scratch_bytes(plan.app.kernels[t.kernel], t);
    if (need > dv.scr.bytes) {
      CU_OK(set_dev(ctx, op.device));
      CU_OK(cudaDeviceSynchronize());
      if (dv.scr.ptr) cudaFree(dv.scr.ptr);
      dv.scr = Scratch{nullptr, 0, nullptr, 0, 0, 0, dv.scr.epoch + 1, {}};
      CU_OK(cudaMalloc(&dv.scr.ptr, need));
      dv.scr.bytes = need;
    }
  }
  if (timing && rt->kev.empty()) {
    rt->kev.assign(plan.ops.size() * 2, nullptr);
    for (size_t i = 0; i < plan.ops.size(); ++i)
      if (plan.ops[i].kind == MM_OPK_KERNEL && ctx->dev[plan.ops[i].device].mine) {
        CU_OK(set_dev(ctx, plan.ops[i].device));
        CU_OK(cudaEventCreate(&rt->kev[2 * i]));
        CU_OK(cudaEventCreate(&rt->kev[2 * i + 1]));
      }
  }
  return MM_OK;
}

void* flush_target(mm_ctx* ctx, const Plan& plan, const mm_run_opts* o, int32_t buf, size_t bytes_total,
                   mm_status* st) {
  *st = MM_OK;
  if (o && o->host && o->host[buf]) return o->host[buf];
  if (ctx->flush_scratch.size() <= (size_t)buf) {
    ctx->flush_scratch.resize(buf + 1, nullptr);
    ctx->flush_scratch_bytes.resize(buf + 1, 0);
  }
  if (ctx->flush_scratch_bytes[buf] < bytes_total) {
    if (ctx->flush_scratch[buf]) cudaFreeHost(ctx->flush_scratch[buf]);
    ctx->flush_scratch[buf] = nullptr;
    if (cudaMallocHost(&ctx->flush_scratch[buf], bytes_total) != cudaSuccess) {
      set_error("pinned flush scratch of %zu bytes", bytes_total);
      *st = MM_ENOMEM;
      return nullptr;
    }
    ctx->flush_scratch_bytes[buf] = bytes_total;
  }
  (void)plan;
  return ctx->flush_scratch[buf];
}

// Issue the op program of an in-process ctx (world == 1) onto the streams.
// Kernel-timing events: inside a stream capture a plain cudaEventRecord only
// orders streams; the external flag makes it an event record node of the
// graph, so graph replays carry the timing too.
cudaError_t rec_kev(cudaEvent_t ev, cudaStream_t s) {
  cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
  cudaStreamIsCapturing(s, &cs);
  return cudaEventRecordWithFlags(ev, s, cs == cudaStreamCaptureStatusActive ? cudaEventRecordExternal
                                                                             : cudaEventRecordDefault);
}

mm_status issue_local(mm_ctx* ctx, Plan& plan, void* const* buffers, const mm_run_opts* o, bool timing,
                      mm_run_stats* st) {
  PlanRt* rt = static_cast<PlanRt*>(plan.rt);
  const int32_t G = ctx->G;
  const App& app = plan.app;
  const int32_t NS = kKinds * G;
  std::vector<uint8_t> used(NS, 0);
  for (int32_t d : plan.task_dev) used[d] = 1;
  for (size_t i = 0; i < plan.ops.size(); ++i)
    if (plan.op_stream[i] >= 0) used[plan.op_stream[i]] = 1;
  const int32_t root = first_owned(ctx);
  used[root] = 1;
  // fork
  CU_OK(set_dev(ctx, root));
  CU_OK(cudaEventRecord(rt->fork, ctx->dev[root].stream));
  for (int32_t sid = 0; sid < NS; ++sid)
    if (used[sid] && sid != root) {
      CU_OK(set_dev(ctx, sid_dev(ctx, sid)));
      CU_OK(cudaStreamWaitEvent(sid_stream(ctx, sid), rt->fork, 0));
    }
  for (size_t i = 0; i < plan.ops.size(); ++i) {
    const mm_op_rec& op = plan.ops[i];
    if (op.kind == MM_OPK_BARRIER) {
      for (int32_t sid = 0; sid < NS; ++sid)
        if (used[sid]) {
          CU_OK(set_dev(ctx, sid_dev(ctx, sid)));
          CU_OK(cudaEventRecord(rt->bar_ev[sid], sid_stream(ctx, sid)));
        }
      for (int32_t sid = 0; sid < NS; ++sid)
        if (used[sid]) {
          CU_OK(set_dev(ctx, sid_dev(ctx, sid)));
          for (int32_t q = 0; q < NS; ++q)
            if (used[q] && q != sid) CU_OK(cudaStreamWaitEvent(sid_stream(ctx, sid), rt->bar_ev[q], 0));
        }
      continue;
    }
    const int32_t d = sid_dev(ctx, plan.op_stream[i]);
    cudaStream_t s = sid_stream(ctx, plan.op_stream[i]);
    if (op.kind == MM_OPK_KERNEL && rt->batch_head[i] >= 0) continue;  // launched with its head
    CU_OK(set_dev(ctx, d));
    for (auto& w : plan.waits[i]) CU_OK(cudaStreamWaitEvent(s, rt->ev[w.op], 0));
    if (op.kind == MM_OPK_KERNEL && !rt->members[i].empty()) {
      for (int64_t m : rt->members[i])
        for (auto& w : plan.waits[m]) CU_OK(cudaStreamWaitEvent(s, rt->ev[w.op], 0));
      if (timing) CU_OK(rec_kev(rt->kev[2 * i], s));
      mm_status r = launch_batch(ctx, plan, rt, (int64_t)i, d, buffers, s);
      if (r) return r;
      if (timing) CU_OK(rec_kev(rt->kev[2 * i + 1], s));
      for (int64_t m : rt->members[i])
        if (plan.needs_event[m]) CU_OK(cudaEventRecord(rt->ev[m], s));
    } else if (op.kind == MM_OPK_KERNEL) {
      if (timing) CU_OK(rec_kev(rt->kev[2 * i], s));
      mm_status r = launch_task(ctx, app, plan.tasks[op.task], d, buffers, s);
      if (r) return r;
      if (timing) CU_OK(rec_kev(rt->kev[2 * i + 1], s));
    } else if (op.kind == MM_OPK_XFER) {
      const int64_t eb = app.buffers[op.buffer].first;
      const size_t bytes = (size_t)((op.r.end - op.r.begin) * eb);
      char* dst = static_cast<char*>(buffers[(size_t)op.buffer * G + d]) + op.r.begin * eb;
      if (op.src < 0) {
        if (!o || !o->host || !o->host[op.buffer]) MM_FAIL(MM_EINVAL, "staged run: no host pointer for slot %d", op.buffer);
        const char* src = static_cast<const char*>(o->host[op.buffer]) + op.r.begin * eb;
        CU_OK(cudaMemcpyAsync(dst, src, bytes, cudaMemcpyHostToDevice, s));
        st->h2d_bytes += (int64_t)bytes;
      } else {
        const char* src = static_cast<const char*>(buffers[(size_t)op.buffer * G + op.src]) + op.r.begin * eb;
        if (ctx->dev[op.src].phys == ctx->dev[d].phys)
          CU_OK(cudaMemcpyAsync(dst, src, bytes, cudaMemcpyDeviceToDevice, s));
        else
          CU_OK(cudaMemcpyPeerAsync(dst, ctx->dev[d].phys, src, ctx->dev[op.src].phys, bytes, s));
        st->xfer_bytes += (int64_t)bytes;
      }
    } else if (op.kind == MM_OPK_FLUSH) {
      const int64_t eb = app.buffers[op.buffer].first;
      const size_t bytes = (size_t)((op.r.end - op.r.begin) * eb);
      mm_status fs;
      char* host = static_cast<char*>(flush_target(ctx, plan, o, op.buffer,
                                                   (size_t)(app.buffers[op.buffer].second * eb), &fs));
      if (fs) return fs;
      const char* src = static_cast<const char*>(buffers[(size_t)op.buffer * G + d]) + op.r.begin * eb;
      CU_OK(cudaMemcpyAsync(host + op.r.begin * eb, src, bytes, cudaMemcpyDeviceToHost, s));
      st->d2h_bytes += (int64_t)bytes;
    }
    if (plan.needs_event[i]) CU_OK(cudaEventRecord(rt->ev[i], s));
  }
  // join
  for (int32_t sid = 0; sid < NS; ++sid)
    if (used[sid] && sid != root) {
      CU_OK(set_dev(ctx, sid_dev(ctx, sid)));
      CU_OK(cudaEventRecord(rt->join_ev[sid], sid_stream(ctx, sid)));
      CU_OK(set_dev(ctx, root));
      CU_OK(cudaStreamWaitEvent(ctx->dev[root].stream, rt->join_ev[sid], 0));
    }
  return MM_OK;
}

// Issue the op program of one rank of a multi-process ctx: kernels of the
// owned device, NCCL send/recv for transfers touching it (grouped), an NCCL
// all-reduce of one float per BARRIER, D2H for its FLUSH ops.
mm_status issue_dist(mm_ctx* ctx, Plan& plan, void* const* buffers, const mm_run_opts* o, bool timing,
                     mm_run_stats* st) {
  PlanRt* rt = static_cast<PlanRt*>(plan.rt);
  const int32_t G = ctx->G;
  const int32_t me = first_owned(ctx);
  const App& app = plan.app;
  cudaStream_t s = ctx->dev[me].stream;
  CU_OK(set_dev(ctx, me));
  bool in_group = false;
  for (size_t i = 0; i < plan.ops.size(); ++i) {
    const mm_op_rec& op = plan.ops[i];
    const bool x = op.kind == MM_OPK_XFER && op.src >= 0 && (op.device == me || op.src == me);
    if (in_group && !(op.kind == MM_OPK_XFER && op.src >= 0)) {
      NCCL_OK(nccl().GroupEnd());
      in_group = false;
    }
    if (op.kind == MM_OPK_BARRIER) {
      NCCL_OK(nccl().AllReduce(ctx->bar_buf, ctx->bar_buf, 1, ncclFloat, ncclSum, ctx->comm, s));
      continue;
    }
    if (op.kind == MM_OPK_KERNEL) {
      if (op.device != me || rt->batch_head[i] >= 0) continue;
      if (timing) CU_OK(rec_kev(rt->kev[2 * i], s));
      mm_status r = rt->members[i].empty() ? launch_task(ctx, app, plan.tasks[op.task], me, buffers, s)
                                            : launch_batch(ctx, plan, rt, (int64_t)i, me, buffers, s);
      if (r) return r;
      if (timing) CU_OK(rec_kev(rt->kev[2 * i + 1], s));
      continue;
    }
    const int64_t eb = app.buffers[op.buffer].first;
    const size_t bytes = (size_t)((op.r.end - op.r.begin) * eb);
    if (op.kind == MM_OPK_XFER && op.src < 0) {
      if (op.device != me) continue;
      if (!o || !o->host || !o->host[op.buffer]) MM_FAIL(MM_EINVAL, "staged run: no host pointer for slot %d", op.buffer);
      char* dst = static_cast<char*>(buffers[(size_t)op.buffer * G + me]) + op.r.begin * eb;
      CU_OK(cudaMemcpyAsync(dst, static_cast<const char*>(o->host[op.buffer]) + op.r.begin * eb, bytes,
                            cudaMemcpyHostToDevice, s));
      st->h2d_bytes += (int64_t)bytes;
      continue;
    }
    if (x) {
      if (!in_group) {
        NCCL_OK(nccl().GroupStart());
        in_group = true;
      }
      char* mine = static_cast<char*>(buffers[(size_t)op.buffer * G + me]) + op.r.begin * eb;
      if (op.device == me)
        NCCL_OK(nccl().Recv(mine, bytes, ncclChar, ctx->dev[op.src].rank, ctx->comm, s));
      else
        NCCL_OK(nccl().Send(mine, bytes, ncclChar, ctx->dev[op.device].rank, ctx->comm, s));
      st->xfer_bytes += op.device == me ? (int64_t)bytes : 0;
      continue;
    }
    if (op.kind == MM_OPK_FLUSH && op.device == me) {
      mm_status fs;
      char* host = static_cast<char*>(flush_target(ctx, plan, o, op.buffer,
                                                   (size_t)(app.buffers[op.buffer].second * eb), &fs));
      if (fs) return fs;
      CU_OK(cudaMemcpyAsync(host + op.r.begin * eb,
                            static_cast<const char*>(buffers[(size_t)op.buffer * G + me]) + op.r.begin * eb,
                            bytes, cudaMemcpyDeviceToHost, s));
      st->d2h_bytes += (int64_t)bytes;
    }
  }
  if (in_group) NCCL_OK(nccl().GroupEnd());
  return MM_OK;
}

// Issue the op program of one rank of a multi-process ctx on the IPC
// transport: the in-process executor's program (four streams, exact
// hazards) restricted to the owned device, with every hazard on another
// rank's op turned into a wait on that rank's completion flag, every op a
// peer waits on followed by a flag signal, pulls copying straight out of the
// peer's buffer (ctx->ipc_bufs), and BARRIER = join, signal, wait for every
// rank, fork.  A run starts by bumping this rank's epoch and waiting for
// every peer to have finished the previous run (cross-run WAR on pulled
// ranges); it ends by signalling its own end.  Capturable as a CUDA graph.
mm_status issue_ipc(mm_ctx* ctx, Plan& plan, void* const* buffers, const mm_run_opts* o, bool timing,
                    mm_run_stats* st) {
  PlanRt* rt = static_cast<PlanRt*>(plan.rt);
  IpcChannel* ch = ctx->ipc;
  const int32_t G = ctx->G, W = ctx->world;
  const int32_t me = first_owned(ctx);
  const App& app = plan.app;
  const int32_t NS = kKinds * G;
  if ((int64_t)plan.ops.size() + kIpcOp0 > kIpcFlagSlots)
    MM_FAIL(MM_ENOTSUP, "ipc: %zu ops exceed the flag slots", plan.ops.size());
  std::vector<uint8_t> used(NS, 0);
  for (size_t i = 0; i < plan.ops.size(); ++i)
    if (plan.op_stream[i] >= 0 && sid_dev(ctx, plan.op_stream[i]) == me) used[plan.op_stream[i]] = 1;
  const int32_t root = me;   // compute stream of the owned device
  used[root] = 1;
  auto rank_of_sid = [&](int32_t sid) { return ctx->dev[sid_dev(ctx, sid)].rank; };
  std::vector<uint64_t*> wp;
  std::vector<int64_t> ws;
  std::vector<uint32_t> wl;
  auto flush_waits = [&](cudaStream_t s) -> mm_status {
    if (wp.empty()) return MM_OK;
    CU_OK(ipc_wait(ch->flags, wp.data(), ws.data(), wl.data(), (int32_t)wp.size(), s));
    wp.clear();
    ws.clear();
    wl.clear();
    return MM_OK;
  };
  auto fork_from_root = [&](cudaEvent_t* evs) -> mm_status {
    CU_OK(cudaEventRecord(evs[root], ctx->dev[me].stream));
    for (int32_t sid = 0; sid < NS; ++sid)
      if (used[sid] && sid != root) CU_OK(cudaStreamWaitEvent(sid_stream(ctx, sid), evs[root], 0));
    return MM_OK;
  };
  auto join_to_root = [&](cudaEvent_t* evs) -> mm_status {
    for (int32_t sid = 0; sid < NS; ++sid)
      if (used[sid] && sid != root) {
        CU_OK(cudaEventRecord(evs[sid], sid_stream(ctx, sid)));
        CU_OK(cudaStreamWaitEvent(ctx->dev[me].stream, evs[sid], 0));
      }
    return MM_OK;
  };
  CU_OK(set_dev(ctx, me));
  cudaStream_t rs = ctx->dev[me].stream;
  // run start: new epoch; every peer has finished the previous run
  CU_OK(ipc_bump_epoch(ch->flags, rs));
  for (int32_t q = 0; q < W; ++q)
    if (q != ctx->my_rank) {
      wp.push_back(ch->peer_flags[q]);
      ws.push_back(kIpcEnd);
      wl.push_back(1);
    }
  if (mm_status r = flush_waits(rs)) return r;
  if (mm_status r = fork_from_root(rt->bar_ev.data())) return r;
  for (size_t i = 0; i < plan.ops.size(); ++i) {
    const mm_op_rec& op = plan.ops[i];
    if (op.kind == MM_OPK_BARRIER) {
      if (mm_status r = join_to_root(rt->join_ev.data())) return r;
      CU_OK(ipc_signal(ch->flags, kIpcOp0 + (int64_t)i, rs));
      for (int32_t q = 0; q < W; ++q)
        if (q != ctx->my_rank) {
          wp.push_back(ch->peer_flags[q]);
          ws.push_back(kIpcOp0 + (int64_t)i);
          wl.push_back(0);
        }
      if (mm_status r = flush_waits(rs)) return r;
      if (mm_status r = fork_from_root(rt->bar_ev.data())) return r;
      continue;
    }
    const int32_t d = sid_dev(ctx, plan.op_stream[i]);
    if (d != me) continue;
    if (op.kind == MM_OPK_KERNEL && rt->batch_head[i] >= 0) continue;   // launched with its head
    cudaStream_t s = sid_stream(ctx, plan.op_stream[i]);
    auto add_waits = [&](size_t j) -> mm_status {
      for (auto& w : plan.waits[j]) {
        if (sid_dev(ctx, w.dev) == me) {
          CU_OK(cudaStreamWaitEvent(s, rt->ev[w.op], 0));
        } else {
          wp.push_back(ch->peer_flags[rank_of_sid(w.dev)]);
          ws.push_back(kIpcOp0 + w.op);
          wl.push_back(0);
        }
      }
      return MM_OK;
    };
    if (mm_status r = add_waits(i)) return r;
    if (op.kind == MM_OPK_KERNEL)
      for (int64_t m : rt->members[i])
        if (mm_status r = add_waits((size_t)m)) return r;
    if (mm_status r = flush_waits(s)) return r;
    if (op.kind == MM_OPK_KERNEL) {
      if (timing) CU_OK(rec_kev(rt->kev[2 * i], s));
      mm_status r = rt->members[i].empty() ? launch_task(ctx, app, plan.tasks[op.task], d, buffers, s)
                                           : launch_batch(ctx, plan, rt, (int64_t)i, d, buffers, s);
      if (r) return r;
      if (timing) CU_OK(rec_kev(rt->kev[2 * i + 1], s));
      for (int64_t m : rt->members[i]) {
        if (plan.needs_event[m]) CU_OK(cudaEventRecord(rt->ev[m], s));
        if (rt->remote_sig[m]) CU_OK(ipc_signal(ch->flags, kIpcOp0 + m, s));
      }
    } else if (op.kind == MM_OPK_XFER) {
      const int64_t eb = app.buffers[op.buffer].first;
      const size_t bytes = (size_t)((op.r.end - op.r.begin) * eb);
      char* dst = static_cast<char*>(buffers[(size_t)op.buffer * G + d]) + op.r.begin * eb;
      if (op.src < 0) {
        if (!o || !o->host || !o->host[op.buffer]) MM_FAIL(MM_EINVAL, "staged run: no host pointer for slot %d", op.buffer);
        CU_OK(cudaMemcpyAsync(dst, static_cast<const char*>(o->host[op.buffer]) + op.r.begin * eb, bytes,
                              cudaMemcpyHostToDevice, s));
        st->h2d_bytes += (int64_t)bytes;
      } else {
        const char* src = ctx->ipc_bufs[(size_t)op.buffer * W + ctx->dev[op.src].rank];
        if (!src) MM_FAIL(MM_EINVAL, "run: rank %d has no buffer %d", ctx->dev[op.src].rank, op.buffer);
        CU_OK(cudaMemcpyAsync(dst, src + op.r.begin * eb, bytes, cudaMemcpyDefault, s));
        st->xfer_bytes += (int64_t)bytes;
      }
    } else if (op.kind == MM_OPK_FLUSH) {
      const int64_t eb = app.buffers[op.buffer].first;
      const size_t bytes = (size_t)((op.r.end - op.r.begin) * eb);
      mm_status fs;
      char* host = static_cast<char*>(flush_target(ctx, plan, o, op.buffer,
                                                   (size_t)(app.buffers[op.buffer].second * eb), &fs));
      if (fs) return fs;
      const char* src = static_cast<const char*>(buffers[(size_t)op.buffer * G + d]) + op.r.begin * eb;
      CU_OK(cudaMemcpyAsync(host + op.r.begin * eb, src, bytes, cudaMemcpyDeviceToHost, s));
      st->d2h_bytes += (int64_t)bytes;
    }
    if (plan.needs_event[i]) CU_OK(cudaEventRecord(rt->ev[i], s));
    if (rt->remote_sig[i]) CU_OK(ipc_signal(ch->flags, kIpcOp0 + (int64_t)i, s));
  }
  // run end: every stream joined, then this rank's end flag
  if (mm_status r = join_to_root(rt->join_ev.data())) return r;
  CU_OK(ipc_signal(ch->flags, kIpcEnd, rs));
  return MM_OK;
}

// ------------------------------------------------------------------------
// Adaptive DP-Perf (P119: "the runtime profiles how fast each device
// processes a partition, and estimates the device busy time ... The
// information is kept and updated to determine which device will be the
// earliest executor for the next coming partition").  Tasks are decided in
// creation order with the frozen rule (R21) on live state: estimates are
// running means seeded by the warm-up profile (counted as its 3 chunks,
// P311) and updated with every completed chunk's event-timed duration;
// busy/ready times come from the device clock (events) and predictions.
// ------------------------------------------------------------------------
mm_status adaptive_event(mm_ctx* ctx, AdaptiveState* ad, size_t i, int32_t d) {
  if (ad->ev_end.size() <= i) {
    ad->ev_end.resize(i + 1, nullptr);
    ad->ev_beg.resize(i + 1, nullptr);
    ad->ev_dev.resize(i + 1, -1);
  }
  if (ad->ev_end[i] && ad->ev_dev[i] != ctx->dev[d].phys) {
    cudaEventDestroy(ad->ev_end[i]);
    cudaEventDestroy(ad->ev_beg[i]);
    ad->ev_end[i] = ad->ev_beg[i] = nullptr;
  }
  if (!ad->ev_end[i]) {
    CU_OK(cudaEventCreate(&ad->ev_end[i]));
    CU_OK(cudaEventCreate(&ad->ev_beg[i]));
    ad->ev_dev[i] = ctx->dev[d].phys;
  }
  return MM_OK;
}

mm_status adaptive_issue_op(mm_ctx* ctx, AdaptiveState* ad, size_t i, void* const* buffers,
                            const mm_run_opts* o, mm_run_stats* st) {
  Plan& ap = ad->ap;
  const App& app = ap.app;
  const int32_t G = ctx->G;
  const mm_op_rec& op = ap.ops[i];
  if (op.kind == MM_OPK_BARRIER) {
    // every stream waits for every other stream's last op
    const int32_t NS = kKinds * G;
    std::vector<cudaEvent_t> evs(NS, nullptr);
    for (int32_t sid = 0; sid < NS; ++sid) {
      CU_OK(set_dev(ctx, sid_dev(ctx, sid)));
      CU_OK(cudaEventCreateWithFlags(&evs[sid], cudaEventDisableTiming));
      CU_OK(cudaEventRecord(evs[sid], sid_stream(ctx, sid)));
    }
    for (int32_t sid = 0; sid < NS; ++sid) {
      CU_OK(set_dev(ctx, sid_dev(ctx, sid)));
      for (int32_t q = 0; q < NS; ++q)
        if (q != sid) CU_OK(cudaStreamWaitEvent(sid_stream(ctx, sid), evs[q], 0));
    }
    for (auto e : evs) cudaEventDestroy(e);
    return MM_OK;
  }
  const int32_t d = sid_dev(ctx, ap.op_stream[i]);
  cudaStream_t s = sid_stream(ctx, ap.op_stream[i]);
  CU_OK(set_dev(ctx, d));
  mm_status r = adaptive_event(ctx, ad, i, d);
  if (r) return r;
  for (auto& w : ap.waits[i]) CU_OK(cudaStreamWaitEvent(s, ad->ev_end[w.op], 0));
  if (op.kind == MM_OPK_KERNEL) {
    CU_OK(cudaEventRecord(ad->ev_beg[i], s));
    r = launch_task(ctx, app, ap.tasks[op.task], d, buffers, s);
    if (r) return r;
  } else if (op.kind == MM_OPK_XFER) {
    const int64_t eb = app.buffers[op.buffer].first;
    const size_t bytes = (size_t)((op.r.end - op.r.begin) * eb);
    char* dst = static_cast<char*>(buffers[(size_t)op.buffer * G + d]) + op.r.begin * eb;
    const char* src = static_cast<const char*>(buffers[(size_t)op.buffer * G + op.src]) + op.r.begin * eb;
    if (ctx->dev[op.src].phys == ctx->dev[d].phys)
      CU_OK(cudaMemcpyAsync(dst, src, bytes, cudaMemcpyDeviceToDevice, s));
    else
      CU_OK(cudaMemcpyPeerAsync(dst, ctx->dev[d].phys, src, ctx->dev[op.src].phys, bytes, s));
    st->xfer_bytes += (int64_t)bytes;
  } else if (op.kind == MM_OPK_FLUSH) {
    const int64_t eb = app.buffers[op.buffer].first;
    const size_t bytes = (size_t)((op.r.end - op.r.begin) * eb);
    mm_status fs;
    char* host = static_cast<char*>(flush_target(ctx, ap, o, op.buffer,
                                                 (size_t)(app.buffers[op.buffer].second * eb), &fs));
    if (fs) return fs;
    const char* src = static_cast<const char*>(buffers[(size_t)op.buffer * G + d]) + op.r.begin * eb;
    CU_OK(cudaMemcpyAsync(host + op.r.begin * eb, src, bytes, cudaMemcpyDeviceToHost, s));
    st->d2h_bytes += (int64_t)bytes;
  }
  CU_OK(cudaEventRecord(ad->ev_end[i], s));
  return MM_OK;
}

mm_status run_adaptive(mm_ctx* ctx, Plan& plan, PlanRt* rt, void* const* buffers, const mm_run_opts* o,
                       mm_run_stats* st) {
  const int32_t G = ctx->G;
  if (!rt->ad) {
    rt->ad = new AdaptiveState();
    Plan& ap = rt->ad->ap;
    ap.app = plan.app;
    ap.prof = plan.prof;
    ap.chunks_per_dev = plan.chunks_per_dev;
    ap.G = G;
    ap.cls = plan.cls;
    ap.strategy = MM_DP_PERF;
    ap.staged = 0;
    ap.tasks = plan.tasks;
    ap.task_dev.assign(plan.tasks.size(), 0);
    ap.task_fin.assign(plan.tasks.size(), 0);
    rt->ad->inc = inc_planner_create(ap.app, ap);
  }
  AdaptiveState* ad = rt->ad;
  Plan& ap = ad->ap;
  const App& app = ap.app;
  const int32_t maxq = o && o->max_inflight > 0 ? o->max_inflight : 4;
  const int32_t root = first_owned(ctx);
  inc_planner_begin(ad->inc);
  ad->decisions.clear();
  // fork + device time base
  CU_OK(set_dev(ctx, root));
  if (!ad->t0) CU_OK(cudaEventCreate(&ad->t0));
  CU_OK(cudaEventRecord(ad->t0, ctx->dev[root].stream));
  CU_OK(cudaEventRecord(rt->fork, ctx->dev[root].stream));
  for (int32_t sid = 0; sid < kKinds * G; ++sid)
    if (sid != root) {
      CU_OK(set_dev(ctx, sid_dev(ctx, sid)));
      CU_OK(cudaStreamWaitEvent(sid_stream(ctx, sid), rt->fork, 0));
    }
  const auto h0 = std::chrono::steady_clock::now();
  auto now_ns = [&]() -> uint64_t {
    return (uint64_t)std::chrono::duration_cast<std::chrono::nanoseconds>(std::chrono::steady_clock::now() - h0)
        .count();
  };
  const int64_t C = (int64_t)ap.chunks_per_dev * G;
  std::vector<int64_t> nominal(app.kernels.size());
  for (size_t k = 0; k < app.kernels.size(); ++k)
    nominal[k] = app.is_dag ? 1 : chunk_size(app.kernels[k].n, app.kernels[k].granule, C);
  std::vector<std::vector<double>> est(G, std::vector<double>(app.kernels.size(), 1.0));
  std::vector<std::vector<double>> cnt(G, std::vector<double>(app.kernels.size(), 3.0));  // warm-up = 3 chunks
  for (int32_t d = 0; d < G; ++d)
    for (size_t k = 0; k < app.kernels.size(); ++k) est[d][k] = (double)std::max<uint64_t>(1, ap.prof.chunk_est_ns[d][k]);
  std::vector<SegMap<int64_t>> lw(app.buffers.size());
  for (size_t b = 0; b < app.buffers.size(); ++b) lw[b].reset(app.buffers[b].second, -1);
  std::vector<uint64_t> fin(ap.tasks.size(), 0);  // predicted, then measured finish (ns, device time)
  std::vector<uint64_t> pred_fin(G, 0);
  std::vector<int64_t> last_task(G, -1);
  struct Out { int64_t t; int32_t d; size_t op; };
  std::deque<Out> outq;
  auto complete = [&](const Out& x) -> mm_status {
    float ms = 0.f, endms = 0.f;
    CU_OK(cudaEventElapsedTime(&ms, ad->ev_beg[x.op], ad->ev_end[x.op]));
    CU_OK(cudaEventElapsedTime(&endms, ad->t0, ad->ev_end[x.op]));
    const Task& t = ap.tasks[x.t];
    const int64_t items = app.is_dag ? 1 : std::max<int64_t>(1, t.e - t.b);
    const double meas = (double)ms * 1e6 * (double)nominal[t.kernel] / (double)items;
    double& e = est[x.d][t.kernel];
    double& c = cnt[x.d][t.kernel];
    e = (e * c + meas) / (c + 1.0);
    c += 1.0;
    fin[x.t] = (uint64_t)((double)endms * 1e6);
    if (last_task[x.d] == x.t) pred_fin[x.d] = fin[x.t];
    return MM_OK;
  };
  auto poll = [&](bool block_oldest) -> mm_status {
    if (block_oldest && !outq.empty()) CU_OK(cudaEventSynchronize(ad->ev_end[outq.front().op]));
    while (!outq.empty()) {
      cudaError_t q = cudaEventQuery(ad->ev_end[outq.front().op]);
      if (q == cudaErrorNotReady) break;
      CU_OK(q);
      mm_status r = complete(outq.front());
      if (r) return r;
      outq.pop_front();
    }
    return MM_OK;
  };
  int32_t last_inv = -1;
  for (size_t t = 0; t < ap.tasks.size(); ++t) {
    const Task& task = ap.tasks[t];
    if (!app.is_dag && task.inv != last_inv) {
      if (last_inv >= 0) {  // R11: a sync point after the previous invocation aligns the devices
        const int32_t kprev = ap.tasks[t - 1].kernel;
        auto it = app.sync.find(kprev);
        if (it != app.sync.end() && it->second != MM_SYNC_NONE) {
          const uint64_t m = *std::max_element(pred_fin.begin(), pred_fin.end());
          std::fill(pred_fin.begin(), pred_fin.end(), m);
        }
      }
      last_inv = task.inv;
    }
    mm_status r = poll(false);
    if (r) return r;
    while ((int64_t)outq.size() >= (int64_t)maxq * G) {
      r = poll(true);
      if (r) return r;
    }
    // producers of what the task reads (RAW), with bytes
    std::map<int64_t, int64_t> preds;
    for (auto& a : task.acc) {
      if (!(a.mode & MM_READ)) continue;
      const int64_t eb = app.buffers[a.buffer].first;
      lw[a.buffer].visit(a.lo, a.hi, [&](int64_t lo, int64_t hi, const int64_t& w) {
        if (w >= 0) preds[w] += (hi - lo) * eb;
      });
    }
    mm_decision dec;
    std::memset(&dec, 0, sizeof(dec));
    dec.task = (int64_t)t;
    dec.kernel = task.kernel;
    dec.now_ns = now_ns();
    const int64_t items = app.is_dag ? 1 : std::max<int64_t>(1, task.e - task.b);
    int32_t best = -1;
    for (int32_t d = 0; d < G; ++d) {
      uint64_t ready = 0, xfer = 0;   // R21/R32 as in the frozen schedule; the pulls go into cost_ns
      for (auto& p : preds) {
        ready = std::max(ready, fin[p.first]);
        if (ap.task_dev[p.first] != d) {
          const uint64_t link = std::max<uint64_t>(1, ap.prof.link_Bps[d]);
          xfer += ap.prof.link_lat_ns[d] + (uint64_t)(((unsigned __int128)p.second * 1000000000ull + link - 1) / link);
        }
      }
      const uint64_t busy = std::max(dec.now_ns, pred_fin[d]);
      const uint64_t cost = xfer + (uint64_t)(est[d][task.kernel] * (double)items / (double)nominal[task.kernel]);
      dec.busy_ns[d] = busy;
      dec.ready_ns[d] = ready;
      dec.cost_ns[d] = cost;
      dec.eft_ns[d] = std::max(busy, ready) + cost;
      if (best < 0 || dec.eft_ns[d] < dec.eft_ns[best]) best = d;
    }
    dec.chosen = best;
    ad->decisions.push_back(dec);
    ap.task_dev[t] = best;
    fin[t] = dec.eft_ns[best];
    pred_fin[best] = fin[t];
    last_task[best] = (int64_t)t;
    for (auto& a : task.acc)
      if (a.mode & MM_WRITE) lw[a.buffer].assign(a.core_lo, a.core_hi, (int64_t)t);
    const size_t n0 = ap.ops.size();
    r = inc_planner_step(ad->inc, (int64_t)t);
    if (r) return r;
    for (size_t i = n0; i < ap.ops.size(); ++i) {
      r = adaptive_issue_op(ctx, ad, i, buffers, o, st);
      if (r) return r;
      if (ap.ops[i].kind == MM_OPK_KERNEL) outq.push_back(Out{(int64_t)t, best, i});
    }
  }
  const size_t n0 = ap.ops.size();
  mm_status r = inc_planner_end(ad->inc);
  if (r) return r;
  for (size_t i = n0; i < ap.ops.size(); ++i) {
    r = adaptive_issue_op(ctx, ad, i, buffers, o, st);
    if (r) return r;
  }
  // join
  for (int32_t sid = 0; sid < kKinds * G; ++sid)
    if (sid != root) {
      CU_OK(set_dev(ctx, sid_dev(ctx, sid)));
      CU_OK(cudaEventRecord(rt->join_ev[sid], sid_stream(ctx, sid)));
      CU_OK(set_dev(ctx, root));
      CU_OK(cudaStreamWaitEvent(ctx->dev[root].stream, rt->join_ev[sid], 0));
    }
  CU_OK(set_dev(ctx, root));
  CU_OK(cudaStreamSynchronize(ctx->dev[root].stream));
  while (!outq.empty()) {
    r = complete(outq.front());
    if (r) return r;
    outq.pop_front();
  }
  for (size_t i = 0; i < ap.ops.size(); ++i) {
    const mm_op_rec& op = ap.ops[i];
    if (op.kind != MM_OPK_KERNEL) continue;
    float ms = 0.f;
    CU_OK(cudaEventElapsedTime(&ms, ad->ev_beg[i], ad->ev_end[i]));
    st->kernel_ms[op.device][op.kernel] += ms;
    st->kernel_launches[op.device][op.kernel]++;
  }
  return MM_OK;
}

}  // namespace

// ===========================================================================
// C ABI: runtime
// ===========================================================================
extern "C" {

mm_status mm_nccl_unique_id(void* out128) {
  if (!out128) MM_FAIL(MM_EINVAL, "null out");
  mm_ctx* ctx = nullptr;
  if (!nccl().ok) MM_FAIL(MM_ENCCL, "libnccl.so.2 could not be loaded");
  ncclUniqueId id;
  NCCL_OK(nccl().GetUniqueId(&id));
  static_assert(sizeof(id) == 128, "ncclUniqueId size");
  std::memcpy(out128, &id, sizeof(id));
  return MM_OK;
}

mm_status mm_rendezvous_id(void* out128) {
  if (!out128) MM_FAIL(MM_EINVAL, "null out");
  std::random_device rd;
  uint32_t* o = static_cast<uint32_t*>(out128);
  for (int i = 0; i < 32; ++i) o[i] = rd();
  return MM_OK;
}

mm_status mm_ctx_create(const mm_device_spec* devs, int32_t G, int32_t my_rank, int32_t world,
                        const void* nccl_id, mm_ctx** out) {
  if (!devs || !out || G < 1 || G > MM_MAX_DEV || world < 1 || my_rank < 0 || my_rank >= world)
    MM_FAIL(MM_EINVAL, "ctx_create: bad arguments (G=%d rank=%d world=%d)", G, my_rank, world);
  mm_ctx* ctx = nullptr;
  try {
    ctx = new mm_ctx();
  } catch (...) {
    MM_FAIL(MM_ENOMEM, "ctx alloc");
  }
  std::unique_ptr<mm_ctx, void (*)(mm_ctx*)> guard(ctx, [](mm_ctx* c) { mm_ctx_destroy(c); });
  ctx->G = G;
  ctx->my_rank = my_rank;
  ctx->world = world;
  ctx->dev.resize(G);
  int ndev = 0;
  CU_OK(cudaGetDeviceCount(&ndev));
  int owned = 0;
  for (int32_t d = 0; d < G; ++d) {
    DevRt& r = ctx->dev[d];
    r.phys = devs[d].cuda_device;
    r.budget = devs[d].sm_budget;
    r.rank = devs[d].rank;
    r.mine = (r.rank == my_rank);
    if (r.rank < 0 || r.rank >= world) MM_FAIL(MM_EINVAL, "device %d: rank %d", d, r.rank);
    if (!r.mine) continue;
    owned++;
    if (r.phys < 0 || r.phys >= ndev) MM_FAIL(MM_EINVAL, "device %d: cuda ordinal %d of %d", d, r.phys, ndev);
    CU_OK(cudaSetDevice(r.phys));
    int sms = 0;
    CU_OK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, r.phys));
    r.sms = sms;
  }
  if (world > 1 && owned != 1) MM_FAIL(MM_EINVAL, "multi-process ctx: rank %d owns %d devices (need 1)", my_rank, owned);
  if (owned == 0) MM_FAIL(MM_EINVAL, "rank %d owns no device", my_rank);
  // SM budgets (HET mode): per physical GPU, split its SMs into green
  // contexts — one group of >= budget SMs per budgeted logical device, the
  // remainder for the unbudgeted one(s).
  for (int32_t d = 0; d < G; ++d) {
    DevRt& r = ctx->dev[d];
    if (!r.mine) continue;
    bool any_budget = false;
    for (int32_t q = 0; q < G; ++q)
      if (ctx->dev[q].mine && ctx->dev[q].phys == r.phys && ctx->dev[q].budget > 0) any_budget = true;
    if (!any_budget) {
      CU_OK(cudaSetDevice(r.phys));
      CU_OK(cudaStreamCreateWithFlags(&r.stream, cudaStreamNonBlocking));
      CU_OK(cudaStreamCreateWithFlags(&r.h2d, cudaStreamNonBlocking));
      CU_OK(cudaStreamCreateWithFlags(&r.d2h, cudaStreamNonBlocking));
      {  // lane 1 carries the critical path: highest stream priority
         // (MM_LANE1_PRIO=0: default priority, development knob)
        int lo = 0, hi = 0;
        CU_OK(cudaDeviceGetStreamPriorityRange(&lo, &hi));
        static const int p1 = getenv("MM_LANE1_PRIO") ? atoi(getenv("MM_LANE1_PRIO")) : 1;
        CU_OK(cudaStreamCreateWithPriority(&r.lane1, cudaStreamNonBlocking, p1 ? hi : lo));
      }
      continue;
    }
    if (r.gctx) continue;
    // build all green contexts of this physical GPU at once
    Drv& D = drv();
    if (!D.ok) MM_FAIL(MM_ENOTSUP, "green contexts: driver entry points unavailable");
    CU_OK(cudaSetDevice(r.phys));
    CU_OK(cudaFree(nullptr));  // make sure the primary context exists
    DRV_OK(D.Init(0));
    CUdevice cudev;
    DRV_OK(D.DeviceGet(&cudev, r.phys));
    CUdevResource all;
    DRV_OK(D.DeviceGetDevResource(cudev, &all, CU_DEV_RESOURCE_TYPE_SM));
    CUdevResource rest = all;
    // devices with equal budgets are split off in ONE call (nbGroups = their
    // count): the driver rejects splitting a remainder again on B200
    std::map<int32_t, std::vector<int32_t>> by_budget;
    for (int32_t q = 0; q < G; ++q) {
      DevRt& rq = ctx->dev[q];
      if (rq.mine && rq.phys == r.phys && rq.budget > 0) by_budget[rq.budget].push_back(q);
    }
    std::map<int32_t, CUdevResource> group_of;
    for (auto& kv : by_budget) {
      std::vector<CUdevResource> grps(kv.second.size());
      CUdevResource remaining;
      unsigned n = (unsigned)kv.second.size();
      DRV_OK(D.DevSmResourceSplitByCount(grps.data(), &n, &rest, &remaining, 0, (unsigned)kv.first));
      if (n < kv.second.size())
        MM_FAIL(MM_ECUDA, "SM split: %u of %zu groups of %d SMs", n, kv.second.size(), kv.first);
      for (size_t i = 0; i < kv.second.size(); ++i) group_of[kv.second[i]] = grps[i];
      rest = remaining;
    }
    for (int32_t q = 0; q < G; ++q) {
      DevRt& rq = ctx->dev[q];
      if (!rq.mine || rq.phys != r.phys || rq.budget <= 0) continue;
      CUdevResource grp = group_of[q];
      CUdevResourceDesc desc;
      DRV_OK(D.DevResourceGenerateDesc(&desc, &grp, 1));
      DRV_OK(D.GreenCtxCreate(&rq.gctx, desc, cudev, CU_GREEN_CTX_DEFAULT_STREAM));
      DRV_OK(D.CtxFromGreenCtx(&rq.gcu, rq.gctx));
      CUstream cs;
      DRV_OK(D.GreenCtxStreamCreate(&cs, rq.gctx, CU_STREAM_NON_BLOCKING, 0));
      rq.stream = (cudaStream_t)cs;
      DRV_OK(D.GreenCtxStreamCreate(&cs, rq.gctx, CU_STREAM_NON_BLOCKING, 0));
      rq.h2d = (cudaStream_t)cs;
      DRV_OK(D.GreenCtxStreamCreate(&cs, rq.gctx, CU_STREAM_NON_BLOCKING, 0));
      rq.d2h = (cudaStream_t)cs;
      DRV_OK(D.GreenCtxStreamCreate(&cs, rq.gctx, CU_STREAM_NON_BLOCKING, -1));
      rq.lane1 = (cudaStream_t)cs;
      rq.sms = (int32_t)grp.sm.smCount;
    }
    for (int32_t q = 0; q < G; ++q) {
      DevRt& rq = ctx->dev[q];
      if (!rq.mine || rq.phys != r.phys || rq.budget > 0) continue;
      CUdevResourceDesc desc;
      DRV_OK(D.DevResourceGenerateDesc(&desc, &rest, 1));
      DRV_OK(D.GreenCtxCreate(&rq.gctx, desc, cudev, CU_GREEN_CTX_DEFAULT_STREAM));
      DRV_OK(D.CtxFromGreenCtx(&rq.gcu, rq.gctx));
      CUstream cs;
      DRV_OK(D.GreenCtxStreamCreate(&cs, rq.gctx, CU_STREAM_NON_BLOCKING, 0));
      rq.stream = (cudaStream_t)cs;
      DRV_OK(D.GreenCtxStreamCreate(&cs, rq.gctx, CU_STREAM_NON_BLOCKING, 0));
      rq.h2d = (cudaStream_t)cs;
      DRV_OK(D.GreenCtxStreamCreate(&cs, rq.gctx, CU_STREAM_NON_BLOCKING, 0));
      rq.d2h = (cudaStream_t)cs;
      DRV_OK(D.GreenCtxStreamCreate(&cs, rq.gctx, CU_STREAM_NON_BLOCKING, 0));
      rq.lane1 = (cudaStream_t)cs;
      rq.sms = (int32_t)rest.sm.smCount;
    }
  }
  const char* tr = getenv("MM_TRANSPORT");
  if (world > 1 && !(tr && std::strcmp(tr, "nccl") == 0)) {
    // IPC transport (default): shared-memory rendezvous + CUDA IPC pulls/flags
    if (!nccl_id) MM_FAIL(MM_EINVAL, "multi-process ctx needs a 128-byte rendezvous id");
    const int32_t me = first_owned(ctx);
    CU_OK(cudaSetDevice(ctx->dev[me].phys));
    ctx->ipc = new (std::nothrow) IpcChannel();
    if (!ctx->ipc) MM_FAIL(MM_ENOMEM, "ipc channel");
    mm_status st = ipc_open(ctx->ipc, nccl_id, my_rank, world);
    if (st) return st;
  } else if (world > 1) {
    if (!nccl_id) MM_FAIL(MM_EINVAL, "multi-process ctx needs an NCCL unique id");
    if (!nccl().ok) MM_FAIL(MM_ENCCL, "libnccl.so.2 could not be loaded");
    ncclUniqueId id;
    std::memcpy(&id, nccl_id, sizeof(id));
    const int32_t me = first_owned(ctx);
    CU_OK(cudaSetDevice(ctx->dev[me].phys));
    NCCL_OK(nccl().CommInitRank(&ctx->comm, world, id, my_rank));
    CU_OK(cudaMalloc(&ctx->bar_buf, sizeof(float)));
    CU_OK(cudaMemset(ctx->bar_buf, 0, sizeof(float)));
  } else {
    // in-process multi-GPU: enable peer access where possible
    for (int32_t a = 0; a < G; ++a)
      for (int32_t b = 0; b < G; ++b) {
        const int pa = ctx->dev[a].phys, pb = ctx->dev[b].phys;
        if (pa == pb) continue;
        int can = 0;
        cudaDeviceCanAccessPeer(&can, pa, pb);
        if (can) {
          cudaSetDevice(pa);
          cudaError_t e = cudaDeviceEnablePeerAccess(pb, 0);
          if (e == cudaErrorPeerAccessAlreadyEnabled) cudaGetLastError();
        }
      }
  }
  *out = guard.release();
  return MM_OK;
}

void mm_ctx_destroy(mm_ctx* ctx) {
  if (!ctx) return;
  if (ctx->ipc && ctx->ipc->shm) {   // collective: no rank unmaps while a peer may still pull from it
    const int32_t me = first_owned(ctx);
    if (me >= 0) {
      set_dev(ctx, me);
      cudaDeviceSynchronize();
    }
    ipc_barrier(ctx->ipc);
  }
  for (auto& r : ctx->dev) {
    if (!r.mine) continue;
    cudaSetDevice(r.phys);
    for (cudaStream_t st : {r.stream, r.h2d, r.d2h, r.lane1}) {
      if (!st) continue;
      if (r.gctx) drv().StreamDestroy((CUstream)st);
      else cudaStreamDestroy(st);
    }
    if (r.scr.ptr) cudaFree(r.scr.ptr);
    const size_t d = (size_t)(&r - ctx->dev.data());
    if (d < ctx->ext_ev.size() && ctx->ext_ev[d]) cudaEventDestroy(ctx->ext_ev[d]);
    if (d < ctx->lib_ev.size() && ctx->lib_ev[d]) cudaEventDestroy(ctx->lib_ev[d]);
    if (r.gctx) drv().GreenCtxDestroy(r.gctx);
  }
  if (ctx->ipc) {
    ipc_close(ctx->ipc);
    delete ctx->ipc;
  }
  if (ctx->comm) nccl().CommDestroy(ctx->comm);
  if (ctx->bar_buf) cudaFree(ctx->bar_buf);
  for (auto p : ctx->flush_scratch)
    if (p) cudaFreeHost(p);
  delete ctx;
}

mm_status mm_ctx_stream(mm_ctx* ctx, int32_t d, void** stream) {
  if (!ctx || !stream || d < 0 || d >= ctx->G) MM_FAIL(MM_EINVAL, "ctx_stream: bad arguments");
  if (!ctx->dev[d].mine) MM_FAIL(MM_EINVAL, "ctx_stream: device %d not owned by this rank", d);
  *stream = (void*)ctx->dev[d].stream;
  return MM_OK;
}

mm_status mm_ctx_sm_count(mm_ctx* ctx, int32_t d, int32_t* sms) {
  if (!ctx || !sms || d < 0 || d >= ctx->G) MM_FAIL(MM_EINVAL, "ctx_sm_count: bad arguments");
  *sms = ctx->dev[d].sms;
  return MM_OK;
}

mm_status mm_ctx_set_stream(mm_ctx* ctx, int32_t d, void* stream) {
  if (!ctx || d < 0 || d >= ctx->G) MM_FAIL(MM_EINVAL, "ctx_set_stream: bad arguments");
  if (!ctx->dev[d].mine) MM_FAIL(MM_EINVAL, "ctx_set_stream: device %d not owned by this rank", d);
  if (ctx->poisoned) MM_FAIL(MM_ESTATE, "ctx poisoned by an earlier CUDA error");
  if (ctx->ext.size() != (size_t)ctx->G) {
    ctx->ext.assign((size_t)ctx->G, nullptr);
    ctx->ext_ev.assign((size_t)ctx->G, nullptr);
    ctx->lib_ev.assign((size_t)ctx->G, nullptr);
  }
  ctx->ext[d] = static_cast<cudaStream_t>(stream);
  return MM_OK;
}

mm_status mm_buffer_register(mm_ctx* ctx, int32_t elem_bytes, int64_t n_elems, void* const* dev_ptrs,
                             int32_t* buf_id) {
  if (!ctx || !dev_ptrs || !buf_id) MM_FAIL(MM_EINVAL, "buffer_register: null argument");
  if (!(elem_bytes == 1 || elem_bytes == 2 || elem_bytes == 4 || elem_bytes == 8) || n_elems < 0)
    MM_FAIL(MM_EINVAL, "buffer_register: elem_bytes %d n %lld", elem_bytes, (long long)n_elems);
  if ((int32_t)ctx->reg.size() >= MM_MAX_BUF) MM_FAIL(MM_EINVAL, "buffer_register: too many buffers");
  for (int32_t d = 0; d < ctx->G; ++d)
    if (ctx->dev[d].mine && n_elems > 0 && !dev_ptrs[d])
      MM_FAIL(MM_EINVAL, "buffer_register: no pointer for owned device %d", d);
  try {
    ctx->reg.emplace_back(dev_ptrs, dev_ptrs + ctx->G);
    ctx->reg_shape.push_back({elem_bytes, n_elems});
  } catch (...) {
    MM_FAIL(MM_ENOMEM, "buffer_register: out of host memory");
  }
  *buf_id = (int32_t)ctx->reg.size() - 1;
  return MM_OK;
}

mm_status mm_fill_uniform(mm_ctx* ctx, int32_t d, float* dst, int64_t n, uint64_t seed, int32_t array_id,
                          int64_t start, float lo, float hi) {
  if (!ctx || d < 0 || d >= ctx->G || !ctx->dev[d].mine || (n > 0 && !dst) || n < 0)
    MM_FAIL(MM_EINVAL, "fill_uniform: bad arguments");
  if (ctx->poisoned) MM_FAIL(MM_ESTATE, "ctx poisoned by an earlier CUDA error");
  CU_OK(set_dev(ctx, d));
  CU_OK(fill_uniform(dst, n, seed, array_id, start, lo, hi, ctx->dev[d].stream));
  CU_OK(cudaStreamSynchronize(ctx->dev[d].stream));
  return MM_OK;
}

mm_status mm_fill_integers(mm_ctx* ctx, int32_t d, float* dst, int64_t n, uint64_t seed, int32_t array_id,
                           int64_t start, int32_t lo, int32_t hi) {
  if (!ctx || d < 0 || d >= ctx->G || !ctx->dev[d].mine || (n > 0 && !dst) || n < 0 || hi < lo)
    MM_FAIL(MM_EINVAL, "fill_integers: bad arguments");
  if (ctx->poisoned) MM_FAIL(MM_ESTATE, "ctx poisoned by an earlier CUDA error");
  CU_OK(set_dev(ctx, d));
  CU_OK(fill_integers(dst, n, seed, array_id, start, lo, hi, ctx->dev[d].stream));
  CU_OK(cudaStreamSynchronize(ctx->dev[d].stream));
  return MM_OK;
}

mm_status mm_fill_spd_tiles(mm_ctx* ctx, int32_t d, float* dst, int64_t n, int64_t b, uint64_t seed,
                            int32_t array_id) {
  if (!ctx || d < 0 || d >= ctx->G || !ctx->dev[d].mine || !dst || n <= 0 || b <= 0 || n % b)
    MM_FAIL(MM_EINVAL, "fill_spd_tiles: bad arguments");
  if (ctx->poisoned) MM_FAIL(MM_ESTATE, "ctx poisoned by an earlier CUDA error");
  CU_OK(set_dev(ctx, d));
  CU_OK(fill_spd_tiles(dst, n, b, seed, array_id, ctx->dev[d].stream));
  CU_OK(cudaStreamSynchronize(ctx->dev[d].stream));
  return MM_OK;
}

namespace {
// buffers == NULL: the registered buffers (slot i = i-th registration), which
// must match the plan's buffer shapes
mm_status resolve_buffers(mm_ctx* ctx, const Plan& plan, void* const*& buffers, std::vector<void*>& tmp) {
  if (buffers) return MM_OK;
  const size_t nb = plan.app.buffers.size();
  if (ctx->reg.size() < nb) MM_FAIL(MM_EINVAL, "run: %zu buffers registered, the app has %zu", ctx->reg.size(), nb);
  tmp.assign(nb * (size_t)ctx->G, nullptr);
  for (size_t i = 0; i < nb; ++i) {
    if (ctx->reg_shape[i] != plan.app.buffers[i])
      MM_FAIL(MM_EINVAL, "run: registered buffer %zu (%d B x %lld) differs from app slot %zu", i,
              ctx->reg_shape[i].first, (long long)ctx->reg_shape[i].second, i);
    for (int32_t d = 0; d < ctx->G; ++d) tmp[i * (size_t)ctx->G + d] = ctx->reg[i][(size_t)d];
  }
  buffers = tmp.data();
  return MM_OK;
}

// mm_ctx_set_stream: order device d's streams after the work already on the
// caller's stream (before), or the caller's stream after the run (after).
// An event must be recorded in its stream's context: the caller's stream
// lives in the primary context of the GPU, the library's streams of an
// SM-budgeted device in its green context; waits may cross contexts.
mm_status join_external(mm_ctx* ctx, bool before) {
  for (int32_t d = 0; d < (int32_t)ctx->ext.size(); ++d) {
    if (!ctx->ext[d] || !ctx->dev[d].mine) continue;
    DevRt& r = ctx->dev[d];
    if (before) {
      CU_OK(cudaSetDevice(r.phys));   // primary context of the caller's stream
      if (!ctx->ext_ev[d]) CU_OK(cudaEventCreateWithFlags(&ctx->ext_ev[d], cudaEventDisableTiming));
      CU_OK(cudaEventRecord(ctx->ext_ev[d], ctx->ext[d]));
      CU_OK(set_dev(ctx, d));
      for (cudaStream_t st : {r.stream, r.h2d, r.d2h, r.lane1})
        if (st) CU_OK(cudaStreamWaitEvent(st, ctx->ext_ev[d], 0));
    } else {
      CU_OK(set_dev(ctx, d));
      if (!ctx->lib_ev[d]) CU_OK(cudaEventCreateWithFlags(&ctx->lib_ev[d], cudaEventDisableTiming));
      CU_OK(cudaEventRecord(ctx->lib_ev[d], r.stream));
      CU_OK(cudaSetDevice(r.phys));
      CU_OK(cudaStreamWaitEvent(ctx->ext[d], ctx->lib_ev[d], 0));
    }
  }
  return MM_OK;
}
}  // namespace

mm_status mm_run(mm_ctx* ctx, mm_plan* plan_h, void* const* buffers, const mm_run_opts* o, mm_run_stats* st) {
  if (!ctx || !plan_h) MM_FAIL(MM_EINVAL, "run: null argument");
  std::vector<void*> reg_bufs;
  if (mm_status rb = resolve_buffers(ctx, plan_h->p, buffers, reg_bufs)) return rb;
  if (ctx->poisoned) MM_FAIL(MM_ESTATE, "ctx poisoned by an earlier CUDA error");
  Plan& plan = plan_h->p;
  if (plan.G != ctx->G) MM_FAIL(MM_EINVAL, "run: plan has G=%d, ctx has G=%d", plan.G, ctx->G);
  mm_run_stats local{};
  mm_run_stats* S = st ? st : &local;
  *S = mm_run_stats{};
  const bool timing = o && o->time_kernels;
  const bool graph = o && o->use_graph && (ctx->world == 1 || ctx->ipc);
  const int32_t reps = (o && o->repeat > 1) ? o->repeat : 1;
  if (o && o->repeat < 0) MM_FAIL(MM_EINVAL, "run: repeat %d < 0", o->repeat);
  mm_status r = ensure_rt(ctx, plan, timing);
  if (r) return r;
  if ((r = join_external(ctx, true))) return r;
  PlanRt* rt = static_cast<PlanRt*>(plan.rt);
  for (auto& dv : ctx->dev) dv.scr.epoch++;   // operand-split caches are per run
  const int32_t root = first_owned(ctx);
  cudaStream_t rs = ctx->dev[root].stream;
  const size_t nbuf = plan.app.buffers.size() * (size_t)ctx->G;
  auto t0 = std::chrono::steady_clock::now();
  if (o && o->adaptive) {
    if (plan.strategy != MM_DP_PERF) MM_FAIL(MM_EINVAL, "run: adaptive needs a DP-Perf plan");
    if (ctx->world != 1) MM_FAIL(MM_ENOTSUP, "run: adaptive DP-Perf is in-process only");
    CU_OK(set_dev(ctx, root));
    CU_OK(cudaEventRecord(rt->t_start, rs));
    const int64_t l0 = g_kernel_launches.load();
    r = run_adaptive(ctx, plan, rt, buffers, o, S);
    S->n_launches = g_kernel_launches.load() - l0;
    if (r) return r;
    CU_OK(set_dev(ctx, root));
    CU_OK(cudaEventRecord(rt->t_stop, rs));
    CU_OK(cudaEventSynchronize(rt->t_stop));
    auto t1a = std::chrono::steady_clock::now();
    S->wall_ms = std::chrono::duration<double, std::milli>(t1a - t0).count();
    float msa = 0.f;
    CU_OK(cudaEventElapsedTime(&msa, rt->t_start, rt->t_stop));
    S->device_ms = msa;
    rt->last_adaptive = true;
    return MM_OK;
  }
  rt->last_adaptive = false;
  if (ctx->ipc) {   // every rank's buffers, mapped into this process (host barrier)
    std::vector<void*> mine(plan.app.buffers.size(), nullptr);
    for (size_t b = 0; b < mine.size(); ++b) mine[b] = buffers[b * (size_t)ctx->G + root];
    if ((r = ipc_exchange_buffers(ctx->ipc, mine, ctx->ipc_bufs))) return r;
  }
  if (graph) {
    // Everything the captured graph bakes in is part of its key: the app
    // buffers, each device's library scratch (operand splits, split-K
    // partials, Cholesky panels and the TMA maps built on them), the host
    // pointers of staged/flush copies and the pinned flush scratch.  Flush
    // scratch is reserved before the key is formed (never inside a capture).
    for (size_t i = 0; i < plan.ops.size(); ++i) {
      const mm_op_rec& op = plan.ops[i];
      if (op.kind != MM_OPK_FLUSH || !ctx->dev[op.device].mine) continue;
      mm_status fs;
      const int64_t eb = plan.app.buffers[op.buffer].first;
      flush_target(ctx, plan, o, op.buffer, (size_t)(plan.app.buffers[op.buffer].second * eb), &fs);
      if (fs) return fs;
    }
    std::vector<void*> key(buffers, buffers + nbuf);
    for (auto& dv : ctx->dev) {
      key.push_back(dv.scr.ptr);
      key.push_back(reinterpret_cast<void*>(dv.scr.bytes));
    }
    for (size_t b = 0; b < plan.app.buffers.size(); ++b)
      key.push_back(o && o->host ? o->host[b] : nullptr);
    for (void* p : ctx->flush_scratch) key.push_back(p);
    for (char* p : ctx->ipc_bufs) key.push_back(p);
    key.push_back(reinterpret_cast<void*>((intptr_t)reps));
    key.push_back(reinterpret_cast<void*>((intptr_t)(timing ? 1 : 0)));
    if (!rt->gexec || key != rt->graph_bufs) {
      if (rt->gexec) cudaGraphExecDestroy(rt->gexec);
      if (rt->graph) cudaGraphDestroy(rt->graph);
      rt->gexec = nullptr;
      rt->graph = nullptr;
      CU_OK(set_dev(ctx, root));
      CU_OK(cudaStreamBeginCapture(rs, cudaStreamCaptureModeThreadLocal));
      mm_run_stats cap{};
      const int64_t l0 = g_kernel_launches.load();
      for (int32_t rep = 0; rep < reps && !r; ++rep)   // kernel timing: event record nodes
        r = ctx->ipc ? issue_ipc(ctx, plan, buffers, o, timing, &cap) : issue_local(ctx, plan, buffers, o, timing, &cap);
      const int64_t captured = g_kernel_launches.load() - l0;
      g_kernel_launches.fetch_sub(captured, std::memory_order_relaxed);   // counted per replay
      cudaGraph_t g = nullptr;
      cudaError_t ce = cudaStreamEndCapture(rs, &g);
      if (r) {
        if (g) cudaGraphDestroy(g);
        return r;
      }
      CU_OK(ce);
      rt->graph = g;
      CU_OK(cudaGraphInstantiate(&rt->gexec, g, 0));
      rt->graph_bufs = key;
      rt->graph_launches = captured;
      rt->graph_xfer = cap.xfer_bytes;
      rt->graph_h2d = cap.h2d_bytes;
      rt->graph_d2h = cap.d2h_bytes;
    }
    t0 = std::chrono::steady_clock::now();
    CU_OK(set_dev(ctx, root));
    // enqueue-only runs report no device time: no start/stop events around them
    const bool ev = !(o && o->no_wait && !timing);
    if (ev) CU_OK(cudaEventRecord(rt->t_start, rs));
    CU_OK(cudaGraphLaunch(rt->gexec, rs));
    if (ev) CU_OK(cudaEventRecord(rt->t_stop, rs));
    S->n_launches = rt->graph_launches;
    S->xfer_bytes = rt->graph_xfer;
    S->h2d_bytes = rt->graph_h2d;
    S->d2h_bytes = rt->graph_d2h;
    g_kernel_launches.fetch_add(rt->graph_launches, std::memory_order_relaxed);
  } else {
    CU_OK(set_dev(ctx, root));
    const bool ev = !(o && o->no_wait && !timing);
    if (ev) CU_OK(cudaEventRecord(rt->t_start, rs));
    const int64_t l0 = g_kernel_launches.load();
    for (int32_t rep = 0; rep < reps && !r; ++rep) {
      if (ctx->world == 1) r = issue_local(ctx, plan, buffers, o, timing, S);
      else if (ctx->ipc) r = issue_ipc(ctx, plan, buffers, o, timing, S);
      else r = issue_dist(ctx, plan, buffers, o, timing, S);
    }
    S->n_launches = g_kernel_launches.load() - l0;
    if (r) return r;
    CU_OK(set_dev(ctx, root));
    if (ev) CU_OK(cudaEventRecord(rt->t_stop, rs));
  }
  if (o && o->no_wait && !timing) {
    // enqueue only: every library stream of this run is joined into the root
    // stream, so the next run (or a caller stream set with mm_ctx_set_stream,
    // or a synchronisation of mm_ctx_stream(root)) is ordered after it
    if ((r = join_external(ctx, false))) return r;
    S->wall_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    S->device_ms = -1.0;
    for (size_t i = 0; i < plan.ops.size(); ++i)
      if (plan.ops[i].kind == MM_OPK_KERNEL && ctx->dev[plan.ops[i].device].mine)
        S->kernel_launches[plan.ops[i].device][plan.ops[i].kernel] += reps;
    return MM_OK;
  }
  CU_OK(cudaEventSynchronize(rt->t_stop));
  auto t1 = std::chrono::steady_clock::now();
  if ((r = join_external(ctx, false))) return r;
  S->wall_ms = std::chrono::duration<double, std::milli>(t1 - t0).count();
  float ms = 0.f;
  CU_OK(cudaEventElapsedTime(&ms, rt->t_start, rt->t_stop));
  S->device_ms = ms;
  // MM_TRACE=<file>: per kernel launch (batch heads) of a timed run, append
  // "kernel,ip0,ip1,ip2,device,tasks,start_ms,end_ms" relative to the run start
  static const char* trace_path = getenv("MM_TRACE");
  FILE* trace = (timing && trace_path) ? fopen(trace_path, "a") : nullptr;
  for (size_t i = 0; i < plan.ops.size(); ++i) {
    const mm_op_rec& op = plan.ops[i];
    if (op.kind != MM_OPK_KERNEL || !ctx->dev[op.device].mine) continue;
    if (trace && rt->kev[2 * i] && rt->batch_head[i] < 0) {
      float a = 0.f, z = 0.f;
      if (cudaEventElapsedTime(&a, rt->t_start, rt->kev[2 * i]) == cudaSuccess &&
          cudaEventElapsedTime(&z, rt->t_start, rt->kev[2 * i + 1]) == cudaSuccess) {
        const Task& t = plan.tasks[op.task];
        fprintf(trace, "%s,%lld,%lld,%lld,%d,%zu,%.4f,%.4f\n", plan.app.kernels[op.kernel].name.c_str(),
                (long long)t.ip[0], (long long)t.ip[1], (long long)t.ip[2], op.device, rt->members[i].size() + 1,
                a, z);
      }
    }
    S->kernel_launches[op.device][op.kernel] += reps;
    if (timing && rt->kev[2 * i] && rt->batch_head[i] < 0) {   // batch members: timed with their head (last run)
      float k = 0.f;
      CU_OK(cudaEventElapsedTime(&k, rt->kev[2 * i], rt->kev[2 * i + 1]));
      S->kernel_ms[op.device][op.kernel] += k;
    }
  }
  if (trace) fclose(trace);
  return MM_OK;
}

mm_status mm_tune_chunks(mm_ctx* ctx, const mm_app* app, const mm_profile* prof, const mm_plan_opts* base,
                         const int32_t* candidates, int32_t n, void* const* buffers, int32_t reps, int32_t* best,
                         double* times_ms) {
  if (!ctx || !app || !prof || !base || !candidates || n < 1 || !buffers || !best)
    MM_FAIL(MM_EINVAL, "tune_chunks: null argument or no candidate");
  if (base->strategy != MM_DP_PERF && base->strategy != MM_DP_DEP && base->strategy != MM_DP_STATIC)
    MM_FAIL(MM_EINVAL, "tune_chunks: strategy %d has no task size (DP strategies only)", base->strategy);
  if (reps < 1) reps = 3;
  std::vector<double> t(n, 0.0);
  for (int32_t c = 0; c < n; ++c) {
    if (candidates[c] < 1) MM_FAIL(MM_EINVAL, "tune_chunks: candidate %d < 1", candidates[c]);
    mm_plan_opts o = *base;
    o.chunks_per_dev = candidates[c];
    mm_plan* p = nullptr;
    mm_status st = mm_plan_build(app, prof, &o, &p);
    if (st) return st;
    std::vector<double> v;
    for (int32_t r = 0; r <= reps && !st; ++r) {   // run 0 = warm-up
      mm_run_stats rs{};
      st = mm_run(ctx, p, buffers, nullptr, &rs);
      if (r > 0) v.push_back(rs.device_ms);
    }
    mm_plan_destroy(p);
    if (st) return st;
    std::sort(v.begin(), v.end());
    t[c] = v[v.size() / 2];
  }
  if (ctx->ipc) {   // every rank must pick the same candidate: max over ranks
    std::vector<uint64_t> row(n), all;
    for (int32_t c = 0; c < n; ++c) std::memcpy(&row[c], &t[c], 8);
    for (int32_t c0 = 0; c0 < n; c0 += 64) {
      const int32_t m = std::min<int32_t>(64, n - c0);
      mm_status st = ipc_allgather_u64(ctx->ipc, row.data() + c0, m, all);
      if (st) return st;
      for (int32_t q = 0; q < ctx->world; ++q)
        for (int32_t c = 0; c < m; ++c) {
          double v;
          std::memcpy(&v, &all[(size_t)q * m + c], 8);
          t[c0 + c] = std::max(t[c0 + c], v);
        }
    }
  } else if (ctx->world > 1) {   // every rank must pick the same candidate: max over ranks
    const int32_t me = first_owned(ctx);
    CU_OK(cudaSetDevice(ctx->dev[me].phys));
    double* dbuf = nullptr;
    CU_OK(cudaMalloc(&dbuf, sizeof(double) * n));
    cudaStream_t s = ctx->dev[me].stream;
    cudaError_t e = cudaMemcpyAsync(dbuf, t.data(), sizeof(double) * n, cudaMemcpyHostToDevice, s);
    ncclResult_t nr = e == cudaSuccess ? nccl().AllReduce(dbuf, dbuf, n, ncclFloat64, ncclMax, ctx->comm, s)
                                       : ncclSuccess;
    if (e == cudaSuccess && nr == ncclSuccess)
      e = cudaMemcpyAsync(t.data(), dbuf, sizeof(double) * n, cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess && nr == ncclSuccess) e = cudaStreamSynchronize(s);
    cudaFree(dbuf);
    if (nr != ncclSuccess) MM_FAIL(MM_ENCCL, "tune_chunks: allreduce failed (%d)", (int)nr);
    CU_OK(e);
  }
  int32_t b = 0;
  for (int32_t c = 1; c < n; ++c)
    if (t[c] < t[b] || (t[c] == t[b] && candidates[c] < candidates[b])) b = c;
  *best = candidates[b];
  if (times_ms)
    for (int32_t c = 0; c < n; ++c) times_ms[c] = t[c];
  return MM_OK;
}

mm_status mm_collect(mm_ctx* ctx, const mm_plan* plan_h, void* const* buffers, int32_t slot, void* dst,
                     int32_t dst_device) {
  if (!ctx || !plan_h || !dst) MM_FAIL(MM_EINVAL, "collect: null argument");
  std::vector<void*> reg_bufs;
  if (mm_status rb = resolve_buffers(ctx, plan_h->p, buffers, reg_bufs)) return rb;
  const PlanRt* prt = static_cast<const PlanRt*>(plan_h->p.rt);
  const Plan& plan = (prt && prt->last_adaptive && prt->ad) ? prt->ad->ap : plan_h->p;
  if (ctx->world != 1) MM_FAIL(MM_ENOTSUP, "collect: in-process contexts only");
  if (ctx->poisoned) MM_FAIL(MM_ESTATE, "ctx poisoned by an earlier CUDA error");
  if (dst_device >= ctx->G) MM_FAIL(MM_EINVAL, "collect: dst_device %d of G=%d", dst_device, ctx->G);
  if (slot < 0 || slot >= (int32_t)plan.app.buffers.size()) MM_FAIL(MM_EINVAL, "collect: slot");
  const int64_t eb = plan.app.buffers[slot].first;
  for (auto& seg : plan.final_owner[slot]) {
    const int32_t o = seg.second;
    if (o < 0) continue;
    const size_t bytes = (size_t)((seg.first.end - seg.first.begin) * eb);
    const char* src = static_cast<const char*>(buffers[(size_t)slot * ctx->G + o]) + seg.first.begin * eb;
    char* d = static_cast<char*>(dst) + seg.first.begin * eb;
    CU_OK(set_dev(ctx, o));
    if (dst_device < 0) CU_OK(cudaMemcpy(d, src, bytes, cudaMemcpyDeviceToHost));
    else if (ctx->dev[dst_device].phys == ctx->dev[o].phys) CU_OK(cudaMemcpy(d, src, bytes, cudaMemcpyDeviceToDevice));
    else CU_OK(cudaMemcpyPeer(d, ctx->dev[dst_device].phys, src, ctx->dev[o].phys, bytes));
  }
  return MM_OK;
}

// Glinda low-cost profiling (P49) + DP-Perf warm-up of 3 task instances per
// device (P311).  Excluded from run timings.
mm_status mm_profile_run(mm_ctx* ctx, const mm_app* app_h, void* const* buffers, const mm_profile_opts* po,
                         mm_profile* out) {
  if (!ctx || !app_h || !buffers || !out) MM_FAIL(MM_EINVAL, "profile: null argument");
  if (ctx->poisoned) MM_FAIL(MM_ESTATE, "ctx poisoned by an earlier CUDA error");
  const App& app = app_h->a;
  const int32_t G = ctx->G, K = (int32_t)app.kernels.size();
  if (K < 1 || K > MM_MAX_K) MM_FAIL(MM_EINVAL, "profile: K=%d", K);
  const int32_t reps = po && po->reps > 0 ? po->reps : 5;
  const int32_t warm = po && po->dp_warmup_chunks > 0 ? po->dp_warmup_chunks : 3;
  const int32_t kpd = po && po->chunks_per_dev > 0 ? po->chunks_per_dev : 8;
  *out = mm_profile{};
  out->G = G;
  out->K = K;
  out->staged = po && po->measure_link == 2 ? 1 : 0;
  std::vector<uint64_t> row(2 * MM_MAX_K + 2, 0);
  try {
    for (int32_t d = 0; d < G; ++d) {
      if (!ctx->dev[d].mine) continue;
      cudaStream_t s = ctx->dev[d].stream;
      CU_OK(set_dev(ctx, d));
      cudaEvent_t a, b;
      CU_OK(cudaEventCreate(&a));
      CU_OK(cudaEventCreate(&b));
      auto time_task = [&](const Task& t, float* ms) -> mm_status {
        ctx->dev[d].scr.epoch++;
        mm_status r = launch_task(ctx, app, t, d, buffers, s);  // warm-up
        if (r) return r;
        ctx->dev[d].scr.epoch++;
        CU_OK(cudaEventRecord(a, s));
        r = launch_task(ctx, app, t, d, buffers, s);
        if (r) return r;
        CU_OK(cudaEventRecord(b, s));
        CU_OK(cudaEventSynchronize(b));
        CU_OK(cudaEventElapsedTime(ms, a, b));
        return MM_OK;
      };
      for (int32_t k = 0; k < K; ++k) {
        const Kernel& kern = app.kernels[k];
        if (app.is_dag) {
          // per-task cost at the device's batch capacity: up to 16 independent
          // tasks of this kernel from its first step, launched as one batch
          // (how the executor runs them); non-batchable kernels: one task.
          std::vector<const Task*> ts;
          for (auto& x : app.dag)
            if (x.kernel == k && (ts.empty() || x.ip[2] == ts[0]->ip[2])) {
              if (!ts.empty() && !is_batchable_op(kern.op)) break;
              ts.push_back(&x);
              if (ts.size() >= 16) break;
            }
          if (ts.empty()) continue;
          std::vector<float> v(reps);
          for (int32_t i = 0; i < reps; ++i) {
            mm_status r = launch_task_batch(ctx, app, ts, d, buffers, s);  // warm-up
            if (r) return r;
            CU_OK(cudaEventRecord(a, s));
            r = launch_task_batch(ctx, app, ts, d, buffers, s);
            if (r) return r;
            CU_OK(cudaEventRecord(b, s));
            CU_OK(cudaEventSynchronize(b));
            CU_OK(cudaEventElapsedTime(&v[i], a, b));
          }
          std::sort(v.begin(), v.end());
          const uint64_t ns = std::max<uint64_t>(1, (uint64_t)(v[reps / 2] * 1e6 / (double)ts.size()));
          out->chunk_est_ns[d][k] = ns;
          out->fs_item[d][k] = ns * 1000000;
          continue;
        }
        // probe: the even share n/G (>= one wave of the kernel), median of reps
        int64_t probe = po && po->probe_items > 0 ? po->probe_items : chunk_size(kern.n, kern.granule, G);
        probe = std::min<int64_t>(std::max<int64_t>(probe, std::min(kern.n, kern.min_items)), kern.n);
        if (probe <= 0) {
          out->fs_item[d][k] = 1;
          out->chunk_est_ns[d][k] = 1;
          continue;
        }
        Task t = range_task(app, k, 0, 0, probe, 0);
        std::vector<float> v(reps);
        for (int32_t i = 0; i < reps; ++i) {
          mm_status r = time_task(t, &v[i]);
          if (r) return r;
        }
        std::sort(v.begin(), v.end());
        out->fs_item[d][k] = std::max<uint64_t>(1, (uint64_t)((double)v[reps / 2] * 1e12 / (double)probe));
        // DP-Perf warm-up (P311): `warm` nominal chunks on this device, issued
        // back to back as a dynamic schedule would, timed together (per-chunk
        // cost at the device's issue rate, launch latency amortised).
        const int64_t cs = chunk_size(kern.n, kern.granule, (int64_t)kpd * G);
        std::vector<Task> ch;
        for (int32_t i = 0; i < warm; ++i) {
          const int64_t b0 = std::min<int64_t>((int64_t)i * cs, std::max<int64_t>(0, kern.n - cs));
          ch.push_back(range_task(app, k, 0, b0, std::min(kern.n, b0 + cs), 0));
        }
        {
          mm_status r = launch_task(ctx, app, ch[0], d, buffers, s);  // warm-up launch
          if (r) return r;
          ctx->dev[d].scr.epoch++;
          CU_OK(cudaEventRecord(a, s));
          for (auto& c : ch) {
            r = launch_task(ctx, app, c, d, buffers, s);
            if (r) return r;
          }
          CU_OK(cudaEventRecord(b, s));
          CU_OK(cudaEventSynchronize(b));
          float ms = 0.f;
          CU_OK(cudaEventElapsedTime(&ms, a, b));
          out->chunk_est_ns[d][k] = std::max<uint64_t>(1, (uint64_t)((double)ms * 1e6 / (double)ch.size()));
        }
      }
      // Glinda's second metric (P49: "the GPU computation to data transfer
      // gap"): bytes/s of the link data crosses to reach device d.
      //  host (staged, measure_link = 2): one pinned host->device copy then one
      //   device->host copy of 64 MiB on d's stream, serialised as P119's
      //   "single host-to-device data transfer before the first kernel ... one
      //   device-to-host data transfer after the last"; B = 2 x 64 MiB / time.
      //  peer (resident, 0/1): a 64 MiB copy into d from another logical
      //   device's memory — cudaMemcpyPeerAsync when that device is another
      //   GPU, else a device-to-device copy (the XFER of logical devices that
      //   share a GPU); with no other device, a copy within d.
      {
        const size_t bytes = 64ull << 20;
        const bool host = po && po->measure_link == 2;
        void *x = nullptr, *y = nullptr;
        int32_t src_phys = ctx->dev[d].phys;
        for (int32_t q = 0; q < G; ++q)
          if (q != d && ctx->dev[q].mine && ctx->dev[q].phys != ctx->dev[d].phys) {
            src_phys = ctx->dev[q].phys;
            break;
          }
        CU_OK(cudaMalloc(&y, bytes));
        void* peer_src = nullptr;   // multi-process: the next rank's buffer, mapped (IPC)
        if (host) {
          CU_OK(cudaMallocHost(&x, bytes));
          std::memset(x, 0, bytes);
        } else if (ctx->ipc) {
          // the exchange link of a rank = a pull out of the next rank's memory
          // through its IPC mapping (NVLink between GPUs), as the XFERs do
          CU_OK(cudaMalloc(&x, bytes));
          CU_OK(cudaMemset(x, 0, bytes));
          CU_OK(cudaDeviceSynchronize());
          std::vector<char*> mapped;
          mm_status st = ipc_exchange_buffers(ctx->ipc, std::vector<void*>{x}, mapped);
          if (st) return st;
          peer_src = mapped[(size_t)((ctx->my_rank + 1) % ctx->world)];
        } else {
          if (src_phys != ctx->dev[d].phys) CU_OK(cudaSetDevice(src_phys));
          CU_OK(cudaMalloc(&x, bytes));
          CU_OK(cudaMemset(x, 0, bytes));
          CU_OK(cudaDeviceSynchronize());
          CU_OK(set_dev(ctx, d));
        }
        // time `nb` bytes of the link's copy (best of the timed repetitions)
        auto time_copy = [&](size_t nb, float* best) -> mm_status {
          *best = 0.f;
          for (int32_t i = 0; i < 1 + std::max<int32_t>(reps, 2); ++i) {   // first = warm-up
            CU_OK(cudaEventRecord(a, s));
            if (host) {
              CU_OK(cudaMemcpyAsync(y, x, nb, cudaMemcpyHostToDevice, s));
              CU_OK(cudaMemcpyAsync(x, y, nb, cudaMemcpyDeviceToHost, s));
            } else if (peer_src) {
              CU_OK(cudaMemcpyAsync(y, peer_src, nb, cudaMemcpyDefault, s));
            } else if (src_phys != ctx->dev[d].phys) {
              CU_OK(cudaMemcpyPeerAsync(y, ctx->dev[d].phys, x, src_phys, nb, s));
            } else {
              CU_OK(cudaMemcpyAsync(y, x, nb, cudaMemcpyDeviceToDevice, s));
            }
            CU_OK(cudaEventRecord(b, s));
            CU_OK(cudaEventSynchronize(b));
            float ms = 0.f;
            CU_OK(cudaEventElapsedTime(&ms, a, b));
            if (i > 0 && (*best == 0.f || ms < *best)) *best = ms;
          }
          return MM_OK;
        };
        float best = 0.f, small = 0.f;
        if (mm_status r = time_copy(bytes, &best)) return r;
        // R32: the fixed cost of one transfer = a 4 KiB copy of the same kind
        if (mm_status r = time_copy(4096, &small)) return r;
        if (peer_src) {   // no rank frees its buffer while a peer may still be pulling from it
          CU_OK(cudaDeviceSynchronize());
          if (mm_status st = ipc_barrier(ctx->ipc)) return st;
        }
        if (host) cudaFreeHost(x);
        else cudaFree(x);
        cudaFree(y);
        out->link_Bps[d] = (uint64_t)((double)(host ? 2 * bytes : bytes) / ((double)best * 1e-3));
        out->link_lat_ns[d] = (uint64_t)((double)small * 1e6 / (host ? 2.0 : 1.0));
      }
      cudaEventDestroy(a);
      cudaEventDestroy(b);
    }
  } catch (const std::bad_alloc&) {
    MM_FAIL(MM_ENOMEM, "profile: host memory");
  }
  if (ctx->ipc) {
    // exchange the per-device rows so every rank holds the same profile
    const int32_t me = first_owned(ctx);
    const int32_t rowlen = 2 * MM_MAX_K + 2;
    for (int32_t k = 0; k < MM_MAX_K; ++k) {
      row[k] = out->fs_item[me][k];
      row[MM_MAX_K + k] = out->chunk_est_ns[me][k];
    }
    row[2 * MM_MAX_K] = out->link_Bps[me];
    row[2 * MM_MAX_K + 1] = out->link_lat_ns[me];
    std::vector<uint64_t> all;
    mm_status st = ipc_allgather_u64(ctx->ipc, row.data(), rowlen, all);
    if (st) return st;
    for (int32_t d = 0; d < G; ++d) {
      const uint64_t* rr = all.data() + (size_t)ctx->dev[d].rank * rowlen;
      for (int32_t k = 0; k < MM_MAX_K; ++k) {
        out->fs_item[d][k] = rr[k];
        out->chunk_est_ns[d][k] = rr[MM_MAX_K + k];
      }
      out->link_Bps[d] = rr[2 * MM_MAX_K];
      out->link_lat_ns[d] = rr[2 * MM_MAX_K + 1];
    }
  } else if (ctx->world > 1) {
    // exchange the per-device rows so every rank holds the same profile
    const int32_t me = first_owned(ctx);
    const size_t rowlen = 2 * MM_MAX_K + 2;
    for (int32_t k = 0; k < MM_MAX_K; ++k) {
      row[k] = out->fs_item[me][k];
      row[MM_MAX_K + k] = out->chunk_est_ns[me][k];
    }
    row[2 * MM_MAX_K] = out->link_Bps[me];
    row[2 * MM_MAX_K + 1] = out->link_lat_ns[me];
    uint64_t *dsend = nullptr, *drecv = nullptr;
    CU_OK(set_dev(ctx, me));
    CU_OK(cudaMalloc(&dsend, rowlen * 8));
    CU_OK(cudaMalloc(&drecv, rowlen * 8 * ctx->world));
    CU_OK(cudaMemcpy(dsend, row.data(), rowlen * 8, cudaMemcpyHostToDevice));
    NCCL_OK(nccl().AllGather(dsend, drecv, rowlen, ncclUint64, ctx->comm, ctx->dev[me].stream));
    std::vector<uint64_t> all(rowlen * ctx->world);
    CU_OK(cudaStreamSynchronize(ctx->dev[me].stream));
    CU_OK(cudaMemcpy(all.data(), drecv, all.size() * 8, cudaMemcpyDeviceToHost));
    cudaFree(dsend);
    cudaFree(drecv);
    for (int32_t d = 0; d < G; ++d) {
      const uint64_t* rr = all.data() + (size_t)ctx->dev[d].rank * rowlen;
      for (int32_t k = 0; k < MM_MAX_K; ++k) {
        out->fs_item[d][k] = rr[k];
        out->chunk_est_ns[d][k] = rr[MM_MAX_K + k];
      }
      out->link_Bps[d] = rr[2 * MM_MAX_K];
      out->link_lat_ns[d] = rr[2 * MM_MAX_K + 1];
    }
  }
  return MM_OK;
}

int64_t mm_kernel_launch_count(void) { return g_kernel_launches.load(); }

mm_status mm_run_decisions(const mm_plan* plan_h, mm_decision* out, int64_t cap, int64_t* count) {
  if (!plan_h || !count) MM_FAIL(MM_EINVAL, "decisions: null argument");
  const PlanRt* rt = static_cast<const PlanRt*>(plan_h->p.rt);
  if (!rt || !rt->ad) {
    *count = 0;
    return MM_OK;
  }
  *count = (int64_t)rt->ad->decisions.size();
  if (cap < *count || (!out && *count)) MM_FAIL(MM_ERANGE, "decisions: cap");
  std::copy(rt->ad->decisions.begin(), rt->ad->decisions.end(), out);
  return MM_OK;
}

}  // extern "C"
