/*
 * mm.h — C ABI of the B200-native matchmaking library ("mm" = matchmaking).
 *
 * Implements the data-parallel hot path of Shen, Varbanescu, Martorell, Sips,
 * "Matchmaking Applications and Partitioning Strategies for Efficient Execution
 * on Heterogeneous Platforms", ICPP 2015 (/root/reference/PAPER.md, cited as
 * P<line> §<section>): register an application's kernels and execution flow
 * (P53 §III-A, Fig 2 P61-73), classify it (§III-B P73-115), rank the
 * partitioning strategies (§III-C Table I P177-197), compute a static split
 * from a profiled throughput model (Glinda, P49 §II-A) or a dynamic chunk
 * schedule (OmpSs DP-Perf / DP-Dep, P119), and run it on 1..8 logical devices
 * (B200 GPUs, or SM-budgeted partitions of one GPU).
 *
 * Conventions (every entry point):
 *  - Returns mm_status; MM_OK = 0.  No C++ exception, abort or exit crosses
 *    the ABI.  mm_last_error() returns a thread-local message for the last
 *    failure on the calling thread.
 *  - All sizes are int64 item / element counts; ranges are half-open
 *    [begin, end).  "Items" index a kernel's partitioned dimension (elements of
 *    a 1-D array, rows of a row-wise split grid/matrix, P311/P319).
 *  - Outputs go to caller-owned arrays with a (cap, *count) pair: a too-small
 *    cap returns MM_ERANGE with *count = the required size.
 *  - Opaque handles are created and destroyed by the library.  An mm_plan
 *    copies what it needs from its mm_app (the app may be destroyed after
 *    mm_plan_build).  A plan must not outlive the ctx it runs on.
 *  - Device memory of application buffers is CALLER-owned (one full-size
 *    allocation per logical device, e.g. torch tensors); the library never
 *    frees it.  Library-owned scratch (streams, events, pinned staging, NCCL
 *    communicator, CUDA graphs) is freed by mm_ctx_destroy / mm_plan_destroy.
 *  - The pure functions (mm_classify, mm_needs_sync, mm_rank, mm_split,
 *    mm_schedule, mm_plan_build and the mm_plan_* getters) touch no GPU and are
 *    deterministic: equal inputs give bit-identical outputs on every host and
 *    every rank.
 *  - A failed CUDA/NCCL call returns MM_ECUDA/MM_ENCCL and poisons the ctx:
 *    every later mm_run/mm_profile on it returns MM_ESTATE.
 */
#ifndef MM_H_
#define MM_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define MM_ABI_VERSION 1

enum { MM_MAX_DEV = 8, MM_MAX_K = 16, MM_MAX_ACCESS = 8, MM_MAX_BUF = 32,
       MM_MAX_PARAM = 8 };

typedef enum {
  MM_OK = 0, MM_EINVAL = -1, MM_ENOMEM = -2, MM_ECUDA = -3, MM_ENCCL = -4,
  MM_ESTATE = -5, MM_ENOTSUP = -6, MM_ERANGE = -7
} mm_status;

/* Application classes, Fig 3 / §III-B (P113-115). */
typedef enum { MM_SK_ONE = 1, MM_SK_LOOP = 2, MM_MK_SEQ = 3, MM_MK_LOOP = 4,
               MM_MK_DAG = 5 } mm_class;

/* Partitioning strategies, §III-C (P117-119).  MM_SP_CYCLIC is the static
 * 2-D block-cyclic owner-computes mapping used as the "static" comparator for
 * MK-DAG apps (P201; BASELINE configs[4]); it is not part of Table I.
 * MM_DP_STATIC is §V's conversion of dynamic partitioning into static (P565):
 * (1) the static ratio from Glinda's model with the task size = the whole
 * problem (SP-Single's split for one kernel, SP-Unified's for several on one
 * index space, else SP-Varied's per kernel); (2) that ratio converted into
 * task-instance counts per device over the DP chunks (largest remainder,
 * ties to the lower device id); (3) each device gets its count of
 * consecutive chunks, in device id order.  Not defined for MK-DAG apps
 * (MM_EINVAL). */
typedef enum { MM_SP_SINGLE = 1, MM_SP_UNIFIED = 2, MM_SP_VARIED = 3,
               MM_DP_PERF = 4, MM_DP_DEP = 5, MM_SP_CYCLIC = 6,
               MM_DP_STATIC = 7 } mm_strategy;

/* Inter-kernel synchronization (P51 taskwait; P119 SP-Varied conditions).
 * BARRIER: all devices finish the kernel before any starts the next.
 * FLUSH:   BARRIER + the kernel's outputs are copied to host memory. */
typedef enum { MM_SYNC_NONE = 0, MM_SYNC_BARRIER = 1, MM_SYNC_FLUSH = 2 } mm_sync;

typedef enum { MM_READ = 1, MM_WRITE = 2, MM_RW = 3 } mm_mode;

typedef struct { int64_t begin, end; } mm_range;

/* One buffer access of a kernel: per item the kernel touches elements
 * [item*elems_per_item, (item+1)*elems_per_item) of `buffer`; reads also
 * touch `halo_items` items on each side (clamped to the buffer). */
typedef struct {
  int32_t buffer;          /* buffer slot (mm_app_add_buffer) */
  int32_t mode;            /* mm_mode */
  int64_t elems_per_item;
  int64_t halo_items;
} mm_access;

/* Built-in sm_100a kernels (one per paper application kernel, Table II). */
typedef enum {
  MM_OP_CUSTOM = 0,          /* launch callback                                */
  MM_OP_STREAM_COPY = 1,     /* ops [a R, c W]        c = a          (P473)    */
  MM_OP_STREAM_SCALE = 2,    /* ops [c R, b W]        b = s c        fparam0 s */
  MM_OP_STREAM_ADD = 3,      /* ops [a R, b R, c W]   c = a + b                */
  MM_OP_STREAM_TRIAD = 4,    /* ops [b R, c R, a W]   a = fma(s,c,b) fparam0 s */
  MM_OP_HOTSPOT = 5,         /* ops [Tin R halo h, P R, Tout W]; iparam rows,cols,h;
                                fparam sdc, rx1, ry1, rz1, amb        (P319).
                                h > 1 (temporal blocking): one
                                launch = h iterations of rows [b,e), reading
                                Tin rows [b-h, e+h); needs cols % 4 == 0 and
                                16-B aligned buffers, h in {2,3,4,6,8}        */
  MM_OP_ROW_RESIDUAL = 6,    /* ops [Tin R, Tout R, rowsum(f64) W]; iparam rows,cols */
  MM_OP_BLACKSCHOLES = 7,    /* ops [S R, X R, T R, call W, put W]; fparam R, V (P311) */
  MM_OP_SGEMM = 8,           /* ops [A R (K per item), B R (whole), C W (N per item)];
                                iparam M, N, K, variant (0 auto,1 ffma,2 tf32x3) (P311) */
  MM_OP_CHOL_POTRF = 9,      /* DAG task ops [A]; task iparam k; kernel iparam T, b */
  MM_OP_CHOL_TRSM = 10,      /* DAG task iparam i, k                              */
  MM_OP_CHOL_SYRK = 11,      /* DAG task iparam i, k                              */
  MM_OP_CHOL_GEMM = 12,      /* DAG task iparam i, j, k                           */
  MM_OP_NBODY = 13           /* ops [pos R (whole), vel R, pos' W, vel' W] float4 bodies;
                                iparam n; fparam dt, eps2                  (P319)   */
} mm_op;

/* User kernel callback (MM_OP_CUSTOM): launch the kernel for `items` on
 * logical device `device` into `stream` (a cudaStream_t).  `operands[i]` is
 * this device's pointer for access i.  Returns 0 or a cudaError_t. */
typedef int32_t (*mm_launch_fn)(void* user, int32_t device, mm_range items,
                                void* const* operands, void* stream);

typedef struct {
  const char* name;             /* copied */
  int32_t op;                   /* mm_op */
  int64_t n_items;              /* size of the partitioned index space */
  int64_t granule;              /* split granularity (P379: warp size = 32) */
  int64_t min_items_per_dev;    /* decision threshold: one full wave (P49)  */
  mm_access access[MM_MAX_ACCESS];
  int32_t n_access;
  double fparam[MM_MAX_PARAM];
  int64_t iparam[MM_MAX_PARAM];
  mm_launch_fn launch;          /* MM_OP_CUSTOM only */
  void* user;
} mm_kernel_desc;

/* One explicit task of an MK-DAG app: element-interval accesses. */
typedef struct {
  int32_t buffer, mode;
  int64_t lo, hi;               /* element interval [lo, hi) */
} mm_task_access;

typedef struct {
  int32_t kernel;               /* kernel id (its op launches the task) */
  int64_t iparam[4];            /* e.g. Cholesky (i, j, k) */
  mm_task_access access[4];
  int32_t n_access;
  int32_t lane;                 /* 0: the kernel's compute lane (mm_app_set_lane),
                                   1: compute lane 1 for this task (R31; the
                                   Cholesky builtin puts SYRK(k+1,k), the update
                                   of the next diagonal tile, there beside
                                   POTRF / TRSM) */
} mm_task_desc;

typedef struct mm_app mm_app;
typedef struct mm_plan mm_plan;
typedef struct mm_ctx mm_ctx;

/* ------------------------------------------------------------------------
 * Application descriptor (D1: kernels, flow, sync; Fig 2 step 1-2)
 * ---------------------------------------------------------------------- */
mm_status mm_app_create(mm_app** out);
void      mm_app_destroy(mm_app* app);
/* elem_bytes in {1,2,4,8}; n_elems >= 0.  Returns the slot id. */
mm_status mm_app_add_buffer(mm_app* app, int32_t elem_bytes, int64_t n_elems, int32_t* slot);
/* Validates accesses against the buffers; returns the kernel id (program order). */
mm_status mm_app_add_kernel(mm_app* app, const mm_kernel_desc* desc, int32_t* kernel_id);
/* Invocation-graph edge (P113: sequence / loop / DAG).  With no edges the
 * kernels form a sequence in id order. */
mm_status mm_app_add_edge(mm_app* app, int32_t from_kernel, int32_t to_kernel);
/* Kernels first..last run `iterations` times (P113 loop).  A loop over only
 * part of the kernels is unrolled for classification (P115). */
mm_status mm_app_set_loop(mm_app* app, int32_t first, int32_t last, int64_t iterations);
/* Sync point after every invocation of `kernel` (P51 taskwait; P475). */
mm_status mm_app_set_sync(mm_app* app, int32_t kernel, int32_t sync);
/* Ping-pong: slots a and b exchange roles after each loop iteration. */
mm_status mm_app_set_swap(mm_app* app, int32_t slot_a, int32_t slot_b);
/* Execution lane of a kernel's tasks on a device (0 default, 1 second compute
 * stream): independent tasks of different lanes overlap (e.g. the MK-DAG
 * critical path POTRF/TRSM of step k+1 under the trailing updates of step k). */
mm_status mm_app_set_lane(mm_app* app, int32_t kernel, int32_t lane);
/* SK-Loop with unstable per-iteration performance (P117 -> MK-Seq). */
mm_status mm_app_set_unstable(mm_app* app, int32_t unstable);
/* Explicit task (MK-DAG).  Tasks are kept in creation order. */
mm_status mm_app_add_task(mm_app* app, const mm_task_desc* task);
/* Freeze the description of an app (P53 §III-A: "an application ... its
 * kernels and execution flow" is the input of the method).
 * Validates what the single calls cannot (>= 1 kernel, no loop over an
 * explicit-task DAG, every reference in range) and makes every later
 * mm_app_add_* / mm_app_set_* call on this app return MM_ESTATE.  Optional:
 * classify / split / plan also accept an unfinalized app.  Idempotent.
 * Errors: MM_EINVAL (null or invalid description; the app stays mutable). */
mm_status mm_app_finalize(mm_app* app);

/* Built-in apps of the paper (Table II) and of BASELINE.json configs. */
typedef enum {
  MM_APP_STREAM = 1,            /* ip0 n, ip1 passes, ip2 sync; fp0 scalar     */
  MM_APP_HOTSPOT = 2,           /* ip0 rows, ip1 cols, ip2 iterations, ip3 granule,
                                   ip4 min rows, ip5 temporal block h (0/1 = none;
                                   iterations % h == 0, else MM_EINVAL)        */
  MM_APP_STENCIL_REDUCTION = 3, /* ip0 rows, ip1 cols, ip2 steps, ip3 sync      */
  MM_APP_BLACKSCHOLES = 4,      /* ip0 n; fp0 R, fp1 V                          */
  MM_APP_SGEMM = 5,             /* ip0 M, ip1 N, ip2 K, ip3 variant             */
  MM_APP_CHOLESKY = 6,          /* ip0 n, ip1 tile b                            */
  MM_APP_NBODY = 7              /* ip0 bodies, ip1 iterations, ip2 granule, ip3 min; fp0 dt, fp1 eps2
                                   (a normal float > 0, else MM_EINVAL) */
} mm_app_id;
typedef struct { int64_t iparam[MM_MAX_PARAM]; double fparam[MM_MAX_PARAM]; } mm_app_params;
mm_status mm_app_builtin(int32_t app_id, const mm_app_params* p, mm_app** out);

/* Introspection. */
mm_status mm_app_info(const mm_app* app, int32_t* n_kernels, int32_t* n_buffers,
                      int64_t* n_tasks);
mm_status mm_app_buffer_info(const mm_app* app, int32_t slot, int32_t* elem_bytes,
                             int64_t* n_elems);

/* ------------------------------------------------------------------------
 * Pure control plane (host only)
 * ---------------------------------------------------------------------- */
/* Fig 3: kernels + flow -> class.  */
mm_status mm_classify(const mm_app* app, int32_t* cls);
/* 1 if any kernel carries a sync flag (P119 case 1). */
mm_status mm_needs_sync(const mm_app* app, int32_t* needs_sync);
/* Table I: ordered suitable strategies for (class, needs_sync). */
mm_status mm_rank(int32_t cls, int32_t needs_sync, int32_t* out, int32_t cap, int32_t* count);

/* Profile (D9): measured per (device, kernel) costs. */
typedef struct {
  int32_t G, K;
  int32_t staged;                            /* 1: host-resident inputs (R_GD term) */
  int32_t _pad;
  uint64_t fs_item[MM_MAX_DEV][MM_MAX_K];    /* femtoseconds per item (R_GC)  */
  uint64_t chunk_est_ns[MM_MAX_DEV][MM_MAX_K]; /* DP-Perf estimate per nominal chunk */
  uint64_t link_Bps[MM_MAX_DEV];             /* bytes/s into device d (R_GD)  */
  uint64_t link_lat_ns[MM_MAX_DEV];          /* fixed cost of one transfer into d (ns):
                                                DP-Perf prices a pull of B bytes as
                                                link_lat_ns + ceil(B 1e9 / link_Bps) (R32) */
} mm_profile;

/* Static split (SP-Single / SP-Unified / SP-Varied): out[k*G + d]. */
mm_status mm_split(const mm_app* app, const mm_profile* prof, int32_t strategy,
                   mm_range* out, int32_t cap, int32_t* devices_used);

typedef struct {
  int32_t strategy;          /* mm_strategy */
  int32_t chunks_per_dev;    /* DP: C = chunks_per_dev * G (default 8) */
  int32_t staged;            /* inputs start on the host; outputs end there */
  int32_t grid_rows;         /* SP-Cyclic process grid rows (0 = auto) */
  int32_t one_shot;          /* resident mode: 1 = program valid only from replicated
                                inputs (one run); 0 (default) = steady-state program,
                                planned from the state the program itself leaves, valid
                                for the first run and every repeated run (R22) */
  int32_t pipeline;          /* staged SP-Single/SP-Unified plans of pointwise apps (no halo,
                                no whole-buffer operand, no sync): split every device range
                                into this many sub-chunks run chunk-major, each flushed to
                                the host as soon as it is final, so H2D, kernels and D2H of
                                different sub-chunks overlap on separate streams (0/1 = off) */
  const mm_range* split;     /* optional SP split override [K*G] */
  int32_t halo_split;        /* SP plans, kernels with halo reads, G > 1 (R33, not in the paper):
                                each device range is run as its interior rows first, then the
                                rows within the halo depth of a neighbouring device's range, so
                                the interior kernel needs no pulled halo and overlaps the pulls
                                (device-to-device pulls run on the copy-in stream) */
  int32_t _pad2;
} mm_plan_opts;

/* One scheduled task. */
typedef struct {
  int32_t kernel;
  int32_t device;
  int64_t iter;
  mm_range items;            /* item range (range kernels) / tile id (DAG) */
  uint64_t finish_ns;        /* DP-Perf model finish time, else 0 */
} mm_chunk;

/* DP schedule (frozen estimates) = mm_plan_build + mm_plan_chunks. */
mm_status mm_schedule(const mm_app* app, const mm_profile* prof, const mm_plan_opts* opts,
                      mm_chunk* out, int64_t cap, int64_t* count);

/* Op program: the per-run sequence every device executes (global order). */
typedef enum { MM_OPK_KERNEL = 1, MM_OPK_XFER = 2, MM_OPK_BARRIER = 3,
               MM_OPK_FLUSH = 4 } mm_op_kind;
typedef struct {
  int32_t kind;              /* mm_op_kind */
  int32_t device;            /* KERNEL: executing device; XFER: destination;
                                FLUSH: source device */
  int32_t src;               /* XFER: source device, -1 = host (staged) */
  int32_t kernel;            /* KERNEL: kernel id */
  int32_t buffer;            /* XFER/FLUSH: physical buffer slot */
  int32_t _pad;
  int64_t task;              /* KERNEL: task index */
  int64_t iter;              /* KERNEL: loop iteration */
  mm_range r;                /* KERNEL: items; XFER/FLUSH: elements */
} mm_op_rec;

mm_status mm_plan_build(const mm_app* app, const mm_profile* prof, const mm_plan_opts* opts,
                        mm_plan** out);
void      mm_plan_destroy(mm_plan* plan);
typedef struct {
  int32_t cls, strategy, G, devices_used;
  int64_t n_tasks, n_ops, n_kernel_ops, n_xfer_ops, n_barriers, n_flush_ops;
  int64_t xfer_bytes, flush_bytes, h2d_bytes;
  int64_t items[MM_MAX_DEV][MM_MAX_K];   /* items per device per kernel (whole run) */
} mm_plan_info_t;
mm_status mm_plan_info(const mm_plan* plan, mm_plan_info_t* out);
mm_status mm_plan_ranges(const mm_plan* plan, mm_range* out, int32_t cap, int32_t* count);
mm_status mm_plan_chunks(const mm_plan* plan, mm_chunk* out, int64_t cap, int64_t* count);
mm_status mm_plan_ops(const mm_plan* plan, mm_op_rec* out, int64_t cap, int64_t* count);
/* Final location of buffer `slot` after the program: disjoint element ranges
 * covering [0, n) and, per range, the device holding its final value (the
 * last writer, else the lowest device with a valid copy, -1 = host only). */
mm_status mm_plan_owners(const mm_plan* plan, int32_t slot, mm_range* ranges, int32_t* owners,
                         int64_t cap, int64_t* count);

/* ------------------------------------------------------------------------
 * Runtime (GPU)
 * ---------------------------------------------------------------------- */
typedef struct {
  int32_t cuda_device;       /* CUDA ordinal (in this process) */
  int32_t sm_budget;         /* 0 = whole GPU; else a green context of >= this many SMs */
  int32_t rank;              /* process that owns this logical device */
  int32_t _pad;
} mm_device_spec;

/* Rendezvous id of a multi-process context (128 random bytes), created on
 * rank 0 and broadcast by the caller (IPC transport, the default). */
mm_status mm_rendezvous_id(void* out128);
/* NCCL unique id (128 bytes) for the NCCL transport (MM_TRANSPORT=nccl). */
mm_status mm_nccl_unique_id(void* out128);
/* G logical devices; this process is `my_rank` of `world` (1 = in-process:
 * every device has rank 0, exchanges are cudaMemcpyAsync on the consumer's
 * stream).  world > 1 (all ranks on one node): each rank owns exactly one
 * logical device; `nccl_id` = the same 128 bytes on every rank.
 *  - IPC transport (default): the ranks meet in a POSIX shared-memory block
 *    named after the id (host barrier, exchange of CUDA IPC handles); every
 *    rank runs the in-process executor's op program for its device, pulls
 *    (XFER) copy straight out of the producer rank's buffer through its IPC
 *    mapping (NVLink peer memory between GPUs; ranks may also share a GPU),
 *    and cross-rank hazards are waits on device-memory completion flags the
 *    producer/reader signals.  mm_run exchanges the buffer handles (a host
 *    barrier) and may capture the rank's program as a CUDA graph.
 *  - NCCL transport (environment MM_TRANSPORT=nccl, id from
 *    mm_nccl_unique_id): XFERs are grouped ncclSend/ncclRecv on the device's
 *    stream, BARRIER a 4-byte all-reduce; no graph capture; one rank per GPU.
 * Errors: MM_EINVAL, MM_ESTATE (a rank never joined the rendezvous within
 * 120 s), MM_ECUDA, MM_ENCCL. */
mm_status mm_ctx_create(const mm_device_spec* devs, int32_t G, int32_t my_rank, int32_t world,
                        const void* nccl_id, mm_ctx** out);
void      mm_ctx_destroy(mm_ctx* ctx);
/* The stream (cudaStream_t) the library launches on for logical device d. */
mm_status mm_ctx_stream(mm_ctx* ctx, int32_t d, void** stream);
/* SMs actually granted to logical device d. */
mm_status mm_ctx_sm_count(mm_ctx* ctx, int32_t d, int32_t* sms);
/* PyTorch stream interop (SURVEY §8(b) mm_ctx_set_stream): order the runs of
 * logical device d with a caller stream (e.g. torch.cuda.current_stream()
 * .cuda_stream).  mm_run then makes all of d's library streams wait for the
 * work already enqueued on `stream`, and `stream` wait for the run's last
 * kernel, so caller kernels before / after mm_run see its inputs / results
 * without a host synchronisation.  The stream stays caller-owned (never
 * destroyed by the library); NULL clears it.  Errors: MM_EINVAL (bad device
 * or a device another rank owns), MM_ESTATE (poisoned ctx). */
mm_status mm_ctx_set_stream(mm_ctx* ctx, int32_t d, void* stream);
/* Register one app buffer (SURVEY §8(b) mm_buffer_register): dev_ptrs[G] are
 * caller-owned device pointers of elem_bytes x n_elems, one full-size copy per
 * logical device (NULL for devices another rank owns); never freed by the
 * library.  The i-th registration stands for app buffer slot i: mm_run and
 * mm_collect called with buffers == NULL use the registered pointers, after
 * checking that every slot's element size and length match the plan's app.
 * Registrations last for the ctx's lifetime (extra registrations beyond the
 * app's buffer count are ignored by its runs).
 * Errors: MM_EINVAL (null / missing pointer of an owned device, bad size,
 * more than MM_MAX_BUF buffers), MM_ENOMEM. */
mm_status mm_buffer_register(mm_ctx* ctx, int32_t elem_bytes, int64_t n_elems, void* const* dev_ptrs,
                             int32_t* buf_id);

/* Device generator = synthgen.uniform (counter hash):
 * x[i] = lo + (hi-lo)*u(seed, array_id, start+i) for i in [0,n) into the
 * float32 device array `dst` of logical device d, on d's stream. */
mm_status mm_fill_uniform(mm_ctx* ctx, int32_t d, float* dst, int64_t n, uint64_t seed,
                          int32_t array_id, int64_t start, float lo, float hi);
/* Integer variant (values as float32): lo + (h24 % (hi-lo+1)). */
mm_status mm_fill_integers(mm_ctx* ctx, int32_t d, float* dst, int64_t n, uint64_t seed,
                           int32_t array_id, int64_t start, int32_t lo, int32_t hi);
/* = synthgen.spd_random(n) in the Cholesky app's tile-major layout (tile size
 * b): A = (S + S^T)/2 + n I with S[r][c] = u(seed, array_id, r*n + c),
 * evaluated in FP64 and rounded once to FP32. */
mm_status mm_fill_spd_tiles(mm_ctx* ctx, int32_t d, float* dst, int64_t n, int64_t b, uint64_t seed,
                            int32_t array_id);

typedef struct {
  int64_t probe_items;       /* 0 = per kernel, >= 4 waves */
  int32_t reps;              /* timed repetitions (median), default 5 */
  int32_t dp_warmup_chunks;  /* DP-Perf warm-up chunks per device per kernel (P311: 3) */
  int32_t chunks_per_dev;    /* nominal DP chunk size = n / (chunks_per_dev*G) */
  int32_t measure_link;      /* link_Bps[d], Glinda's transfer metric (P49):
                                0/1 (MM_LINK_PEER): 64 MiB copy into d from another
                                logical device (peer GPU, else a device-to-device copy
                                on the shared GPU; multi-process: a pull out of the
                                next rank's memory through its IPC mapping); the
                                resident exchange link.
                                2 (MM_LINK_HOST): pinned host->device + device->host of
                                64 MiB each, serialised (P119's staged transfers); sets
                                mm_profile.staged = 1 so mm_split adds the transfer term */
} mm_profile_opts;
enum { MM_LINK_PEER = 1, MM_LINK_HOST = 2 };

/* Glinda's low-cost profiling (P49) + the DP-Perf warm-up (P311), excluded
 * from run timings.  Runs kernels on the buffers (their contents change).
 * link_Bps: best of max(reps, 2) timed copies after one warm-up copy.
 * buffers[slot*G + d] = device pointer of the slot on logical device d
 * (NULL where this rank does not own d).  With world > 1 the per-device rows
 * are exchanged so every rank returns the same profile. */
mm_status mm_profile_run(mm_ctx* ctx, const mm_app* app, void* const* buffers,
                         const mm_profile_opts* opts, mm_profile* out);

typedef struct {
  int32_t use_graph;         /* capture the op program once, replay it (CUDA graph) */
  int32_t time_kernels;      /* CUDA events around every kernel op -> kernel_ms */
  int32_t adaptive;          /* DP-Perf plans, in-process only: decide each chunk's device
                                at run time from estimates updated with the measured times
                                of completed chunks (P119 "kept and updated"); the
                                decisions are logged (mm_run_decisions) */
  int32_t max_inflight;      /* adaptive: chunks in flight per device before the scheduler
                                waits for completions (default 4) */
  void* const* host;         /* staged / flush: host (pinned) pointer per slot, or NULL */
  int32_t no_wait;           /* 1: return once the run is enqueued (not with time_kernels or
                                adaptive): its streams are joined into the first owned device's
                                stream (mm_ctx_stream), so later runs and a caller stream set by
                                mm_ctx_set_stream are ordered after it; device_ms = -1; host
                                buffers must not be touched before that stream completes */
  int32_t repeat;            /* run the op program this many times back to back (0/1 = once;
                                with use_graph ONE graph holds all of them, so the runs pay
                                one launch); stats count every run, kernel_ms (time_kernels,
                                which use_graph then captures as event nodes) is the last
                                run's */
} mm_run_opts;

/* One adaptive DP-Perf decision: the snapshot it was taken on.  All times in
 * ns since the start of the run; eft_d = max(busy_d, ready_d) + cost_d and
 * chosen = argmin eft (ties -> lowest id).  Unused devices hold 0. */
typedef struct {
  int64_t task;
  int32_t chosen;
  int32_t kernel;
  uint64_t now_ns;
  uint64_t busy_ns[MM_MAX_DEV];
  uint64_t ready_ns[MM_MAX_DEV];
  uint64_t cost_ns[MM_MAX_DEV];
  uint64_t eft_ns[MM_MAX_DEV];
} mm_decision;

typedef struct {
  double wall_ms;                        /* host-observed, start -> all streams done */
  double device_ms;                      /* CUDA events: first op start -> last op end */
  double kernel_ms[MM_MAX_DEV][MM_MAX_K];/* sum of event-timed kernel ops (time_kernels) */
  int64_t kernel_launches[MM_MAX_DEV][MM_MAX_K];
  int64_t n_launches;                    /* kernels launched by this process */
  int64_t xfer_bytes;                    /* device<->device bytes moved */
  int64_t h2d_bytes, d2h_bytes;
} mm_run_stats;

/* Execute the plan's op program (blocking unless opts->no_wait: returns when
 * this process's devices are done).  buffers as in mm_profile_run, or NULL for the buffers
 * registered with mm_buffer_register; runs are ordered with the streams set
 * by mm_ctx_set_stream. */
mm_status mm_run(mm_ctx* ctx, mm_plan* plan, void* const* buffers, const mm_run_opts* opts,
                 mm_run_stats* stats);

/* Task-size auto-tuning (§V, P565: "the task size variation leads to
 * performance variation. Thus, auto-tuning is recommended to find the best
 * performing one").  For each of the n candidate task counts per device
 * (chunks_per_dev >= 1), builds the plan `base` with that count (base must
 * be DP-Perf, DP-Dep or DP-Static, else MM_EINVAL), runs it reps times after
 * one warm-up run (reps < 1 -> 3) and takes the median device time
 * (mm_run_stats.device_ms; multi-process: max over ranks, so every rank
 * picks the same value).  *best = the fastest candidate (ties -> the smaller
 * count); times_ms[n] (optional, caller-owned) = each candidate's median.
 * The buffers' contents are overwritten by the runs. */
mm_status mm_tune_chunks(mm_ctx* ctx, const mm_app* app, const mm_profile* prof, const mm_plan_opts* base,
                         const int32_t* candidates, int32_t n, void* const* buffers, int32_t reps,
                         int32_t* best, double* times_ms);

/* Decisions of the last adaptive run of this plan (creation order). */
mm_status mm_run_decisions(const mm_plan* plan, mm_decision* out, int64_t cap, int64_t* count);

/* Assemble buffer `slot` after a run: every element range is copied from the
 * device that holds its final value into `dst` (device memory of logical
 * device `dst_device`, or host memory if dst_device < 0).  In-process only.
 * buffers == NULL: the registered buffers (mm_buffer_register). */
mm_status mm_collect(mm_ctx* ctx, const mm_plan* plan, void* const* buffers, int32_t slot,
                     void* dst, int32_t dst_device);

/* Number of sm_100a kernel launches issued by this process so far (launches
 * replayed inside CUDA graphs are counted per replay). */
int64_t mm_kernel_launch_count(void);

/* sizeof of every ABI struct, in this order: mm_range, mm_access,
 * mm_kernel_desc, mm_task_access, mm_task_desc, mm_app_params, mm_profile,
 * mm_plan_opts, mm_chunk, mm_op_rec, mm_plan_info_t, mm_device_spec,
 * mm_profile_opts, mm_run_opts, mm_run_stats, mm_decision (bindings check
 * their mirrors). */
mm_status mm_abi_sizes(int64_t* out, int32_t cap, int32_t* count);

/* Thread-local message describing the last error on this thread. */
const char* mm_last_error(void);
const char* mm_strategy_name(int32_t strategy);
const char* mm_class_name(int32_t cls);

#ifdef __cplusplus
}
#endif
#endif /* MM_H_ */
