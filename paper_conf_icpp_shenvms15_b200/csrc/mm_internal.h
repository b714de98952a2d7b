// Internal data structures of the matchmaking library (host side).
// Nothing here is visible through the C ABI (include/mm.h).
#pragma once

#include <cstdint>
#include <map>
#include <string>
#include <vector>

#include "mm.h"

namespace mm {

// Thread-local error reporting (mm_last_error).
void set_error(const char* fmt, ...);
#define MM_FAIL(code, ...) do { ::mm::set_error(__VA_ARGS__); return (code); } while (0)

struct Access {
  int32_t buffer = 0, mode = 0;
  int64_t epi = 1, halo = 0;
};

struct Kernel {
  std::string name;
  int32_t op = MM_OP_CUSTOM;
  int64_t n = 0, granule = 32, min_items = 1;
  std::vector<Access> acc;
  double fp[MM_MAX_PARAM] = {0};
  int64_t ip[MM_MAX_PARAM] = {0};
  mm_launch_fn launch = nullptr;
  void* user = nullptr;
  int32_t lane = 0;          // compute stream of the device its tasks run on
};

// A task's access in element units of a physical buffer.  Reads cover
// [lo,hi) (core plus halo); the non-halo part is [core_lo, core_hi).
struct TaskAcc {
  int32_t buffer = 0, mode = 0;
  int64_t lo = 0, hi = 0, core_lo = 0, core_hi = 0;
};

struct Task {
  int32_t kernel = 0;
  int32_t inv = 0;          // invocation index (range apps), 0 for DAG tasks
  int64_t iter = 0;
  int64_t b = 0, e = 0;     // item range (range apps) / tile id (DAG)
  int64_t ip[4] = {0, 0, 0, 0};
  std::vector<TaskAcc> acc;
  int32_t lane = 0;         // DAG tasks: 1 = compute lane 1 whatever the kernel's lane
};

// Compute lane of a task (R31): lane 1 if its kernel or the task itself asks for it.
struct Kernel;
struct App;
int32_t task_lane(const App& app, const Task& t);

struct App {
  std::vector<std::pair<int32_t, int64_t>> buffers;  // (elem_bytes, n_elems)
  std::vector<Kernel> kernels;
  std::vector<std::pair<int32_t, int32_t>> edges;
  bool has_loop = false;
  int32_t loop_first = 0, loop_last = 0;
  int64_t loop_iters = 1;
  std::map<int32_t, int32_t> sync;
  bool unstable = false;
  std::vector<std::pair<int32_t, int32_t>> swaps;
  std::vector<Task> dag;    // explicit DAG tasks (creation order)
  bool is_dag = false;
};

struct Invocation { int32_t kernel; int64_t iter; };

// Cross-stream dependency of an op (in-process execution): wait for op `op`
// issued on the stream of logical device `dev`.
struct Wait { int32_t dev; int64_t op; };

struct Plan {
  App app;                  // copy of the app (plans outlive apps)
  mm_profile prof{};        // the profile the plan was built from
  int32_t chunks_per_dev = 8;
  int32_t cls = 0, strategy = 0, G = 1, devices_used = 0;
  int32_t staged = 0;
  std::vector<mm_range> ranges;       // SP: [K*G]
  std::vector<Task> tasks;            // creation order
  std::vector<int32_t> task_dev;
  std::vector<uint64_t> task_fin;     // DP-Perf model finish (ns)
  bool pipelined = false;             // staged sub-chunk pipeline (mm_plan_opts.pipeline)
  std::vector<uint8_t> flush_after;   // pipelined: flush the group's outputs after task t
  std::vector<mm_op_rec> ops;         // global op program
  std::vector<int32_t> op_stream;     // executing logical device (-1 barrier)
  std::vector<std::vector<Wait>> waits;   // per op
  std::vector<uint8_t> needs_event;       // op is waited on by another stream
  // final location of every element: per buffer, segments (lo, hi, owner dev)
  std::vector<std::vector<std::pair<mm_range, int32_t>>> final_owner;
  mm_plan_info_t info{};
  // runtime cache (owned by the runtime, freed by mm_plan_destroy)
  void* rt = nullptr;
};

// core.cpp
int32_t classify(const App& app);
bool needs_sync(const App& app);
std::vector<int32_t> rank(int32_t cls, bool with_sync);
std::vector<Invocation> invocations(const App& app);
int32_t phys_buffer(const App& app, int32_t slot, int64_t iter);
Task range_task(const App& app, int32_t k, int64_t iter, int64_t b, int64_t e, int32_t inv);
int64_t chunk_size(int64_t n, int64_t granule, int64_t C);
mm_status split_items(int64_t n, int64_t granule, const std::vector<uint64_t>& cost,
                      int64_t min_items, std::vector<mm_range>& out);
mm_status sp_split(const App& app, const mm_profile& prof, int32_t strategy,
                   std::vector<mm_range>& out);
mm_status build_plan(const App& app, const mm_profile& prof, const mm_plan_opts& opts, Plan& plan);

// Incremental op-program builder (adaptive DP-Perf): the caller sets
// plan.task_dev[t] and appends task t's ops with inc_planner_step; the
// ownership directory persists across begin/end cycles (runs).
struct IncPlanner;
IncPlanner* inc_planner_create(const App& app, Plan& plan);
void inc_planner_begin(IncPlanner* ip);
mm_status inc_planner_step(IncPlanner* ip, int64_t t);
mm_status inc_planner_end(IncPlanner* ip);
void inc_planner_destroy(IncPlanner* ip);

// runtime.cu
void plan_runtime_free(Plan* plan);

}  // namespace mm

struct mm_app {
  mm::App a;
  bool frozen = false;   // mm_app_finalize: no further mutation
};
struct mm_plan { mm::Plan p; };
