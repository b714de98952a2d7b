// Built-in application descriptors: the paper's evaluation apps (Table II,
// P205-247; workloads P311, P319, P473, P533) and the BASELINE.json configs
// (stencil+reduction MK-Loop, tiled Cholesky MK-DAG).  Host-only.
#include <algorithm>
#include <cstring>
#include <new>

#include "mm_internal.h"

using namespace mm;

namespace {

constexpr int64_t kSMs = 148;

mm_kernel_desc kd(const char* name, int32_t op, int64_t n, int64_t g, int64_t mn) {
  mm_kernel_desc d;
  std::memset(&d, 0, sizeof(d));
  d.name = name;
  d.op = op;
  d.n_items = n;
  d.granule = g;
  d.min_items_per_dev = mn;
  return d;
}

void acc(mm_kernel_desc& d, int32_t buf, int32_t mode, int64_t epi = 1, int64_t halo = 0) {
  d.access[d.n_access++] = mm_access{buf, mode, epi, halo};
}

// HotSpot coefficients (R15): Rodinia's model at its 1024^2 grid [ext]:
// chip 0.016 m, t_chip 5e-4 m, K_SI 100, SPEC_HEAT_SI 1.75e6, FACTOR_CHIP 0.5,
// MAX_PD 3e6, PRECISION 1e-3 -> Rx = Ry = 1/(2 K t) = 10, Rz = t/(K g^2),
// step/Cap = PRECISION (FACTOR_CHIP t SPEC_HEAT) / (MAX_PD FACTOR_CHIP SPEC_HEAT t g^2).
void hot_params(double* fp, const double* user) {
  const double g = 0.016 / 1024.0;
  const double t = 5e-4, K = 100.0;
  const double step_div_cap = 1e-3 / (3e6 * g * g);   // = 4096/3000
  const double def[5] = {step_div_cap, 2.0 * K * t, 2.0 * K * t, K * g * g / t, 80.0};
  for (int i = 0; i < 5; ++i) fp[i] = (user && user[i] != 0.0) ? user[i] : def[i];
}

mm_status stream_app(const mm_app_params& p, mm_app* app) {
  const int64_t n = p.iparam[0], passes = std::max<int64_t>(1, p.iparam[1]);
  const int32_t sync = (int32_t)p.iparam[2];
  const int64_t g = p.iparam[3] > 0 ? p.iparam[3] : 32;
  const int64_t mn = p.iparam[4] > 0 ? p.iparam[4] : kSMs * 8 * 1024 * 4;  // one wave of CTAs
  const double s = p.fparam[0] != 0.0 ? p.fparam[0] : 3.0;                 // STREAM scalar
  if (n < 0) MM_FAIL(MM_EINVAL, "stream: n");
  int32_t a, b, c;
  mm_app_add_buffer(app, 4, n, &a);
  mm_app_add_buffer(app, 4, n, &b);
  mm_app_add_buffer(app, 4, n, &c);
  mm_kernel_desc k1 = kd("copy", MM_OP_STREAM_COPY, n, g, mn);
  acc(k1, a, MM_READ); acc(k1, c, MM_WRITE);
  mm_kernel_desc k2 = kd("scale", MM_OP_STREAM_SCALE, n, g, mn);
  acc(k2, c, MM_READ); acc(k2, b, MM_WRITE); k2.fparam[0] = s;
  mm_kernel_desc k3 = kd("add", MM_OP_STREAM_ADD, n, g, mn);
  acc(k3, a, MM_READ); acc(k3, b, MM_READ); acc(k3, c, MM_WRITE);
  mm_kernel_desc k4 = kd("triad", MM_OP_STREAM_TRIAD, n, g, mn);
  acc(k4, b, MM_READ); acc(k4, c, MM_READ); acc(k4, a, MM_WRITE); k4.fparam[0] = s;
  for (auto* k : {&k1, &k2, &k3, &k4}) {
    mm_status st = mm_app_add_kernel(app, k, nullptr);
    if (st) return st;
  }
  if (passes > 1) mm_app_set_loop(app, 0, 3, passes);
  if (sync) for (int k = 0; k < 4; ++k) mm_app_set_sync(app, k, sync);
  return MM_OK;
}

int64_t hot_wave_rows(int64_t cols) {
  const int64_t ctas_per_strip = std::max<int64_t>(1, (cols / 4 + 255) / 256);
  return ((kSMs + ctas_per_strip - 1) / ctas_per_strip) * 32;
}

mm_status hotspot_app(const mm_app_params& p, mm_app* app) {
  const int64_t rows = p.iparam[0], cols = p.iparam[1], iters = std::max<int64_t>(1, p.iparam[2]);
  const int64_t g = p.iparam[3] > 0 ? p.iparam[3] : 1;
  const int64_t mn = p.iparam[4] > 0 ? p.iparam[4] : hot_wave_rows(cols);
  // temporal blocking: each launch advances tb iterations
  // with a halo of tb rows; the loop runs iters / tb times
  const int64_t tb = p.iparam[5] > 1 ? p.iparam[5] : 1;
  if (rows <= 0 || cols <= 0) MM_FAIL(MM_EINVAL, "hotspot: shape");
  if (tb > 1 && (iters % tb != 0 || cols % 4 != 0 || !(tb <= 4 || tb == 6 || tb == 8)))
    MM_FAIL(MM_EINVAL, "hotspot: temporal block %lld needs iterations %% tb == 0, cols %% 4 == 0, tb in {2,3,4,6,8}",
            (long long)tb);
  int32_t tin, tout, pw;
  mm_app_add_buffer(app, 4, rows * cols, &tin);
  mm_app_add_buffer(app, 4, rows * cols, &tout);
  mm_app_add_buffer(app, 4, rows * cols, &pw);
  mm_kernel_desc k = kd("hotspot", MM_OP_HOTSPOT, rows, g, mn);
  acc(k, tin, MM_READ, cols, (int32_t)tb); acc(k, pw, MM_READ, cols); acc(k, tout, MM_WRITE, cols);
  k.iparam[0] = rows; k.iparam[1] = cols; k.iparam[2] = tb;
  hot_params(k.fparam, p.fparam);
  mm_status st = mm_app_add_kernel(app, &k, nullptr);
  if (st) return st;
  mm_app_set_swap(app, tin, tout);
  if (iters / tb > 1) mm_app_set_loop(app, 0, 0, iters / tb);
  return MM_OK;
}

mm_status stencil_reduction_app(const mm_app_params& p, mm_app* app) {
  const int64_t rows = p.iparam[0], cols = p.iparam[1], steps = std::max<int64_t>(1, p.iparam[2]);
  const int32_t sync = (int32_t)p.iparam[3];
  const int64_t g = p.iparam[4] > 0 ? p.iparam[4] : 1;
  const int64_t mn = p.iparam[5] > 0 ? p.iparam[5] : hot_wave_rows(cols);
  if (rows <= 0 || cols <= 0) MM_FAIL(MM_EINVAL, "stencil_reduction: shape");
  int32_t tin, tout, pw, rs;
  mm_app_add_buffer(app, 4, rows * cols, &tin);
  mm_app_add_buffer(app, 4, rows * cols, &tout);
  mm_app_add_buffer(app, 4, rows * cols, &pw);
  mm_app_add_buffer(app, 8, rows, &rs);
  mm_kernel_desc a = kd("stencil", MM_OP_HOTSPOT, rows, g, mn);
  acc(a, tin, MM_READ, cols, 1); acc(a, pw, MM_READ, cols); acc(a, tout, MM_WRITE, cols);
  a.iparam[0] = rows; a.iparam[1] = cols;
  hot_params(a.fparam, p.fparam);
  mm_kernel_desc b = kd("residual", MM_OP_ROW_RESIDUAL, rows, g, mn);
  acc(b, tin, MM_READ, cols); acc(b, tout, MM_READ, cols); acc(b, rs, MM_WRITE, 1);
  b.iparam[0] = rows; b.iparam[1] = cols;
  mm_status st = mm_app_add_kernel(app, &a, nullptr);
  if (!st) st = mm_app_add_kernel(app, &b, nullptr);
  if (st) return st;
  mm_app_set_swap(app, tin, tout);
  mm_app_set_loop(app, 0, 1, steps);
  if (sync) mm_app_set_sync(app, 1, sync);
  return MM_OK;
}

mm_status bs_app(const mm_app_params& p, mm_app* app) {
  const int64_t n = p.iparam[0];
  const int64_t g = p.iparam[1] > 0 ? p.iparam[1] : 32;
  const int64_t mn = p.iparam[2] > 0 ? p.iparam[2] : kSMs * 8 * 256 * 4;
  if (n < 0) MM_FAIL(MM_EINVAL, "blackscholes: n");
  int32_t S, X, T, C, P;
  mm_app_add_buffer(app, 4, n, &S);
  mm_app_add_buffer(app, 4, n, &X);
  mm_app_add_buffer(app, 4, n, &T);
  mm_app_add_buffer(app, 4, n, &C);
  mm_app_add_buffer(app, 4, n, &P);
  mm_kernel_desc k = kd("blackscholes", MM_OP_BLACKSCHOLES, n, g, mn);
  acc(k, S, MM_READ); acc(k, X, MM_READ); acc(k, T, MM_READ); acc(k, C, MM_WRITE); acc(k, P, MM_WRITE);
  k.fparam[0] = p.fparam[0] != 0.0 ? p.fparam[0] : 0.02;   // NVIDIA SDK riskfree
  k.fparam[1] = p.fparam[1] != 0.0 ? p.fparam[1] : 0.30;   // NVIDIA SDK volatility
  return mm_app_add_kernel(app, &k, nullptr);
}

mm_status sgemm_app(const mm_app_params& p, mm_app* app) {
  const int64_t M = p.iparam[0], N = p.iparam[1], K = p.iparam[2];
  const int64_t g = p.iparam[4] > 0 ? p.iparam[4] : 128;   // CTA M-tile
  const int64_t tiles_n = std::max<int64_t>(1, (N + 127) / 128);
  const int64_t mn = p.iparam[5] > 0 ? p.iparam[5] : ((kSMs + tiles_n - 1) / tiles_n) * 128;
  if (M <= 0 || N <= 0 || K <= 0) MM_FAIL(MM_EINVAL, "sgemm: shape");
  int32_t A, B, C;
  mm_app_add_buffer(app, 4, M * K, &A);
  mm_app_add_buffer(app, 4, K * N, &B);
  mm_app_add_buffer(app, 4, M * N, &C);
  mm_kernel_desc k = kd("sgemm", MM_OP_SGEMM, M, g, mn);
  acc(k, A, MM_READ, K); acc(k, B, MM_READ, 0); acc(k, C, MM_WRITE, N);
  k.iparam[0] = M; k.iparam[1] = N; k.iparam[2] = K; k.iparam[3] = p.iparam[3];
  return mm_app_add_kernel(app, &k, nullptr);
}

mm_status cholesky_app(const mm_app_params& p, mm_app* app) {
  const int64_t n = p.iparam[0], b = p.iparam[1] > 0 ? p.iparam[1] : 1024;
  if (n <= 0 || n % b) MM_FAIL(MM_EINVAL, "cholesky: n must be a multiple of the tile");
  const int64_t T = n / b, bb = b * b;
  int32_t A;
  mm_app_add_buffer(app, 4, n * n, &A);   // tile-major: tile (i,j) at (i*T+j)*b*b
  const int32_t ops[4] = {MM_OP_CHOL_POTRF, MM_OP_CHOL_TRSM, MM_OP_CHOL_SYRK, MM_OP_CHOL_GEMM};
  const char* names[4] = {"potrf", "trsm", "syrk", "gemm"};
  for (int i = 0; i < 4; ++i) {
    mm_kernel_desc k = kd(names[i], ops[i], 1, 1, 1);
    k.iparam[0] = T; k.iparam[1] = b;
    mm_status st = mm_app_add_kernel(app, &k, nullptr);
    if (st) return st;
  }
  const int32_t e[7][2] = {{0, 1}, {1, 2}, {1, 3}, {2, 0}, {3, 1}, {3, 2}, {3, 3}};
  for (auto& x : e) mm_app_add_edge(app, x[0], x[1]);
  // critical path on lane 1: POTRF, TRSM and the update of the next
  // diagonal tile, SYRK(k+1,k), so POTRF(k+1) does not wait behind step k-1's
  // trailing updates on lane 0 (R31).  MM_CHOL_LOOKAHEAD_LANE: 0 = SYRK(k+1,k)
  // on lane 0 as well, 2 = also the GEMMs of column k+1 on lane 1 (32768^2:
  // 62.2 / 61.7 / 65.0 ms for 0 / 1 / 2 — POTRF(k+1) then queues behind them)
  mm_app_set_lane(app, 0, 1);
  mm_app_set_lane(app, 1, 1);
  static const int lookahead_lane = getenv("MM_CHOL_LOOKAHEAD_LANE") ? atoi(getenv("MM_CHOL_LOOKAHEAD_LANE")) : 1;
  auto tile = [&](int64_t i, int64_t j) { return (i * T + j) * bb; };
  auto task = [&](int32_t kern, int64_t i, int64_t j, int64_t k,
                  std::initializer_list<std::pair<int32_t, std::pair<int64_t, int64_t>>> a) {
    mm_task_desc t;
    std::memset(&t, 0, sizeof(t));
    t.kernel = kern;
    t.iparam[0] = i; t.iparam[1] = j; t.iparam[2] = k;
    t.lane = (j == k + 1 && (kern == 2 ? lookahead_lane >= 1 : kern == 3 && lookahead_lane >= 2)) ? 1 : 0;
    for (auto& x : a) {
      const int64_t lo = tile(x.second.first, x.second.second);
      t.access[t.n_access++] = mm_task_access{A, x.first, lo, lo + bb};
    }
    return mm_app_add_task(app, &t);
  };
  for (int64_t k = 0; k < T; ++k) {
    mm_status st = task(0, k, k, k, {{MM_RW, {k, k}}});
    if (st) return st;
    for (int64_t i = k + 1; i < T; ++i)
      if ((st = task(1, i, k, k, {{MM_READ, {k, k}}, {MM_RW, {i, k}}}))) return st;
    // the updates of column k+1 first (lookahead, R34), then the rest
    auto syrk = [&](int64_t i) { return task(2, i, i, k, {{MM_READ, {i, k}}, {MM_RW, {i, i}}}); };
    auto gemm = [&](int64_t i, int64_t j) {
      return task(3, i, j, k, {{MM_READ, {i, k}}, {MM_READ, {j, k}}, {MM_RW, {i, j}}});
    };
    if (k + 1 < T) {
      if ((st = syrk(k + 1))) return st;
      for (int64_t i = k + 2; i < T; ++i)
        if ((st = gemm(i, k + 1))) return st;
    }
    for (int64_t i = k + 2; i < T; ++i)
      if ((st = syrk(i))) return st;
    for (int64_t j = k + 2; j < T; ++j)
      for (int64_t i = j + 1; i < T; ++i)
        if ((st = gemm(i, j))) return st;
  }
  return MM_OK;
}

mm_status nbody_app(const mm_app_params& p, mm_app* app) {
  // Nbody (P223-227, P319): one all-pairs kernel iterated (SK-Loop); bodies are
  // float4 (4 elements per item); positions are read whole (every body needs
  // every position), velocities and outputs per body; ping-pong buffers.
  const int64_t n = p.iparam[0], iters = std::max<int64_t>(1, p.iparam[1]);
  const int64_t g = p.iparam[2] > 0 ? p.iparam[2] : 256;
  const int64_t mn = p.iparam[3] > 0 ? p.iparam[3] : kSMs * 256;
  if (n <= 0) MM_FAIL(MM_EINVAL, "nbody: n");
  int32_t p0, p1, v0, v1;
  mm_app_add_buffer(app, 4, 4 * n, &p0);
  mm_app_add_buffer(app, 4, 4 * n, &p1);
  mm_app_add_buffer(app, 4, 4 * n, &v0);
  mm_app_add_buffer(app, 4, 4 * n, &v1);
  mm_kernel_desc k = kd("nbody", MM_OP_NBODY, n, g, mn);
  acc(k, p0, MM_READ, 0); acc(k, v0, MM_READ, 4); acc(k, p1, MM_WRITE, 4); acc(k, v1, MM_WRITE, 4);
  k.iparam[0] = n;
  k.fparam[0] = p.fparam[0] != 0.0 ? p.fparam[0] : 1e-3;   // dt
  k.fparam[1] = p.fparam[1] != 0.0 ? p.fparam[1] : 1e-2;   // softening eps^2
  if (!((float)k.fparam[1] >= 1.17549435e-38f)) MM_FAIL(MM_EINVAL, "nbody: eps2 must be a normal float > 0");
  mm_status st = mm_app_add_kernel(app, &k, nullptr);
  if (st) return st;
  mm_app_set_swap(app, p0, p1);
  mm_app_set_swap(app, v0, v1);
  if (iters > 1) mm_app_set_loop(app, 0, 0, iters);
  return MM_OK;
}

}  // namespace

extern "C" mm_status mm_app_builtin(int32_t app_id, const mm_app_params* p, mm_app** out) {
  if (!p || !out) MM_FAIL(MM_EINVAL, "null argument");
  mm_app* app = nullptr;
  mm_status st = mm_app_create(&app);
  if (st) return st;
  try {
    switch (app_id) {
      case MM_APP_STREAM: st = stream_app(*p, app); break;
      case MM_APP_HOTSPOT: st = hotspot_app(*p, app); break;
      case MM_APP_STENCIL_REDUCTION: st = stencil_reduction_app(*p, app); break;
      case MM_APP_BLACKSCHOLES: st = bs_app(*p, app); break;
      case MM_APP_SGEMM: st = sgemm_app(*p, app); break;
      case MM_APP_CHOLESKY: st = cholesky_app(*p, app); break;
      case MM_APP_NBODY: st = nbody_app(*p, app); break;
      default: set_error("unknown builtin app %d", app_id); st = MM_EINVAL;
    }
  } catch (const std::bad_alloc&) {
    set_error("out of host memory");
    st = MM_ENOMEM;
  }
  if (st) {
    mm_app_destroy(app);
    return st;
  }
  *out = app;
  return MM_OK;
}
