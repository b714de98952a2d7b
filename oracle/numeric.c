/*
 * ORACLE — numeric kernels of the paper's applications, plain single-threaded C.
 *
 * TEST INFRASTRUCTURE ONLY: only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  It shares no code,
 * header or constant generator with the CUDA path (paper_conf_icpp_shenvms15_b200/csrc).
 *
 * Build: gcc -O2 -ffp-contract=off -fno-fast-math -shared -fPIC (oracle/numeric.py).
 * -ffp-contract=off keeps every a*b+c as two roundings unless fmaf() is written.
 *
 * Precision: the paper never names one; its footprints fix 4-byte elements
 * (P311: 6144^2 x3 = 0.4 GB, 80,530,632 x5 = 1.5 GB; P319: 8192^2 x3 = 0.75 GB;
 * P473: 62,914,560 x3 = 0.7 GB) -> FP32 storage (R13).  STREAM and
 * HotSpot are computed in FP32 with the operation order written below (the GPU
 * must match bit for bit); BlackScholes, MatrixMul and Cholesky are computed in
 * FP64 and compared within the north_star tolerances.
 */
#include <math.h>
#include <stdint.h>
#include <stddef.h>

/* ---------------------------------------------------------------------------
 * STREAM (P203, P235-245 Table II "The STREAM benchmark [22]", P473: four
 * kernels copy/scale/add/triad on 1-D arrays).  Kernel bodies are McCalpin's
 * STREAM [22] definitions: c=a; b=s*c; c=a+b; a=b+s*c.  Triad is one fused
 * multiply-add (R14).  Each works on the element range [lo,hi).
 * ------------------------------------------------------------------------- */
void or_stream_copy(const float *a, float *c, int64_t lo, int64_t hi) {
    for (int64_t j = lo; j < hi; ++j) c[j] = a[j];
}
void or_stream_scale(float *b, const float *c, float s, int64_t lo, int64_t hi) {
    for (int64_t j = lo; j < hi; ++j) b[j] = s * c[j];
}
void or_stream_add(const float *a, const float *b, float *c, int64_t lo, int64_t hi) {
    for (int64_t j = lo; j < hi; ++j) c[j] = a[j] + b[j];
}
void or_stream_triad(float *a, const float *b, const float *c, float s, int64_t lo, int64_t hi) {
    for (int64_t j = lo; j < hi; ++j) a[j] = fmaf(s, c[j], b[j]);
}
/* STREAM-Seq = 1 pass (P203 "limiting the number of iterations"); STREAM-Loop
 * = `passes` passes (P533). */
void or_stream_run(float *a, float *b, float *c, int64_t n, float s, int32_t passes) {
    for (int32_t p = 0; p < passes; ++p) {
        or_stream_copy(a, c, 0, n);
        or_stream_scale(b, c, s, 0, n);
        or_stream_add(a, b, c, 0, n);
        or_stream_triad(a, b, c, s, 0, n);
    }
}

/* ---------------------------------------------------------------------------
 * HotSpot (P229-233 Table II "Rodinia [2]", P319: 8192x8192 grid, iterated).
 * The thermal update is Rodinia's explicit 5-point scheme [ext]:
 *   T' = T + sdc * ( P + (S + N - 2T)*ry1 + (E + W - 2T)*rx1 + (amb - T)*rz1 )
 * with out-of-grid neighbours replaced by the cell itself (zero lateral flux at
 * the chip edge), coefficients fixed at Rodinia's 1024^2 values (R15).
 * FP32 operation order (R16):
 *   two = c + c; dv = ((s + n) - two) * ry1; dh = ((e + w) - two) * rx1;
 *   dz = (amb - c) * rz1; sum = ((p + dv) + dh) + dz; out = c + sdc * sum
 * Rows [r0, r1) of Tout are written.
 * ------------------------------------------------------------------------- */
typedef struct { float sdc, rx1, ry1, rz1, amb; } or_hot_coef;

void or_hotspot_rows(const float *tin, const float *pw, float *tout, int64_t rows,
                     int64_t cols, int64_t r0, int64_t r1, const or_hot_coef *k) {
    for (int64_t y = r0; y < r1; ++y) {
        for (int64_t x = 0; x < cols; ++x) {
            float c = tin[y * cols + x];
            float n = (y > 0) ? tin[(y - 1) * cols + x] : c;
            float s = (y < rows - 1) ? tin[(y + 1) * cols + x] : c;
            float w = (x > 0) ? tin[y * cols + x - 1] : c;
            float e = (x < cols - 1) ? tin[y * cols + x + 1] : c;
            float two = c + c;
            float dv = ((s + n) - two) * k->ry1;
            float dh = ((e + w) - two) * k->rx1;
            float dz = (k->amb - c) * k->rz1;
            float sum = ((pw[y * cols + x] + dv) + dh) + dz;
            float prod = k->sdc * sum;
            tout[y * cols + x] = c + prod;
        }
    }
}

/* `iters` ping-pong iterations starting from t0; the result is left in t0 when
 * iters is even and in t1 when odd (returns 0 or 1 = index of the result). */
int32_t or_hotspot_run(float *t0, float *t1, const float *pw, int64_t rows, int64_t cols,
                       int32_t iters, const or_hot_coef *k) {
    float *in = t0, *out = t1;
    for (int32_t it = 0; it < iters; ++it) {
        or_hotspot_rows(in, pw, out, rows, cols, 0, rows, k);
        float *tmp = in; in = out; out = tmp;
    }
    return (iters % 2 == 0) ? 0 : 1;
}

/* MK-Loop second kernel (BASELINE configs[3]): per-row FP64 sum of squared
 * change, rowsum[y] = sum_x ((double)t1 - (double)t0)^2, x ascending. */
void or_row_residual(const float *t0, const float *t1, double *rowsum, int64_t cols,
                     int64_t r0, int64_t r1) {
    for (int64_t y = r0; y < r1; ++y) {
        double acc = 0.0;
        for (int64_t x = 0; x < cols; ++x) {
            double d = (double)t1[y * cols + x] - (double)t0[y * cols + x];
            acc += d * d;
        }
        rowsum[y] = acc;
    }
}

/* ---------------------------------------------------------------------------
 * BlackScholes (P217-221 Table II "Nvidia OpenCL SDK", P311: 80,530,632
 * options in a 1-D array).  European call/put, NVIDIA-SDK formulation [ext]:
 *   d1 = (ln(S/X) + (R + V^2/2) T) / (V sqrt T),  d2 = d1 - V sqrt T
 *   call = S N(d1) - X e^{-RT} N(d2),  put = X e^{-RT} (1 - N(d2)) - S (1 - N(d1))
 * N(.) = Abramowitz-Stegun 26.2.17 polynomial.  Computed in FP64.
 * ------------------------------------------------------------------------- */
static double or_cnd(double d) {
    const double A1 = 0.31938153, A2 = -0.356563782, A3 = 1.781477937,
                 A4 = -1.821255978, A5 = 1.330274429;
    const double RSQRT2PI = 0.39894228040143267793994605993438;
    double kk = 1.0 / (1.0 + 0.2316419 * fabs(d));
    double cnd = RSQRT2PI * exp(-0.5 * d * d) *
                 (kk * (A1 + kk * (A2 + kk * (A3 + kk * (A4 + kk * A5)))));
    if (d > 0) cnd = 1.0 - cnd;
    return cnd;
}
double or_cnd_public(double d) { return or_cnd(d); }

void or_blackscholes(const float *S, const float *X, const float *T, double *call,
                     double *put, int64_t n, double R, double V) {
    for (int64_t i = 0; i < n; ++i) {
        double s = S[i], x = X[i], t = T[i];
        double sqrtT = sqrt(t);
        double d1 = (log(s / x) + (R + 0.5 * V * V) * t) / (V * sqrtT);
        double d2 = d1 - V * sqrtT;
        double n1 = or_cnd(d1), n2 = or_cnd(d2);
        double expRT = exp(-R * t);
        call[i] = s * n1 - x * expRT * n2;
        put[i] = x * expRT * (1.0 - n2) - s * (1.0 - n1);
    }
}

/* ---------------------------------------------------------------------------
 * MatrixMul (P211-215 Table II, P311: C = A x B, row-wise split).  Definition
 * C[i][j] = sum_k A[i][k] B[k][j]; i-k-j loop, FP64 accumulation, rows [r0,r1).
 * ------------------------------------------------------------------------- */
void or_sgemm_rows(const float *A, const float *B, float *C, int64_t M, int64_t N,
                   int64_t K, int64_t r0, int64_t r1, double *rowacc /* N scratch */) {
    (void)M;
    for (int64_t i = r0; i < r1; ++i) {
        for (int64_t j = 0; j < N; ++j) rowacc[j] = 0.0;
        for (int64_t k = 0; k < K; ++k) {
            double a = (double)A[i * K + k];
            const float *brow = B + k * N;
            for (int64_t j = 0; j < N; ++j) rowacc[j] += a * (double)brow[j];
        }
        for (int64_t j = 0; j < N; ++j) C[i * N + j] = (float)rowacc[j];
    }
}

/* ---------------------------------------------------------------------------
 * Cholesky (MK-DAG stand-in; BASELINE configs[4]; not in the paper, P201).
 * Definition A = L L^T, L lower with positive diagonal; Cholesky-Banachiewicz
 * in FP64, row-major n x n, upper triangle of L zeroed.  Returns 0, or -(i+1)
 * if the pivot of row i is not positive.
 * ------------------------------------------------------------------------- */
int32_t or_cholesky(const double *A, double *L, int64_t n) {
    for (int64_t i = 0; i < n * n; ++i) L[i] = 0.0;
    for (int64_t i = 0; i < n; ++i) {
        for (int64_t j = 0; j <= i; ++j) {
            double s = A[i * n + j];
            for (int64_t k = 0; k < j; ++k) s -= L[i * n + k] * L[j * n + k];
            if (i == j) {
                if (!(s > 0.0)) return (int32_t)(-(i + 1));
                L[i * n + i] = sqrt(s);
            } else {
                L[i * n + j] = s / L[j * n + j];
            }
        }
    }
    return 0;
}

/* ---------------------------------------------------------------------------
 * Nbody (P223-227 Table II "Mont-Blanc benchmark suite", P319: 1,048,576
 * bodies, 64 MB, iterated -> SK-Loop).  All-pairs gravitational acceleration
 * with Plummer softening and a semi-implicit Euler step (the CUDA SDK nbody
 * integrator [ext]):
 *   a_i = sum_j m_j (p_j - p_i) / (|p_j - p_i|^2 + eps2)^{3/2}
 *   v_i' = v_i + a_i dt,   p_i' = p_i + v_i' dt
 * Bodies are float4 (x, y, z, m) positions and (vx, vy, vz, 0) velocities;
 * computed in FP64, stored in FP32 (R13).  Bodies [r0, r1) are written.
 * ------------------------------------------------------------------------- */
void or_nbody_step(const float *pin, const float *vin, float *pout, float *vout, int64_t n,
                   int64_t r0, int64_t r1, double dt, double eps2) {
    for (int64_t i = r0; i < r1; ++i) {
        const double xi = pin[4 * i], yi = pin[4 * i + 1], zi = pin[4 * i + 2];
        double ax = 0.0, ay = 0.0, az = 0.0;
        for (int64_t j = 0; j < n; ++j) {
            const double dx = (double)pin[4 * j] - xi, dy = (double)pin[4 * j + 1] - yi,
                         dz = (double)pin[4 * j + 2] - zi;
            const double d2 = dx * dx + dy * dy + dz * dz + eps2;
            const double s = (double)pin[4 * j + 3] / (d2 * sqrt(d2));
            ax += dx * s;
            ay += dy * s;
            az += dz * s;
        }
        const double vx = vin[4 * i] + ax * dt, vy = vin[4 * i + 1] + ay * dt, vz = vin[4 * i + 2] + az * dt;
        vout[4 * i] = (float)vx;
        vout[4 * i + 1] = (float)vy;
        vout[4 * i + 2] = (float)vz;
        vout[4 * i + 3] = vin[4 * i + 3];
        pout[4 * i] = (float)(xi + vx * dt);
        pout[4 * i + 1] = (float)(yi + vy * dt);
        pout[4 * i + 2] = (float)(zi + vz * dt);
        pout[4 * i + 3] = pin[4 * i + 3];
    }
}
