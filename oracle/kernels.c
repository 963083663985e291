/*
 * oracle/kernels.c -- TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, obviously correct single-device semantics of the five benchmark
 * kernels ("for every thread of the FULL grid (one
 * device), apply the kernel's per-element formula; iterate with ping-pong
 * buffers").  The paper partitions a kernel so that it computes exactly the
 * single-GPU result (§1, §7), so the oracle is
 * the single-device definition and nothing else.
 *
 * Everything is computed in double (task rule: fp64 unless the paper fixes the
 * precision; PAPER.md never states one).  Inputs arrive as double arrays.
 * No blocking, fusion or reordering: one loop nest per definition.  OpenMP only
 * distributes independent output elements over host cores (it never changes an
 * element's operation order).  Built with -O2 -fopenmp -ffp-contract=off.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
 * reference leg may load this library.  It shares no code with the CUDA path.
 *
 * Kernel definitions (PAPER.md gives none; the readings are DESIGN.md §3):
 *   jacobi2d  -- C1, reading Q15 (Dirichlet, interior 0.25*(((N+S)+W)+E)).
 *   hotspot2d -- C2, reading Q14 (Rodinia form, frozen N=1024 constants,
 *                replicate/clamped borders).  P:L977-984 (§9.1 "Hotspot is a
 *                5-point stencil operating on a quadratic grid").
 *   heat3d    -- C3, reading Q15 (clamped 7-point, alpha = 1/8).
 *   gemm      -- C4, P:L995-1002 (§9.1 "Matmul computes the product of two
 *                dense, quadratic matrices"), reading Q17: C = A*B.
 *   nbody     -- C5, P:L986-993 (§9.1 "direct gravitational N-Body"),
 *                reading Q16: softened all-pairs, kick-drift Euler.
 */
#include <math.h>
#include <stdint.h>
#include <stddef.h>

static inline int64_t clampi(int64_t v, int64_t lo, int64_t hi) {
    return v < lo ? lo : (v > hi ? hi : v);
}

/* ---------------- C1: 2-D 5-point Jacobi, Dirichlet boundary ---------------- */
/* One sweep: for 1 <= i <= h-2, 1 <= j <= w-2
 *   out[i][j] = 0.25 * (((in[i-1][j] + in[i+1][j]) + in[i][j-1]) + in[i][j+1])
 * Boundary cells of `out` are left untouched (both buffers carry the boundary). */
void oracle_jacobi2d_sweep(const double* in, double* out, int64_t h, int64_t w) {
    #pragma omp parallel for schedule(static)
    for (int64_t i = 1; i < h - 1; ++i)
        for (int64_t j = 1; j < w - 1; ++j)
            out[i * w + j] = 0.25 * (((in[(i - 1) * w + j] + in[(i + 1) * w + j])
                                      + in[i * w + j - 1]) + in[i * w + j + 1]);
}

/* `iters` sweeps ping-ponging u0 -> u1 -> u0 ...; result left in u[iters % 2]. */
void oracle_jacobi2d(double* u0, double* u1, int64_t h, int64_t w, int iters) {
    for (int t = 0; t < iters; ++t) {
        if (t % 2 == 0) oracle_jacobi2d_sweep(u0, u1, h, w);
        else            oracle_jacobi2d_sweep(u1, u0, h, w);
    }
}

/* The same sweeps in fp32 storage AND arithmetic, each operation rounded to nearest as
 * written (-ffp-contract=off: no fused multiply-add; x86-64 SSE: no extended precision).
 * Not the reference for tolerances (that is the fp64 definition above): SURVEY.md §8(c)'s
 * optional strong pin -- a kernel that evaluates the same expression in the same order in
 * fp32 (jacobi2d, jacobi2d_tb use __fadd_rn / __fmul_rn) must match it bit for bit. */
void oracle_jacobi2d_f32(float* u0, float* u1, int64_t h, int64_t w, int iters) {
    for (int t = 0; t < iters; ++t) {
        const float* in = t % 2 == 0 ? u0 : u1;
        float* out = t % 2 == 0 ? u1 : u0;
        #pragma omp parallel for schedule(static)
        for (int64_t i = 1; i < h - 1; ++i)
            for (int64_t j = 1; j < w - 1; ++j)
                out[i * w + j] = 0.25f * (((in[(i - 1) * w + j] + in[(i + 1) * w + j])
                                           + in[i * w + j - 1]) + in[i * w + j + 1]);
    }
}

/* ---------------- C2: Hotspot (Rodinia form), clamped borders ---------------- */
/* For every cell (i, j), with N/S/E/W neighbours clamped to the grid:
 *   out = C + cap * (P + (S + N - 2C) * ry1 + (E + W - 2C) * rx1 + (amb - C) * rz1)
 */
void oracle_hotspot2d_sweep(const double* t, const double* p, double* out,
                            int64_t h, int64_t w, double cap, double rx1,
                            double ry1, double rz1, double amb) {
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < h; ++i)
        for (int64_t j = 0; j < w; ++j) {
            double c = t[i * w + j];
            double n = t[clampi(i - 1, 0, h - 1) * w + j];
            double s = t[clampi(i + 1, 0, h - 1) * w + j];
            double e = t[i * w + clampi(j + 1, 0, w - 1)];
            double ww = t[i * w + clampi(j - 1, 0, w - 1)];
            out[i * w + j] = c + cap * (p[i * w + j] + (s + n - 2.0 * c) * ry1
                                        + (e + ww - 2.0 * c) * rx1 + (amb - c) * rz1);
        }
}

void oracle_hotspot2d(double* t0, double* t1, const double* p, int64_t h, int64_t w,
                      int iters, double cap, double rx1, double ry1, double rz1,
                      double amb) {
    for (int it = 0; it < iters; ++it) {
        if (it % 2 == 0) oracle_hotspot2d_sweep(t0, p, t1, h, w, cap, rx1, ry1, rz1, amb);
        else             oracle_hotspot2d_sweep(t1, p, t0, h, w, cap, rx1, ry1, rz1, amb);
    }
}

/* ---------------- C3: 3-D 7-point heat, clamped (Neumann) ---------------- */
/* u'[k][i][j] = u + alpha * ((sum of the 6 clamped neighbours) - 6u) */
void oracle_heat3d_sweep(const double* u, double* out, int64_t d, int64_t h,
                         int64_t w, double alpha) {
    #pragma omp parallel for schedule(static)
    for (int64_t k = 0; k < d; ++k)
        for (int64_t i = 0; i < h; ++i)
            for (int64_t j = 0; j < w; ++j) {
                double c = u[(k * h + i) * w + j];
                double zm = u[(clampi(k - 1, 0, d - 1) * h + i) * w + j];
                double zp = u[(clampi(k + 1, 0, d - 1) * h + i) * w + j];
                double ym = u[(k * h + clampi(i - 1, 0, h - 1)) * w + j];
                double yp = u[(k * h + clampi(i + 1, 0, h - 1)) * w + j];
                double xm = u[(k * h + i) * w + clampi(j - 1, 0, w - 1)];
                double xp = u[(k * h + i) * w + clampi(j + 1, 0, w - 1)];
                out[(k * h + i) * w + j] =
                    c + alpha * ((zm + zp + ym + yp + xm + xp) - 6.0 * c);
            }
}

void oracle_heat3d(double* u0, double* u1, int64_t d, int64_t h, int64_t w,
                   int iters, double alpha) {
    for (int it = 0; it < iters; ++it) {
        if (it % 2 == 0) oracle_heat3d_sweep(u0, u1, d, h, w, alpha);
        else             oracle_heat3d_sweep(u1, u0, d, h, w, alpha);
    }
}

/* ---------------- C4: dense GEMM C = A * B (row-major) ---------------- */
/* C[i][j] = sum_{k=0}^{K-1} A[i][k] * B[k][j], accumulated in k order in double. */
void oracle_gemm(const double* a, const double* b, double* c, int64_t m, int64_t n,
                 int64_t k) {
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < m; ++i)
        for (int64_t j = 0; j < n; ++j) {
            double acc = 0.0;
            for (int64_t kk = 0; kk < k; ++kk) acc += a[i * k + kk] * b[kk * n + j];
            c[i * n + j] = acc;
        }
}

/* Same definition evaluated only at the sampled entries (rows[s], cols[s]).
 * A and B are passed as float (the stored operand values) and widened. */
void oracle_gemm_entries_f32(const float* a, const float* b, int64_t n, int64_t k,
                             const int64_t* rows, const int64_t* cols, int64_t ns,
                             double* out) {
    #pragma omp parallel for schedule(static)
    for (int64_t s = 0; s < ns; ++s) {
        int64_t i = rows[s], j = cols[s];
        double acc = 0.0;
        for (int64_t kk = 0; kk < k; ++kk)
            acc += (double)a[i * k + kk] * (double)b[kk * n + j];
        out[s] = acc;
    }
}

/* ---------------- C5: all-pairs N-body ---------------- */
/* pos[4*i] = (x, y, z, m).  a_i = sum_j m_j d_ij (|d_ij|^2 + eps2)^(-3/2),
 * d_ij = p_j - p_i (the j = i term is 0 because d = 0). */
static void nbody_accel_one(const double* pos, int64_t n, int64_t i, double eps2,
                            double* acc) {
    double ax = 0.0, ay = 0.0, az = 0.0;
    double xi = pos[4 * i], yi = pos[4 * i + 1], zi = pos[4 * i + 2];
    for (int64_t j = 0; j < n; ++j) {
        double dx = pos[4 * j] - xi, dy = pos[4 * j + 1] - yi, dz = pos[4 * j + 2] - zi;
        double r2 = dx * dx + dy * dy + dz * dz + eps2;
        double inv = 1.0 / (r2 * sqrt(r2));
        double s = pos[4 * j + 3] * inv;
        ax += dx * s; ay += dy * s; az += dz * s;
    }
    acc[0] = ax; acc[1] = ay; acc[2] = az;
}

/* Accelerations of the sampled targets only (acc_out[3*s .. 3*s+2]). */
void oracle_nbody_accel(const double* pos, int64_t n, const int64_t* targets,
                        int64_t nt, double eps2, double* acc_out) {
    #pragma omp parallel for schedule(static)
    for (int64_t s = 0; s < nt; ++s) nbody_accel_one(pos, n, targets[s], eps2, acc_out + 3 * s);
}

/* One kick-drift Euler step: v' = v + a dt ; x' = x + v' dt ; m' = m. */
void oracle_nbody_step(const double* pos, const double* vel, double* pos_out,
                       double* vel_out, int64_t n, double dt, double eps2) {
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i) {
        double a[3];
        nbody_accel_one(pos, n, i, eps2, a);
        for (int c = 0; c < 3; ++c) {
            vel_out[4 * i + c] = vel[4 * i + c] + a[c] * dt;
            pos_out[4 * i + c] = pos[4 * i + c] + vel_out[4 * i + c] * dt;
        }
        vel_out[4 * i + 3] = vel[4 * i + 3];
        pos_out[4 * i + 3] = pos[4 * i + 3];
    }
}

/* Threads OpenMP will use (reported as cpu_baseline.cores). */
#ifdef _OPENMP
#include <omp.h>
int oracle_num_threads(void) { return omp_get_max_threads(); }
#else
int oracle_num_threads(void) { return 1; }
#endif
