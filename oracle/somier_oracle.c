/*
 * somier_oracle.c -- plain sequential fp64 CPU oracle (TEST INFRASTRUCTURE).
 * See somier_oracle.h for the contract, citations and readings.
 *
 * Build: gcc -O2 -std=c11 -ffp-contract=off -fPIC -shared (oracle/build_oracle.py).
 * -ffp-contract=off: no fused multiply-add anywhere (reading S13), so every
 * expression below is evaluated with one IEEE round-to-nearest rounding per
 * operation, in the order written.
 */
#include "somier_oracle.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>
#include <time.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define IDX(p, i, j, k) ((((i) * (p)->n[1]) + (j)) * (p)->n[2] + (k))

static int valid(const oracle_params* p) {
    if (!p) return 0;
    for (int d = 0; d < 3; d++)
        if (p->n[d] < 3) return 0;
    if (!(p->mass > 0) || !(p->dt > 0)) return 0;
    if (!isfinite(p->spacing) || !isfinite(p->rest_len) || !isfinite(p->k_spring) ||
        !isfinite(p->amplitude) || !isfinite(p->mass) || !isfinite(p->dt))
        return 0;
    return 1;
}

static int64_t nnodes(const oracle_params* p) { return p->n[0] * p->n[1] * p->n[2]; }

static int is_interior(const oracle_params* p, int64_t i, int64_t j, int64_t k) {
    return i > 0 && i < p->n[0] - 1 && j > 0 && j < p->n[1] - 1 && k > 0 && k < p->n[2] - 1;
}

/* SplitMix64 (Steele, Lea, Flood 2014): state advances by the golden gamma
 * 0x9E3779B97F4A7C15; output = mix(state). The idx-th output of the stream
 * seeded with `seed` uses state = seed + (idx+1)*gamma (mod 2^64). */
uint64_t oracle_splitmix64_at(uint64_t seed, uint64_t idx) {
    uint64_t z = seed + (idx + 1u) * 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

/* Reading S7 / SURVEY §8(c) item 1: x0 = (i - (n0-1)/2) * spacing, etc. */
void oracle_rest_position(const oracle_params* p, int64_t i, int64_t j, int64_t k, double out[3]) {
    const int64_t idx[3] = {i, j, k};
    for (int c = 0; c < 3; c++) {
        double centre = (double)(p->n[c] - 1) / 2.0;
        out[c] = ((double)idx[c] - centre) * p->spacing;
    }
}

int oracle_init(const oracle_params* p, double* x, double* y, double* z,
                double* vx, double* vy, double* vz) {
    if (!valid(p)) return -1;
    double* X[3] = {x, y, z};
    for (int64_t i = 0; i < p->n[0]; i++)
        for (int64_t j = 0; j < p->n[1]; j++)
            for (int64_t k = 0; k < p->n[2]; k++) {
                int64_t g = IDX(p, i, j, k);
                double x0[3];
                oracle_rest_position(p, i, j, k, x0);
                for (int c = 0; c < 3; c++) {
                    double v = x0[c];
                    if (is_interior(p, i, j, k)) {
                        uint64_t r = oracle_splitmix64_at(p->seed, 3u * (uint64_t)g + (uint64_t)c);
                        double u = (double)(r >> 11) * 0x1.0p-53; /* u in [0,1), 53 bits */
                        double s = 2.0 * u - 1.0;                 /* exact */
                        v = x0[c] + p->amplitude * s;             /* 2 roundings */
                    }
                    X[c][g] = v;
                }
                vx[g] = 0.0;
                vy[g] = 0.0;
                vz[g] = 0.0;
            }
    return 0;
}

int oracle_init_window(const oracle_params* p, const int64_t lo[3], const int64_t w[3], double* x, double* y,
                       double* z, double* vx, double* vy, double* vz) {
    if (!valid(p)) return -1;
    for (int d = 0; d < 3; d++)
        if (lo[d] < 0 || w[d] < 0 || lo[d] + w[d] > p->n[d]) return -1;
    double* X[3] = {x, y, z};
    for (int64_t a = 0; a < w[0]; a++)
        for (int64_t b = 0; b < w[1]; b++)
            for (int64_t e = 0; e < w[2]; e++) {
                const int64_t i = lo[0] + a, j = lo[1] + b, k = lo[2] + e;
                const int64_t g = IDX(p, i, j, k);
                const int64_t l = (a * w[1] + b) * w[2] + e;
                double x0[3];
                oracle_rest_position(p, i, j, k, x0);
                for (int c = 0; c < 3; c++) {
                    double v = x0[c];
                    if (is_interior(p, i, j, k)) {
                        uint64_t r = oracle_splitmix64_at(p->seed, 3u * (uint64_t)g + (uint64_t)c);
                        double u = (double)(r >> 11) * 0x1.0p-53;
                        double s = 2.0 * u - 1.0;
                        v = x0[c] + p->amplitude * s;
                    }
                    X[c][l] = v;
                }
                vx[l] = 0.0;
                vy[l] = 0.0;
                vz[l] = 0.0;
            }
    return 0;
}

void oracle_spring(const double xp[3], const double xq[3], double K, double L, double g[3]) {
    double dx = xq[0] - xp[0];
    double dy = xq[1] - xp[1];
    double dz = xq[2] - xp[2];
    double d2 = (dx * dx + dy * dy) + dz * dz;
    double d = sqrt(d2);
    double f = (K * (d - L)) / d;
    g[0] = f * dx;
    g[1] = f * dy;
    g[2] = f * dz;
}

double oracle_acceleration_1(double f, double m) { return f / m; }
double oracle_velocity_1(double v, double a, double dt) { return v + a * dt; }
double oracle_position_1(double x, double v, double dt) { return x + v * dt; }

void oracle_forces(const oracle_params* p, const double* x, const double* y, const double* z,
                   double* fx, double* fy, double* fz) {
    const int64_t n0 = p->n[0], n1 = p->n[1], n2 = p->n[2];
    /* the optional all-cores build (-fopenmp, liboracle_omp.so) splits the i
     * loop of the node-independent kernels; every node is computed by the same
     * expressions, so the results are bit-identical to the sequential build */
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n0; i++)
        for (int64_t j = 0; j < n1; j++)
            for (int64_t k = 0; k < n2; k++) {
                int64_t g = IDX(p, i, j, k);
                if (!is_interior(p, i, j, k)) {
                    fx[g] = 0.0;
                    fy[g] = 0.0;
                    fz[g] = 0.0;
                    continue;
                }
                /* neighbours in the order -i, +i, -j, +j, -k, +k */
                const int64_t nb[6] = {IDX(p, i - 1, j, k), IDX(p, i + 1, j, k),
                                       IDX(p, i, j - 1, k), IDX(p, i, j + 1, k),
                                       IDX(p, i, j, k - 1), IDX(p, i, j, k + 1)};
                const double xp[3] = {x[g], y[g], z[g]};
                double gs[6][3];
                for (int s = 0; s < 6; s++) {
                    const double xq[3] = {x[nb[s]], y[nb[s]], z[nb[s]]};
                    oracle_spring(xp, xq, p->k_spring, p->rest_len, gs[s]);
                }
                double F[3];
                for (int c = 0; c < 3; c++)
                    F[c] = ((gs[0][c] + gs[1][c]) + (gs[2][c] + gs[3][c])) + (gs[4][c] + gs[5][c]);
                fx[g] = F[0];
                fy[g] = F[1];
                fz[g] = F[2];
            }
}

void oracle_accelerations(const oracle_params* p, const double* fx, const double* fy, const double* fz,
                          double* ax, double* ay, double* az) {
    const int64_t n = nnodes(p);
#pragma omp parallel for schedule(static)
    for (int64_t g = 0; g < n; g++) {
        ax[g] = oracle_acceleration_1(fx[g], p->mass);
        ay[g] = oracle_acceleration_1(fy[g], p->mass);
        az[g] = oracle_acceleration_1(fz[g], p->mass);
    }
}

void oracle_velocities(const oracle_params* p, const double* ax, const double* ay, const double* az,
                       double* vx, double* vy, double* vz) {
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < p->n[0]; i++)
        for (int64_t j = 0; j < p->n[1]; j++)
            for (int64_t k = 0; k < p->n[2]; k++) {
                if (!is_interior(p, i, j, k)) continue;
                int64_t g = IDX(p, i, j, k);
                vx[g] = oracle_velocity_1(vx[g], ax[g], p->dt);
                vy[g] = oracle_velocity_1(vy[g], ay[g], p->dt);
                vz[g] = oracle_velocity_1(vz[g], az[g], p->dt);
            }
}

void oracle_positions(const oracle_params* p, const double* x, const double* y, const double* z,
                      const double* vx, const double* vy, const double* vz,
                      double* xn, double* yn, double* zn) {
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < p->n[0]; i++)
        for (int64_t j = 0; j < p->n[1]; j++)
            for (int64_t k = 0; k < p->n[2]; k++) {
                int64_t g = IDX(p, i, j, k);
                if (!is_interior(p, i, j, k)) {
                    xn[g] = x[g];
                    yn[g] = y[g];
                    zn[g] = z[g];
                    continue;
                }
                xn[g] = oracle_position_1(x[g], vx[g], p->dt);
                yn[g] = oracle_position_1(y[g], vy[g], p->dt);
                zn[g] = oracle_position_1(z[g], vz[g], p->dt);
            }
}

/* round-half-even(x * 2^60) as an exact int128 (reading S15). x*2^60 is exact
 * in fp64 (power-of-two scaling, |x| < 2^10); nearbyint() rounds half to even in
 * the default rounding mode and is the identity once |x*2^60| >= 2^52. */
static __int128 quantise(double v) {
    double s = ldexp(v, 60);
    return (__int128)nearbyint(s);
}

void oracle_centers(const oracle_params* p, const double* x, const double* y, const double* z,
                    const double* vx, const double* vy, const double* vz, oracle_stats* out) {
    const int64_t n = nnodes(p);
    const double* X[3] = {x, y, z};
    __int128 sum[3] = {0, 0, 0};
    double vmax2 = 0.0;
    for (int64_t g = 0; g < n; g++) {
        for (int c = 0; c < 3; c++) sum[c] += quantise(X[c][g]);
        double v2 = (vx[g] * vx[g] + vy[g] * vy[g]) + vz[g] * vz[g];
        if (v2 > vmax2 || isnan(v2)) vmax2 = isnan(vmax2) ? vmax2 : v2;
    }
    for (int c = 0; c < 3; c++) {
        out->sum_lo[c] = (uint64_t)(unsigned __int128)sum[c];
        out->sum_hi[c] = (int64_t)(sum[c] >> 64);
        out->centre[c] = ldexp((double)sum[c], -60) / (double)n;
    }
    memcpy(&out->vmax2_bits, &vmax2, sizeof vmax2);
    out->vmax = sqrt(vmax2);
}

int oracle_step(const oracle_params* p, const double* x, const double* y, const double* z,
                double* vx, double* vy, double* vz, double* xn, double* yn, double* zn,
                oracle_stats* stats) {
    if (!valid(p)) return -1;
    const int64_t n = nnodes(p);
    double* scratch = (double*)malloc(sizeof(double) * (size_t)n * 6);
    if (!scratch) return -1;
    double *fx = scratch, *fy = fx + n, *fz = fy + n, *ax = fz + n, *ay = ax + n, *az = ay + n;
    oracle_forces(p, x, y, z, fx, fy, fz);             /* forces        */
    oracle_accelerations(p, fx, fy, fz, ax, ay, az);   /* accelerations */
    oracle_velocities(p, ax, ay, az, vx, vy, vz);      /* velocities    */
    oracle_positions(p, x, y, z, vx, vy, vz, xn, yn, zn); /* positions  */
    if (stats) oracle_centers(p, xn, yn, zn, vx, vy, vz, stats); /* centers */
    free(scratch);
    return 0;
}

int oracle_run_timed(const oracle_params* p, int64_t nsteps, double* x, double* y, double* z,
                     double* vx, double* vy, double* vz, oracle_stats* stats, double* seconds) {
    if (!valid(p) || nsteps < 0) return -1;
    const int64_t n = nnodes(p);
    double* buf = (double*)malloc(sizeof(double) * (size_t)n * 3);
    if (!buf) return -1;
    double *xa = x, *ya = y, *za = z;
    double *xb = buf, *yb = buf + n, *zb = buf + 2 * n;
    struct timespec t0, t1;
    clock_gettime(CLOCK_MONOTONIC, &t0);
    for (int64_t s = 0; s < nsteps; s++) {
        if (oracle_step(p, xa, ya, za, vx, vy, vz, xb, yb, zb, stats) != 0) {
            free(buf);
            return -1;
        }
        double* t;
        t = xa; xa = xb; xb = t;
        t = ya; ya = yb; yb = t;
        t = za; za = zb; zb = t;
    }
    clock_gettime(CLOCK_MONOTONIC, &t1);
    if (seconds) *seconds = (double)(t1.tv_sec - t0.tv_sec) + 1e-9 * (double)(t1.tv_nsec - t0.tv_nsec);
    if (xa != x) {
        memcpy(x, xa, sizeof(double) * (size_t)n);
        memcpy(y, ya, sizeof(double) * (size_t)n);
        memcpy(z, za, sizeof(double) * (size_t)n);
    }
    if (nsteps == 0 && stats) oracle_centers(p, x, y, z, vx, vy, vz, stats);
    free(buf);
    return 0;
}

int oracle_run(const oracle_params* p, int64_t nsteps, double* x, double* y, double* z,
               double* vx, double* vy, double* vz, oracle_stats* stats) {
    return oracle_run_timed(p, nsteps, x, y, z, vx, vy, vz, stats, NULL);
}

int oracle_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

void oracle_stencil3(const double* a, double* b, int64_t n) {
    for (int64_t i = 1; i < n - 1; i++) b[i] = a[i - 1] + a[i] + a[i + 1];
}
