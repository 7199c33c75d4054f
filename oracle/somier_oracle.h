/*
 * somier_oracle.h -- plain sequential fp64 CPU oracle for the Somier time step.
 *
 * TEST INFRASTRUCTURE ONLY. Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library. The product path
 * (paper_conf_ipps_torresft22_b200/) never includes, links or calls it, and this
 * oracle shares no code, header, table or constant generator with the CUDA path.
 *
 * What it computes: the Somier mini-app step of Torres, Ferrer, Teruel,
 * "A Novel Set of Directives for Multi-device Programming with OpenMP"
 * (§V): per time step the kernels
 *   forces -> accelerations -> velocities -> positions -> centers
 * (PAPER.md:321-330, 354), on 4 variables x 3 separate 3-D fp64 grids
 * (PAPER.md:338-342). Where the paper is silent the readings S1-S16 of
 * SURVEY.md §8(c) / DESIGN.md §3 are used; each function names the ones it
 * relies on.
 *
 * Grid convention: n[0] x n[1] x n[2] nodes, i outermost, k contiguous;
 * linear index g = (i*n1 + j)*n2 + k. Each variable is three separate grids
 * (x, y, z components), like the paper's "3 3D-grids" per variable.
 *
 * Pins: every function below is pinned by tests/test_oracle_pins.py against
 * closed forms, invariants, brute force or printed values,
 * including mass M != 1 and rest length L != spacing (C2, C4, C7, C8); 22
 * one-line mutants of this file each fail a pin (tools/mutate_oracle.py).
 * No function is "parity unpinned".
 */
#ifndef SOMIER_ORACLE_H
#define SOMIER_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct {
    int64_t  n[3];       /* grid nodes per dimension, i outermost, each >= 3 */
    double   spacing;    /* lattice spacing of the rest positions            */
    double   rest_len;   /* spring rest length L                              */
    double   k_spring;   /* spring stiffness K                                */
    double   mass;       /* node mass M                                       */
    double   dt;         /* time step h                                       */
    double   amplitude;  /* initial random displacement amplitude a           */
    uint64_t seed;       /* SplitMix64 seed of the initial displacement       */
} oracle_params;

typedef struct {
    double   centre[3];     /* mean position over all n0*n1*n2 nodes           */
    double   vmax;          /* sqrt(max over nodes of v.v)                      */
    uint64_t sum_lo[3];     /* exact int128 fixed-point sum (2^-60 units), low  */
    int64_t  sum_hi[3];     /* ... and high 64 bits (two's complement)          */
    uint64_t vmax2_bits;    /* IEEE bit pattern of max v.v                      */
} oracle_stats;

/* Counter-based SplitMix64: the idx-th output (0-based) of the sequential
 * SplitMix64 stream seeded with `seed`. Reading S7. */
uint64_t oracle_splitmix64_at(uint64_t seed, uint64_t idx);

/* Centred rest lattice position of node (i,j,k). Reading S7 / item 1. */
void oracle_rest_position(const oracle_params* p, int64_t i, int64_t j, int64_t k, double out[3]);

/* Initial state (reading S7): interior nodes x = x0 + a*(2u-1), u from the
 * generator at counter 3g+c; fixed (face) nodes at x0; V = 0. Returns 0, or -1
 * on invalid parameters. Arrays are caller-owned, n0*n1*n2 doubles each. */
int oracle_init(const oracle_params* p, double* x, double* y, double* z,
                double* vx, double* vy, double* vz);

/* The same initial state restricted to the window [lo[d], lo[d]+w[d]) of the
 * global grid p->n (global indices, so the values equal the corresponding
 * entries of oracle_init); arrays hold w0*w1*w2 doubles. Used to check single
 * nodes of full-size GPU runs through their light cone. Returns 0 or -1. */
int oracle_init_window(const oracle_params* p, const int64_t lo[3], const int64_t w[3], double* x, double* y,
                       double* z, double* vx, double* vy, double* vz);

/* One central Hooke spring (reading S1): force on node p from the spring to q.
 * d = xq - xp; |d| = sqrt((dx*dx+dy*dy)+dz*dz); f = (K*(|d|-L))/|d|; g = f*d. */
void oracle_spring(const double xp[3], const double xq[3], double K, double L, double g[3]);

/* Per-node primitives of kernels 2-4, called by the grid loops below (and by
 * the two-mass pin, which cannot be built inside a grid with fixed faces). */
double oracle_acceleration_1(double f, double m);           /* a = f / M      */
double oracle_velocity_1(double v, double a, double dt);    /* v + a*h        */
double oracle_position_1(double x, double v, double dt);    /* x + v*h        */

/* Kernel 1, "forces": F at every interior node from its 6
 * face neighbours, summed ((g-i + g+i) + (g-j + g+j)) + (g-k + g+k); F = 0 on
 * the fixed faces (reading S6). */
void oracle_forces(const oracle_params* p, const double* x, const double* y, const double* z,
                   double* fx, double* fy, double* fz);

/* Kernel 2, "accelerations": A = F / M at every node. */
void oracle_accelerations(const oracle_params* p, const double* fx, const double* fy, const double* fz,
                          double* ax, double* ay, double* az);

/* Kernel 3, "velocities": V = V + A*h at interior nodes
 * (semi-implicit Euler, reading S4). Fixed nodes keep V. */
void oracle_velocities(const oracle_params* p, const double* ax, const double* ay, const double* az,
                       double* vx, double* vy, double* vz);

/* Kernel 4, "positions": Xn = X + V*h at interior nodes using
 * the already-updated V; fixed nodes Xn = X. Xn is a separate buffer (Jacobi,
 * reading S5). */
void oracle_positions(const oracle_params* p, const double* x, const double* y, const double* z,
                      const double* vx, const double* vy, const double* vz,
                      double* xn, double* yn, double* zn);

/* Kernel 5, "centers": centre of mass of all nodes via an exact
 * int128 sum of round-half-even(x * 2^60), then S*2^-60/N; vmax = sqrt(max v.v).
 * Reading S8, S15. */
void oracle_centers(const oracle_params* p, const double* x, const double* y, const double* z,
                    const double* vx, const double* vy, const double* vz, oracle_stats* out);

/* One full time step: the five kernels in the paper's order.
 * Reads X (t), updates V in place, writes Xn (t+1). Returns 0 or -1. */
int oracle_step(const oracle_params* p, const double* x, const double* y, const double* z,
                double* vx, double* vy, double* vz, double* xn, double* yn, double* zn,
                oracle_stats* stats);

/* nsteps steps in place on (x,y,z,vx,vy,vz); stats of the last step. */
int oracle_run(const oracle_params* p, int64_t nsteps, double* x, double* y, double* z,
               double* vx, double* vy, double* vz, oracle_stats* stats);

/* oracle_run with the step loop timed by CLOCK_MONOTONIC (the steady clock):
 * *seconds = wall time of the nsteps steps (every step's five kernels, stats
 * included), without the setup and the final copy. For bench.py's CPU
 * baseline. */
int oracle_run_timed(const oracle_params* p, int64_t nsteps, double* x, double* y, double* z,
                     double* vx, double* vy, double* vz, oracle_stats* stats, double* seconds);

/* Threads the node loops use: 1 for the sequential build; omp_get_max_threads()
 * for the optional all-cores build (liboracle_omp.so, same source compiled with
 * -fopenmp; the i loops of forces / velocities / positions and the node loop of
 * accelerations split statically; bit-identical results, tested). */
int oracle_threads(void);

/* Listing 2-4 toy loop: B[i] = A[i-1]+A[i]+A[i+1] for
 * i in [1, N-1), evaluated left to right. */
void oracle_stencil3(const double* a, double* b, int64_t n);

#ifdef __cplusplus
}
#endif
#endif
