// stats_layout.hpp -- device-resident stats accumulator shared by the kernels
// (writers) and the host driver (reader). 64 bytes, one per chunk per slot.
#pragma once
#include <cuda_runtime.h>

#include <cmath>

namespace paper {

struct StatsAccum {
    unsigned long long lo[3];  // int128 fixed-point sums of x, y, z (units of 2^-60), low words
    unsigned long long hi[3];  // ... high words (two's complement)
    unsigned long long vmax2;  // max over nodes of the IEEE bits of v.v
    unsigned long long xmax;   // IEEE bits of an upper bound on max |x| over the nodes this slot
                               // covers (exact-stats domain, see xbound_step); 0: not tracked
};

// Exact-stats domain (S18): the centre sums are exact while every
// position is finite with |x| < 2^23 (stats.cuh). No per-node test runs in
// the step kernels; instead each state carries an upper bound B on max |x|:
// exact for a state the stats kernels sum (init / load: atomicMax of |x|),
// and for a state K1 produces, from the previous state's bound and this
// step's vmax: x' = x + v' h rounded once or twice, so
//   |x'| <= (|x| + |v'| |h| (1 + u)) (1 + u),  |v'| <= sqrt(vmax2) (1 + 2u),
// which the factor 1 + 2^-40 covers with margin (u = 2^-53; every operation
// below adds at most one more u). NaN / inf in vmax2 or B propagate: a state
// is inside the domain iff its bound is < 2^23 (false for NaN).
constexpr double kStatsDomain = 8388608.0;  // 2^23
__host__ __device__ inline double xbound_step(double B, double vmax2, double dt) {
    const double h = dt < 0.0 ? -dt : dt;
    return (B + sqrt(vmax2) * h) * (1.0 + 0x1p-40);
}
__host__ __device__ inline bool xbound_ok(double B) { return B < kStatsDomain; }

// Per-step stats history of a resident chunk ("centers" of every step,
// PAPER.md:330, 354): a ring of kStatsRing slots; the stats of the state after
// s steps live in slot ring_slot(s). A launch advancing steps [t, t+n) writes
// the slots of states t+1 .. t+n and zeroes those of t+n+1 and t+n+2 (the next
// launch advances at most two steps), so the ring holds the last
// kStatsRing - 2 states.
constexpr int kStatsRing = 128;  // power of two
static_assert((kStatsRing & (kStatsRing - 1)) == 0, "kStatsRing must be a power of two");
constexpr int kStatsHistory = kStatsRing - 2;
__host__ __device__ inline int ring_slot(unsigned long long state) {
    return (int)((state + (unsigned long long)(kStatsRing - 1)) & (unsigned long long)(kStatsRing - 1));
}

}  // namespace paper
