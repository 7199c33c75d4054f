// stats_layout.hpp -- device-resident stats accumulator shared by the kernels
// (writers) and the host driver (reader). 64 bytes, one per chunk per slot.
#pragma once
#include <cuda_runtime.h>

namespace paper {

struct StatsAccum {
    unsigned long long lo[3];  // int128 fixed-point sums of x, y, z (units of 2^-60), low words
    unsigned long long hi[3];  // ... high words (two's complement)
    unsigned long long vmax2;  // max over nodes of the IEEE bits of v.v
    unsigned long long pad;
};

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
