// stats_layout.hpp -- device-resident stats accumulator shared by the kernels
// (writers) and the host driver (reader). 64 bytes, one per chunk per slot.
#pragma once

namespace paper {

struct StatsAccum {
    unsigned long long lo[3];  // int128 fixed-point sums of x, y, z (units of 2^-60), low words
    unsigned long long hi[3];  // ... high words (two's complement)
    unsigned long long vmax2;  // max over nodes of the IEEE bits of v.v
    unsigned long long pad;
};

}  // namespace paper
