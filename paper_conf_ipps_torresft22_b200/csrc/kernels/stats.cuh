// stats.cuh -- the "centers" reduction fused into the step
// kernels: exact int128 fixed-point sums of the positions (reading S15:
// order-independent, so every launch configuration and every chunk partition
// gives the same bits) and the max of v.v as an unsigned bit pattern.
#pragma once
#include <cstdint>

#include "../stats_layout.hpp"
#include "node_math.cuh"

namespace paper {

// round_half_even(x * 2^60) as an exact int128. x*2^60 is exact (power-of-two
// scale). Below 2^62 in magnitude __double2ll_rn rounds half to even; above it
// the value is already an integer and is rebuilt from its significand.
// Non-finite inputs contribute 0 (their v.v makes vmax non-finite instead).
__device__ __forceinline__ __int128 quantise_2p60(double x) {
    const double s = __dmul_rn(x, 0x1p60);
    if (fabs(s) < 0x1p62) return (__int128)__double2ll_rn(s);
    const unsigned long long bits = (unsigned long long)__double_as_longlong(s);
    const int e = (int)((bits >> 52) & 0x7FF);
    if (e == 0x7FF) return 0;
    const unsigned long long m = (bits & ((1ull << 52) - 1)) | (1ull << 52);
    const int shift = e - 1075;  // >= 10 here
    const __int128 q = (shift < 74) ? ((__int128)m << shift) : (__int128)0;
    return (bits >> 63) ? -q : q;
}

struct NodeStats {
    __int128 s[3];
    unsigned long long vmax2;

    __device__ __forceinline__ void zero() {
        s[0] = s[1] = s[2] = 0;
        vmax2 = 0ull;
    }
    __device__ __forceinline__ void add_position(const Vec3& x) {
        s[0] += quantise_2p60(x.x);
        s[1] += quantise_2p60(x.y);
        s[2] += quantise_2p60(x.z);
    }
    __device__ __forceinline__ void add_velocity(const Vec3& v) {
        const unsigned long long b = (unsigned long long)__double_as_longlong(dot_self(v));
        vmax2 = b > vmax2 ? b : vmax2;
    }
};

__device__ __forceinline__ __int128 shfl_xor_i128(__int128 v, int m) {
    unsigned long long lo = (unsigned long long)v;
    unsigned long long hi = (unsigned long long)(v >> 64);
    lo = __shfl_xor_sync(0xffffffffu, lo, m);
    hi = __shfl_xor_sync(0xffffffffu, hi, m);
    return (__int128)(((unsigned __int128)hi << 64) | lo);
}

__device__ __forceinline__ void warp_reduce(NodeStats& st) {
#pragma unroll
    for (int m = 16; m > 0; m >>= 1) {
#pragma unroll
        for (int c = 0; c < 3; c++) st.s[c] += shfl_xor_i128(st.s[c], m);
        const unsigned long long o = __shfl_xor_sync(0xffffffffu, st.vmax2, m);
        st.vmax2 = o > st.vmax2 ? o : st.vmax2;
    }
}

// Exact 128-bit atomic accumulation from 64-bit atomics: the lo word wraps
// modulo 2^64 and the block whose addition wrapped it carries 1 into hi.
__device__ __forceinline__ void atomic_add_i128(unsigned long long* lo_word, unsigned long long* hi_word,
                                                __int128 v) {
    const unsigned long long lo = (unsigned long long)v;
    const unsigned long long hi = (unsigned long long)(v >> 64);
    if (lo) {
        const unsigned long long old = atomicAdd(lo_word, lo);
        const unsigned long long carry = (old + lo < old) ? 1ull : 0ull;
        if (hi + carry) atomicAdd(hi_word, hi + carry);
    } else if (hi) {
        atomicAdd(hi_word, hi);
    }
}

// Block-wide reduction of per-thread NodeStats into the step's accumulator.
// All threads of the block must call it. `scratch` holds >= nwarps entries.
struct WarpStats {
    unsigned long long lo[3], hi[3], vmax2, pad;
};

__device__ __forceinline__ void block_accumulate(NodeStats st, WarpStats* scratch, StatsAccum* acc) {
    warp_reduce(st);
    const int lane = threadIdx.x & 31;
    const int tid = threadIdx.x + blockDim.x * (threadIdx.y + blockDim.y * threadIdx.z);
    const int warp = tid >> 5;
    const int nwarps = (blockDim.x * blockDim.y * blockDim.z + 31) >> 5;
    if (lane == 0) {
        for (int c = 0; c < 3; c++) {
            scratch[warp].lo[c] = (unsigned long long)st.s[c];
            scratch[warp].hi[c] = (unsigned long long)(st.s[c] >> 64);
        }
        scratch[warp].vmax2 = st.vmax2;
    }
    __syncthreads();
    if (warp == 0) {
        NodeStats t;
        t.zero();
        if (lane < nwarps) {
            for (int c = 0; c < 3; c++)
                t.s[c] = (__int128)(((unsigned __int128)scratch[lane].hi[c] << 64) | scratch[lane].lo[c]);
            t.vmax2 = scratch[lane].vmax2;
        }
        warp_reduce(t);
        if (lane == 0) {
            for (int c = 0; c < 3; c++) atomic_add_i128(&acc->lo[c], &acc->hi[c], t.s[c]);
            if (t.vmax2) atomicMax(&acc->vmax2, t.vmax2);
        }
    }
}

}  // namespace paper
