// stats.cuh -- the "centers" reduction fused into the step
// kernels: the exact sum over nodes of q(x) = round_half_even(x * 2^60) for
// each coordinate (reading S15: order-independent, so every launch
// configuration and chunk partition gives the same bits) and the max of v.v.
//
// Per thread the exact sum is carried in fp64 registers without any integer
// work (the integer-heavy int128 path made K1 issue-bound, profiles/r01_v1):
//   y = x * 2^28                      exact (power-of-two scale)
//   h = (y + C) - C,  C = 1.5 * 2^52  = round_half_even(y), an integer, |y| < 2^51
//   r = y - h                         exact, |r| <= 1/2
//   l = fma(r, 2^32, C) - C           = round_half_even(r * 2^32), an integer
// Since h * 2^32 is an even integer, q(x) = h * 2^32 + l exactly. The sums of
// h and of l stay exact in fp64 while they are below 2^53: |x| < 2^18 (checked
// by somier_init) and at most kMaxNodesPerThread nodes per thread give
// |sum h| < 2^46 * 128 and |sum l| < 2^31 * 128. The block reduction converts
// to int128 once; the device accumulator adds int128 with 64-bit atomics.
#pragma once
#include <cstdint>

#include "../stats_layout.hpp"
#include "node_math.cuh"

namespace paper {

constexpr int kMaxNodesPerThread = 128;  // STATS_FP64_ACC variant only
constexpr double kRoundC = 6755399441055744.0;  // 1.5 * 2^52
constexpr double kRoundK0 = kRoundC * 0x1p32 + kRoundC;  // 1.5 * 2^84 + 1.5 * 2^52, exact (34 significant bits)

// The two words of q(x) = round_half_even(x 2^60) = h 2^32 + l as C + h and
// C + l (|x| < 2^18), three fp64 operations; see NodeStats below.
__device__ __forceinline__ void split_q(double x, double& hd, double& ld) {
    hd = __fma_rn(x, 0x1p28, kRoundC);
    ld = __fma_rn(x, 0x1p60, __fma_rn(-hd, 0x1p32, kRoundK0));
}

#ifndef STATS_FP64_ACC
// Per thread, the exact sums are carried as the BIT PATTERNS of the rounded
// doubles (fp64 work: 3 operations per coordinate, the accumulation on the
// integer pipe):
//   hd = fma(x, 2^28, C)                   = C + h, h = round_half_even(x 2^28), |h| < 2^51
//   b  = fma(-hd, 2^32, C 2^32 + C)        = C - h 2^32 exactly (a multiple of 2^32 below 2^79
//                                            in magnitude: 47 significant bits)
//   ld = fma(x, 2^60, b)                   = RN(C + r 2^32), r = x 2^28 - h (|r| <= 1/2)
//                                          = C + l, l = round_half_even(r 2^32)
// (the same two words as the 4-operation form r = fma(x, 2^28, -(hd - C)),
// ld = fma(r, 2^32, C): one rounding of the same exact value).
// C + m with |m| < 2^51 lies in [2^52, 2^53), where one unit of the mantissa
// is 1, so bits(C + m) = bits(C) + m: sum h = sum bits(hd) - n bits(C) and
// sum l = sum bits(ld) - n bits(C), computed modulo 2^64, which is exact while
// the true sums stay below 2^63 in magnitude: |h| < 2^46 for |x| < 2^18, so up
// to 2^17 nodes per thread (K1_TB2: at most 2 rows x 256 planes = 512).
// q(x) = h 2^32 + l as in the fp64 form below. Adding x = 0 adds exactly
// bits(C) to both words and 1 to n: a neutral element.
struct NodeStats {
    unsigned long long hb[3], lb[3];
    unsigned int n;  // nodes added (positions)
    double vmax2;    // NaN-sticky max of v.v

    __device__ __forceinline__ void zero() {
        hb[0] = hb[1] = hb[2] = 0ull;
        lb[0] = lb[1] = lb[2] = 0ull;
        n = 0u;
        vmax2 = 0.0;
    }
    __device__ __forceinline__ void add_coord(int c, double x) {
        double hd, ld;
        split_q(x, hd, ld);
        hb[c] += (unsigned long long)__double_as_longlong(hd);
        lb[c] += (unsigned long long)__double_as_longlong(ld);
    }
    __device__ __forceinline__ void add_position(const Vec3& x) {
        add_coord(0, x.x);
        add_coord(1, x.y);
        add_coord(2, x.z);
        n++;
    }
    // a position whose node is counted by another NodeStats over the same node
    // set (K1_TB2's two steps): set n from that one before sum()
    __device__ __forceinline__ void add_position_nc(const Vec3& x) {
        add_coord(0, x.x);
        add_coord(1, x.y);
        add_coord(2, x.z);
    }
    __device__ __forceinline__ void copy_count(const NodeStats& o) { n = o.n; }
    __device__ __forceinline__ void add_velocity(const Vec3& v) {
        const double v2 = dot_self(v);
        vmax2 = (v2 > vmax2 || v2 != v2) ? v2 : vmax2;
    }
    // exact int128 value of sum q(x) for coordinate c
    __device__ __forceinline__ __int128 sum(int c) const {
        const unsigned long long cb = (unsigned long long)__double_as_longlong(kRoundC) * n;
        const long long h = (long long)(hb[c] - cb), l = (long long)(lb[c] - cb);
        return (__int128)h * ((__int128)1 << 32) + (__int128)l;
    }
    __device__ __forceinline__ unsigned long long vmax2_bits() const {
        return (unsigned long long)__double_as_longlong(vmax2);
    }
};
#else
struct NodeStats {
    double h[3], l[3];
    double vmax2;  // NaN-sticky max of v.v

    __device__ __forceinline__ void zero() {
        h[0] = h[1] = h[2] = 0.0;
        l[0] = l[1] = l[2] = 0.0;
        vmax2 = 0.0;
    }
    __device__ __forceinline__ void add_coord(int c, double x) {
        // fma with an exact power-of-two product == the unfused sequence above
        const double hh = __dsub_rn(__fma_rn(x, 0x1p28, kRoundC), kRoundC);
        const double r = __fma_rn(x, 0x1p28, -hh);
        const double ll = __dsub_rn(__fma_rn(r, 0x1p32, kRoundC), kRoundC);
        h[c] = __dadd_rn(h[c], hh);
        l[c] = __dadd_rn(l[c], ll);
    }
    __device__ __forceinline__ void add_position(const Vec3& x) {
        add_coord(0, x.x);
        add_coord(1, x.y);
        add_coord(2, x.z);
    }
    __device__ __forceinline__ void add_position_nc(const Vec3& x) { add_position(x); }
    __device__ __forceinline__ void copy_count(const NodeStats&) {}
    __device__ __forceinline__ void add_velocity(const Vec3& v) {
        const double v2 = dot_self(v);
        vmax2 = (v2 > vmax2 || v2 != v2) ? v2 : vmax2;
    }
    // exact int128 value of sum q(x) for coordinate c
    __device__ __forceinline__ __int128 sum(int c) const {
        return (__int128)__double2ll_rn(h[c]) * ((__int128)1 << 32) + (__int128)__double2ll_rn(l[c]);
    }
    __device__ __forceinline__ unsigned long long vmax2_bits() const {
        return (unsigned long long)__double_as_longlong(vmax2);
    }
};

#endif

// The stats slots of one launch that advances `nsteps` (1 or 2) steps. With a
// step word (resident handles, stats_layout.hpp) the step number t comes from
// device memory -- written by the previous launch's last CTA, read after any
// griddepcontrol.wait -- and the slots from the ring: states t+1 (mid) and
// t+nsteps (fin); block 0 zeroes the slots of states t+nsteps+1, t+nsteps+2.
// Without one the explicit a.acc / a.acc_mid / a.acc_clear are used.
struct LaunchSlots {
    StatsAccum* fin;
    StatsAccum* mid;
    unsigned long long t;
};

template <class Args>
__device__ __forceinline__ LaunchSlots launch_slots(const Args& a, int nsteps, bool block0, int tid) {
    LaunchSlots s;
    if (a.step_word) {
        unsigned long long t;
        asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(t) : "l"(a.step_word) : "memory");
        s.t = t;
        s.fin = a.acc_ring + ring_slot(t + nsteps);
        s.mid = a.acc_ring + ring_slot(t + 1);
        if (block0 && tid < 16) {
            StatsAccum* c = a.acc_ring + ring_slot(t + nsteps + 1 + (tid >> 3));
            reinterpret_cast<unsigned long long*>(c)[tid & 7] = 0ull;
        }
    } else {
        s.t = 0;
        s.fin = a.acc;
        s.mid = a.acc_mid;
        if (a.acc_clear && block0 && tid < 8) reinterpret_cast<unsigned long long*>(a.acc_clear)[tid] = 0ull;
    }
    return s;
}

struct I128Stats {
    __int128 s[3];
    unsigned long long vmax2;
};

__device__ __forceinline__ __int128 shfl_xor_i128(__int128 v, int m) {
    unsigned long long lo = (unsigned long long)v;
    unsigned long long hi = (unsigned long long)(v >> 64);
    lo = __shfl_xor_sync(0xffffffffu, lo, m);
    hi = __shfl_xor_sync(0xffffffffu, hi, m);
    return (__int128)(((unsigned __int128)hi << 64) | lo);
}

__device__ __forceinline__ void warp_reduce(I128Stats& st) {
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

// max |x| of the nodes a warp's threads hold (IEEE bits of |x|: non-negative
// doubles order as unsigned integers, NaN above inf) into acc->xmax -- the
// exact-stats domain bound of a state the stats kernels sum (stats_layout.hpp).
// All 32 lanes of the warp must call it.
__device__ __forceinline__ unsigned long long abs_bits(double x) {
    return (unsigned long long)__double_as_longlong(fabs(x));
}
__device__ __forceinline__ void warp_xmax(unsigned long long b, StatsAccum* acc) {
#pragma unroll
    for (int m = 16; m > 0; m >>= 1) {
        const unsigned long long o = __shfl_xor_sync(0xffffffffu, b, m);
        b = o > b ? o : b;
    }
    const int tid = threadIdx.x + blockDim.x * (threadIdx.y + blockDim.y * threadIdx.z);
    if ((tid & 31) == 0 && b) atomicMax(&acc->xmax, b);
}

struct WarpStats {
    unsigned long long lo[3], hi[3], vmax2, pad;
};

// Block-wide reduction of per-thread NodeStats into the step's accumulator.
// All threads of the block must call it. `scratch` holds >= nwarps entries.
__device__ __forceinline__ void block_accumulate(const NodeStats& ns, WarpStats* scratch, StatsAccum* acc) {
    I128Stats st;
    for (int c = 0; c < 3; c++) st.s[c] = ns.sum(c);
    st.vmax2 = ns.vmax2_bits();
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
        I128Stats t;
        t.s[0] = t.s[1] = t.s[2] = 0;
        t.vmax2 = 0ull;
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
