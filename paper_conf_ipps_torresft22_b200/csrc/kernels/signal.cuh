// signal.cuh -- completion signal of the fused halo exchange. Every CTA that
// stored into a neighbour's halo fences at system scope; the last CTA of the
// launch to finish publishes the step number to the neighbours' flags with a
// release store. The neighbour's stream waits on the flag (cuStreamWaitValue64,
// no SM spinning) before its next step, which both makes the halo visible (RAW)
// and proves this step no longer reads the neighbour's halo buffer (WAR).
#pragma once
#include "../kernels.hpp"

namespace paper {

__device__ __forceinline__ void st_release_sys_u64(unsigned long long* p, unsigned long long v) {
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// Call once per CTA, by all threads, after the CTA's last store. lo_side /
// hi_side: this CTA's work touches that neighbour (see StepArgs). The last
// lo-side (hi-side) CTA to finish publishes the left (right) neighbour's flag
// -- the neighbour's next launch needs only those CTAs done, so it can start
// while this launch's interior CTAs still run. The last CTA of the whole grid
// advances the step word (stats ring; t = the step the launch started from).
__device__ __forceinline__ void finish_launch(const StepArgs& a, unsigned long long t, int nsteps, bool lo_side,
                                              bool hi_side) {
    const bool sig_lo = a.signal_lo && lo_side, sig_hi = a.signal_hi && hi_side;
    if (!a.signal_lo && !a.signal_hi && !a.step_word) return;
    __syncthreads();  // every thread's stores precede the leader's fence
    const bool leader = threadIdx.x == 0 && threadIdx.y == 0 && threadIdx.z == 0;
    if (!leader) return;
    if (sig_lo || sig_hi) __threadfence_system();
    if (sig_lo && atomicAdd(&a.side_counter[0], 1u) == a.lo_ctas - 1) {
        __threadfence_system();
        a.side_counter[0] = 0u;  // self-reset for the next launch (stream-ordered)
        st_release_sys_u64(a.signal_lo, a.signal_value);
    }
    if (sig_hi && atomicAdd(&a.side_counter[1], 1u) == a.hi_ctas - 1) {
        __threadfence_system();
        a.side_counter[1] = 0u;
        st_release_sys_u64(a.signal_hi, a.signal_value);
    }
    if (a.step_word) {
        const unsigned int nblocks = gridDim.x * gridDim.y * gridDim.z;
        __threadfence();  // this CTA's stats atomics (block_accumulate, same thread) before its count
        if (atomicAdd(a.done_counter, 1u) == nblocks - 1) {
            __threadfence();
            *a.done_counter = 0u;
            // exact-stats domain bound of the states this launch produced
            // (stats_layout.hpp): from the previous state's bound and each
            // step's vmax, now complete
            volatile StatsAccum* r = a.acc_ring;
            double B = __longlong_as_double((long long)r[ring_slot(t)].xmax);
            for (int s = 1; s <= nsteps; s++) {
                volatile StatsAccum* q = r + ring_slot(t + (unsigned long long)s);
                B = xbound_step(B, __longlong_as_double((long long)q->vmax2), a.dt);
                q->xmax = (unsigned long long)__double_as_longlong(B);
            }
            *a.step_word = t + (unsigned long long)nsteps;
        }
    }
}

}  // namespace paper
