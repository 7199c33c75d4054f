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

// Call once per CTA, by all threads, after the CTA's last store. The last CTA
// of the launch to finish advances the step word (stats ring, t = the step the
// launch started from) and publishes the neighbours' flags.
__device__ __forceinline__ void finish_launch(const StepArgs& a, unsigned long long t, int nsteps) {
    const bool sig = a.signal_lo || a.signal_hi;
    if (!sig && !a.step_word) return;
    __shared__ unsigned int s_last;
    __syncthreads();
    const bool leader = threadIdx.x == 0 && threadIdx.y == 0 && threadIdx.z == 0;
    if (leader) {
        if (sig) __threadfence_system();
        const unsigned int nblocks = gridDim.x * gridDim.y * gridDim.z;
        const unsigned int prev = atomicAdd(a.done_counter, 1u);
        s_last = (prev == nblocks - 1) ? 1u : 0u;
    }
    __syncthreads();
    if (leader && s_last) {
        if (sig) __threadfence_system();
        *a.done_counter = 0u;  // self-reset for the next step (stream-ordered)
        if (a.step_word) *a.step_word = t + (unsigned long long)nsteps;
        if (a.signal_lo) st_release_sys_u64(a.signal_lo, a.signal_value);
        if (a.signal_hi) st_release_sys_u64(a.signal_hi, a.signal_value);
    }
}

}  // namespace paper
