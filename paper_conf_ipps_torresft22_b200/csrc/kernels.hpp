// kernels.hpp -- launch wrappers of the sm_100a kernels (host-callable).
//
// Slab layout of one chunk: positions X are two buffers (t and
// t+1) of (size+2) planes, plane p <-> global i = start-1+p (planes 0 and
// size+1 are the halo planes of the map A[start-1 : size+2]);
// velocities V are `size` planes, plane p <-> global i = start+p. A plane is
// three component-planar n1 x ld blocks (x, then y, then z), each row
// ld >= n2 doubles (ld a multiple of 32: 256-byte aligned rows).
#pragma once
#include <type_traits>
#include <cstdint>

#include <cuda_runtime.h>

#include "stats_layout.hpp"

namespace paper {

struct SlabGeom {
    int64_t n0, n1, n2;  // global grid
    int64_t ld;          // row pitch in doubles
    int64_t start;       // global i of the first owned plane (omp_spread_start)
    int64_t size;        // owned planes (omp_spread_size)

    __host__ __device__ int64_t comp_stride() const { return n1 * ld; }
    __host__ __device__ int64_t plane_stride() const { return 3 * n1 * ld; }
};

struct StepArgs {
    const double* x_cur;    // X_t slab (size+2 planes)
    double* x_nxt;          // X_{t+1} slab (size+2 planes)
    double* v;              // V slab (size planes), updated in place
    double* lo_dst;         // left neighbour's hi-halo plane in ITS X_{t+1} buffer, or null
    double* hi_dst;         // right neighbour's lo-halo plane in ITS X_{t+1} buffer, or null
    SlabGeom g;
    double K, L, M, dt;
    StatsAccum* acc;        // this step's stats slot (accumulated); K1_TB2: the last step's
    StatsAccum* acc_clear;  // the next step's slot (zeroed by block 0)
    StatsAccum* acc_mid;    // K1_TB2 two-step launch: stats of the intermediate state t+1 (or null)
    // Resident handles: per-step stats history (stats_layout.hpp). When
    // step_word is non-null the launch reads the step number t from it, takes
    // its slots in acc_ring (acc / acc_mid / acc_clear are ignored), and its last
    // CTA advances *step_word by the steps it computed -- so a CUDA graph of
    // launches needs no per-step arguments.
    unsigned long long* step_word;
    StatsAccum* acc_ring;
    // Completion signal for neighbours on other streams (fused exchange): the
    // last CTA stores `signal_value` with release semantics at system scope
    // into each non-null flag after every CTA's halo stores are fenced.
    unsigned long long* signal_lo;   // left neighbour's "from_right" flag
    unsigned long long* signal_hi;   // right neighbour's "from_left" flag
    unsigned long long signal_value;
    unsigned int* done_counter;      // per-chunk CTA completion counter (self-resetting)
    // Early neighbour signals: the flag to a neighbour is published when the
    // CTAs whose work touches that side (they store the boundary planes into
    // its halo, or read this chunk's halo planes it will overwrite next) are
    // done, not the whole grid. side_counter[0] / [1] count them (self-
    // resetting); lo_ctas / hi_ctas are set by the launcher from its grid.
    unsigned int* side_counter;
    unsigned int lo_ctas, hi_ctas;
    // K1_MARCH: host pointers to the CUtensorMaps of x_cur and v (passed to the
    // kernel by value as __grid_constant__ parameters).
    const void* tmap_x_cur;
    const void* tmap_v;
    // K1_MARCH2 (32 x 16 tiles): the same slabs with its box shapes
    const void* tmap_x2_cur;
    const void* tmap_v2;
    // Host-streamed mode: x_nxt is a fresh buffer, so fixed face nodes of the
    // owned planes are copied into it too (resident mode leaves them in place).
    int write_fixed;
    // SOMIER_MATH_FMA: the step's arithmetic with the FMA contractions of
    // node_math.cuh (kFma); 0 = uncontracted (the oracle's operation order).
    int fma;
    // K1_MARCH2: launch with programmatic stream serialization (PDL): the
    // kernel's prologue (barrier init, tensor-map prefetch) overlaps the tail
    // of the previous kernel on the stream; every thread executes
    // griddepcontrol.wait before touching global memory.
    int pdl;
};

struct InitArgs {
    double* x0;  // both X buffers, all size+2 planes
    double* x1;
    SlabGeom g;
    double spacing, amplitude;
    uint64_t seed;
};

// Host-side: calls f(std::integral_constant<bool, b>...) so that launchers
// turn runtime flags into kernel template arguments without spelling out
// every combination.
template <class F>
inline void dispatch_bools(F&& f) { f(); }
template <class F, class... B>
inline void dispatch_bools(F&& f, bool b0, B... rest) {
    if (b0)
        dispatch_bools([&](auto... v) { f(std::true_type{}, v...); }, rest...);
    else
        dispatch_bools([&](auto... v) { f(std::false_type{}, v...); }, rest...);
}

enum class K1Variant { Direct = 1, March = 2, March2 = 3 };

// K1_TB2: warps per CTA; the CTA's ring-extended tile is 32 x (2 * kTB2Warps)
// and its TMA boxes are 34 x (2 * kTB2Warps + 2) (X) and 34 x (2 * kTB2Warps) (V).
#ifndef TB2_WARPS
#define TB2_WARPS 12
#endif
constexpr int kTB2Warps = TB2_WARPS;

cudaError_t launch_k1(K1Variant variant, const StepArgs& a, bool unit_mass, cudaStream_t stream);

// K1_TB2 slab layout (deep halo): X slabs hold planes [start-2, start+size+2)
// (two halo planes per face), V slabs [start-1, start+size+1) (one), both
// double-buffered; the launch reads X_t, V_t through a.tmap_x_cur / a.tmap_v
// (box shapes kTB2*Box*) and writes the owned planes of X_{t+2}, V_{t+2} (one
// step: X_{t+1}, V_{t+1}) to x_out / v_out, plus the first two X planes and
// the first V plane to the left neighbour's halo (a.lo_dst = ITS out-buffer X
// plane of global i = start, lo_vdst = its V plane of i = start) and the last
// two / last one to the right neighbour's (a.hi_dst = its X plane of i =
// start+size-2, hi_vdst = its V plane of i = start+size-1); a.signal_* /
// a.done_counter / a.signal_value as for the one-step kernels. Stats of both
// steps: the ring (a.step_word) or a.acc_mid (state t+1) and a.acc (last state).
struct Tb2Out {
    double* x_out;
    double* v_out;
    double* lo_vdst;
    double* hi_vdst;
    bool two;  // two steps (else one)
    // global planes [stats_lo, stats_hi) whose nodes enter the stats (both 0:
    // the launch's own planes [start, start+size)); a widened launch of a
    // host-streamed trip counts only the chunk it maps out
    int64_t stats_lo, stats_hi;
};
cudaError_t launch_k1_tb2(const StepArgs& a, const Tb2Out& o, bool unit_mass, cudaStream_t stream);
cudaError_t launch_init(const InitArgs& a, cudaStream_t stream);
// max |x| over planes [p0, p0+np) of an X slab (plane index inside the slab)
// into acc->xmax (atomicMax of the IEEE bits): the exact-stats domain bound
// of a mapped-in state (stats_layout.hpp, xbound_step)
cudaError_t launch_xmax(const double* x_slab, const SlabGeom& g, int64_t p0, int64_t np, StatsAccum* acc,
                        cudaStream_t stream);
// Test hook (somier_stream_set_delay): one CTA that spins ~ns nanoseconds on the
// stream, emulating a slower device.
cudaError_t launch_delay(int64_t ns, cudaStream_t stream);
// Stats of planes [p0, p0+np) of an X slab (plane index inside the slab) and,
// if v != null, of V planes [p0-1, ...) (V has no halo planes).
// k_interior_only: skip the k-face columns (k = 0, n2-1).
cudaError_t launch_stats(const double* x_slab, const double* v_slab, const SlabGeom& g, int64_t p0, int64_t np,
                         StatsAccum* acc, cudaStream_t stream, bool k_interior_only = false);
// Positions of the k-face columns (k = 0, n2-1) of X slab planes [p0, p0+np):
// K1_TB2 tiles the interior k columns only, so these constant nodes go to the
// static stats slot.
cudaError_t launch_kface_stats(const double* x_slab, const SlabGeom& g, int64_t p0, int64_t np, StatsAccum* acc,
                               cudaStream_t stream);

}  // namespace paper
