// k_init_stats.cu -- K2 (initial state) and K3 (stats of a resident state).
//
// K2 generates every plane a chunk maps, halos included, from the global node
// index alone, so neighbouring chunks agree on their shared planes without an
// initial exchange. Reading S7: x = x0 + a*(2u-1) on interior
// nodes, u = (r >> 11) * 2^-53 with r the SplitMix64 output at counter 3g+c;
// x0 = (i - (n0-1)/2) * spacing; faces at x0; V = 0 (memset by the driver).
// Explicit _rn intrinsics: the same two roundings the CPU oracle performs.
#include "../kernels.hpp"
#include "node_math.cuh"
#include "stats.cuh"

namespace paper {

namespace {

constexpr int kBX = 32, kBY = 8;

// SplitMix64 (Steele, Lea, Flood 2014), counter form: the idx-th output of the
// stream seeded with `seed`.
__device__ __forceinline__ uint64_t splitmix64_at(uint64_t seed, uint64_t idx) {
    uint64_t z = seed + (idx + 1ull) * 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

__global__ void __launch_bounds__(kBX* kBY) init_kernel(InitArgs a) {
    const SlabGeom& g = a.g;
    const int64_t k = (int64_t)blockIdx.x * kBX + threadIdx.x;
    const int64_t j = (int64_t)blockIdx.y * kBY + threadIdx.y;
    const int64_t p = blockIdx.z;          // slab plane 0..size+1
    const int64_t i = g.start - 1 + p;     // global plane
    if (j >= g.n1 || k >= g.n2) return;
    const bool interior = i >= 1 && i < g.n0 - 1 && j >= 1 && j < g.n1 - 1 && k >= 1 && k < g.n2 - 1;
    const int64_t idx[3] = {i, j, k};
    const int64_t n[3] = {g.n0, g.n1, g.n2};
    const uint64_t gidx = (uint64_t)((i * g.n1 + j) * g.n2 + k);
    const int64_t off = p * g.plane_stride() + j * g.ld + k;
    for (int c = 0; c < 3; c++) {
        const double centre = (double)(n[c] - 1) / 2.0;  // exact (half-integer)
        const double x0 = __dmul_rn(__dsub_rn((double)idx[c], centre), a.spacing);
        double x = x0;
        if (interior) {
            const uint64_t r = splitmix64_at(a.seed, 3ull * gidx + (uint64_t)c);
            const double u = __dmul_rn((double)(r >> 11), 0x1p-53);
            const double s = __dsub_rn(__dmul_rn(2.0, u), 1.0);
            x = __dadd_rn(x0, __dmul_rn(a.amplitude, s));
        }
        a.x0[off + c * g.comp_stride()] = x;
        a.x1[off + c * g.comp_stride()] = x;
    }
}

__global__ void __launch_bounds__(kBX* kBY)
    stats_kernel(const double* __restrict__ x, const double* __restrict__ v, SlabGeom g, int64_t p0,
                 StatsAccum* acc, int k_interior_only) {
    __shared__ WarpStats scratch[kBX * kBY / 32];
    const int64_t k = (int64_t)blockIdx.x * kBX + threadIdx.x;
    const int64_t j = (int64_t)blockIdx.y * kBY + threadIdx.y;
    const int64_t p = p0 + blockIdx.z;
    NodeStats st;
    st.zero();
    unsigned long long xm = 0ull;  // max |x| bits (exact-stats domain bound)
    if (j < g.n1 && k < g.n2 && !(k_interior_only && (k == 0 || k == g.n2 - 1))) {
        const int64_t cs = g.comp_stride();
        const double* xp = x + p * g.plane_stride() + j * g.ld + k;
        st.add_position(Vec3{xp[0], xp[cs], xp[2 * cs]});
        xm = max(abs_bits(xp[0]), max(abs_bits(xp[cs]), abs_bits(xp[2 * cs])));
        if (v) {
            const double* vp = v + (p - 1) * g.plane_stride() + j * g.ld + k;
            st.add_velocity(Vec3{vp[0], vp[cs], vp[2 * cs]});
        }
    }
    block_accumulate(st, scratch, acc);
    warp_xmax(xm, acc);
}

// max |x| over the owned planes [p0, p0 + gridDim.z) of an X slab into
// acc->xmax: the exact-stats domain bound of a state the host-streamed mode
// maps in at the start of a run (its stats are not summed).
__global__ void __launch_bounds__(kBX* kBY) xmax_kernel(const double* __restrict__ x, SlabGeom g, int64_t p0,
                                                         StatsAccum* acc) {
    const int64_t k = (int64_t)blockIdx.x * kBX + threadIdx.x;
    const int64_t j = (int64_t)blockIdx.y * kBY + threadIdx.y;
    const int64_t p = p0 + blockIdx.z;
    unsigned long long xm = 0ull;
    if (j < g.n1 && k < g.n2) {
        const int64_t cs = g.comp_stride();
        const double* xp = x + p * g.plane_stride() + j * g.ld + k;
        xm = max(abs_bits(xp[0]), max(abs_bits(xp[cs]), abs_bits(xp[2 * cs])));
    }
    warp_xmax(xm, acc);
}

// Positions of the fixed k-face columns (k = 0 and k = n2-1, every j) of
// planes [p0, p0 + gridDim.y): the nodes K1_TB2's tiles do not own.
__global__ void __launch_bounds__(256) kface_stats_kernel(const double* __restrict__ x, SlabGeom g, int64_t p0,
                                                         StatsAccum* acc) {
    __shared__ WarpStats scratch[256 / 32];
    const int64_t j = (int64_t)blockIdx.x * 256 + threadIdx.x;
    const int64_t p = p0 + blockIdx.y;
    NodeStats st;
    st.zero();
    unsigned long long xm = 0ull;
    if (j < g.n1) {
        const int64_t cs = g.comp_stride();
        const double* xp = x + p * g.plane_stride() + j * g.ld;
        st.add_position(Vec3{xp[0], xp[cs], xp[2 * cs]});
        const int64_t k1 = g.n2 - 1;
        st.add_position(Vec3{xp[k1], xp[cs + k1], xp[2 * cs + k1]});
        xm = max(max(abs_bits(xp[0]), max(abs_bits(xp[cs]), abs_bits(xp[2 * cs]))),
                 max(abs_bits(xp[k1]), max(abs_bits(xp[cs + k1]), abs_bits(xp[2 * cs + k1]))));
    }
    block_accumulate(st, scratch, acc);
    warp_xmax(xm, acc);
}

}  // namespace

cudaError_t launch_kface_stats(const double* x_slab, const SlabGeom& g, int64_t p0, int64_t np, StatsAccum* acc,
                               cudaStream_t stream) {
    if (np <= 0) return cudaSuccess;
    dim3 grid((unsigned)((g.n1 + 255) / 256), (unsigned)np);
    kface_stats_kernel<<<grid, 256, 0, stream>>>(x_slab, g, p0, acc);
    return cudaGetLastError();
}

cudaError_t launch_xmax(const double* x_slab, const SlabGeom& g, int64_t p0, int64_t np, StatsAccum* acc,
                        cudaStream_t stream) {
    if (np <= 0) return cudaSuccess;
    dim3 block(kBX, kBY);
    dim3 grid((unsigned)((g.n2 + kBX - 1) / kBX), (unsigned)((g.n1 + kBY - 1) / kBY), (unsigned)np);
    xmax_kernel<<<grid, block, 0, stream>>>(x_slab, g, p0, acc);
    return cudaGetLastError();
}

cudaError_t launch_init(const InitArgs& a, cudaStream_t stream) {
    dim3 block(kBX, kBY);
    dim3 grid((unsigned)((a.g.n2 + kBX - 1) / kBX), (unsigned)((a.g.n1 + kBY - 1) / kBY), (unsigned)(a.g.size + 2));
    init_kernel<<<grid, block, 0, stream>>>(a);
    return cudaGetLastError();
}

cudaError_t launch_stats(const double* x_slab, const double* v_slab, const SlabGeom& g, int64_t p0, int64_t np,
                         StatsAccum* acc, cudaStream_t stream, bool k_interior_only) {
    if (np <= 0) return cudaSuccess;
    dim3 block(kBX, kBY);
    dim3 grid((unsigned)((g.n2 + kBX - 1) / kBX), (unsigned)((g.n1 + kBY - 1) / kBY), (unsigned)np);
    stats_kernel<<<grid, block, 0, stream>>>(x_slab, v_slab, g, p0, acc, k_interior_only ? 1 : 0);
    return cudaGetLastError();
}

namespace {
__global__ void delay_kernel(long long ns) {
    const long long t0 = clock64();
    const long long cycles = ns * 2;  // ~2 GHz SM clock: a lower bound on the delay
    while (clock64() - t0 < cycles) __nanosleep(1000);
}
}  // namespace

cudaError_t launch_delay(int64_t ns, cudaStream_t stream) {
    if (ns <= 0) return cudaSuccess;
    delay_kernel<<<1, 32, 0, stream>>>((long long)ns);
    return cudaGetLastError();
}

}  // namespace paper
