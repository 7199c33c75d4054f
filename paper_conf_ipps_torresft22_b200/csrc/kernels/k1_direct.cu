// k1_direct.cu -- SOMIER_K1_DIRECT: the fused Somier step, one thread per node.
// Each interior node loads its 6 neighbours (L1/L2 serve the reuse), evaluates
// the 6 springs, and runs forces -> accelerations -> velocities -> positions
// -> centers in registers. The simple, obviously
// correct CUDA path; K1_MARCH is the fast one. Both are bit-identical.
#include "../kernels.hpp"
#include "node_math.cuh"
#include "signal.cuh"
#include "stats.cuh"

namespace paper {

namespace {

constexpr int kBX = 32, kBY = 8;

template <bool kUnitMass, bool kFma>
__global__ void __launch_bounds__(kBX* kBY) k1_direct_kernel(StepArgs a) {
    __shared__ WarpStats scratch[kBX * kBY / 32];
    const SlabGeom& g = a.g;
    const int64_t k = (int64_t)blockIdx.x * kBX + threadIdx.x;
    const int64_t j = (int64_t)blockIdx.y * kBY + threadIdx.y;
    const int64_t p = blockIdx.z;  // owned plane 0..size-1 -> X slab plane p+1
    const LaunchSlots slots = launch_slots(a, 1, blockIdx.x == 0 && blockIdx.y == 0 && blockIdx.z == 0,
                                           threadIdx.y * kBX + threadIdx.x);

    NodeStats st;
    st.zero();
    if (j < g.n1 && k < g.n2) {
        const int64_t cs = g.comp_stride(), ps = g.plane_stride();
        const int64_t off = j * g.ld + k;
        const double* xc = a.x_cur + (p + 1) * ps + off;
        const Vec3 xp{xc[0], xc[cs], xc[2 * cs]};
        const bool interior = j >= 1 && j < g.n1 - 1 && k >= 1 && k < g.n2 - 1;
        if (interior) {
            auto ld3 = [&](const double* q) { return Vec3{q[0], q[cs], q[2 * cs]}; };
            const Vec3 gmi = spring_force<false, kFma>(xp, ld3(xc - ps), a.K, a.L);
            const Vec3 gpi = spring_force<false, kFma>(xp, ld3(xc + ps), a.K, a.L);
            const Vec3 gmj = spring_force<false, kFma>(xp, ld3(xc - g.ld), a.K, a.L);
            const Vec3 gpj = spring_force<false, kFma>(xp, ld3(xc + g.ld), a.K, a.L);
            const Vec3 gmk = spring_force<false, kFma>(xp, ld3(xc - 1), a.K, a.L);
            const Vec3 gpk = spring_force<false, kFma>(xp, ld3(xc + 1), a.K, a.L);
            const Vec3 F = sum_forces(gmi, gpi, gmj, gpj, gmk, gpk);
            double* vp = a.v + p * ps + off;
            Vec3 v{vp[0], vp[cs], vp[2 * cs]};
            Vec3 xn;
            kick_drift<kUnitMass, kFma>(F, a.M, a.dt, v, xp, xn);
            vp[0] = v.x;
            vp[cs] = v.y;
            vp[2 * cs] = v.z;
            double* xo = a.x_nxt + (p + 1) * ps + off;
            xo[0] = xn.x;
            xo[cs] = xn.y;
            xo[2 * cs] = xn.z;
            if (p == 0 && a.lo_dst) {
                a.lo_dst[off] = xn.x;
                a.lo_dst[off + cs] = xn.y;
                a.lo_dst[off + 2 * cs] = xn.z;
            }
            if (p == g.size - 1 && a.hi_dst) {
                a.hi_dst[off] = xn.x;
                a.hi_dst[off + cs] = xn.y;
                a.hi_dst[off + 2 * cs] = xn.z;
            }
            st.add_position(xn);
            st.add_velocity(v);
        } else {
            st.add_position(xp);  // fixed node: X_{t+1} == X_t, V == 0
            if (a.write_fixed) {
                double* xo = a.x_nxt + (p + 1) * g.plane_stride() + off;
                xo[0] = xp.x;
                xo[g.comp_stride()] = xp.y;
                xo[2 * g.comp_stride()] = xp.z;
            }
        }
    }
    block_accumulate(st, scratch, slots.fin);
    finish_launch(a, slots.t, 1, blockIdx.z == 0, blockIdx.z == gridDim.z - 1);
}

}  // namespace

cudaError_t launch_k1_direct(const StepArgs& a, bool unit_mass, cudaStream_t stream) {
    if (a.g.size <= 0) return cudaSuccess;
    dim3 block(kBX, kBY);
    dim3 grid((unsigned)((a.g.n2 + kBX - 1) / kBX), (unsigned)((a.g.n1 + kBY - 1) / kBY), (unsigned)a.g.size);
    StepArgs b = a;
    b.lo_ctas = b.hi_ctas = grid.x * grid.y;  // one plane per grid z: the first / last plane's CTAs
    auto* kern = unit_mass ? (a.fma ? k1_direct_kernel<true, true> : k1_direct_kernel<true, false>)
                           : (a.fma ? k1_direct_kernel<false, true> : k1_direct_kernel<false, false>);
    kern<<<grid, block, 0, stream>>>(b);
    return cudaGetLastError();
}

}  // namespace paper
