// k1_tb2.cu -- SOMIER_K1_TB2: TWO time steps per pass over HBM (2.5-D
// temporal blocking), for a chunk without neighbour chunks (one slab per
// device, no halo exchange).
//
// Why: K1 is energy-bound under the 1 kW cap and the HBM traffic is ~3/4 of
// its energy (tools/power_probe.py). Doing steps t and t+1 in
// one pass halves the bytes per node-update (96 B -> 48 B) at the price of
// recomputing step t on a one-node ring around each tile.
//
// Layout of the work: a CTA = 16 warps x 32 lanes = the ring-extended region
// R1 (32 k x 16 j) of an owned tile R2 (30 k x 14 j, lanes 1..30, rows
// 1..14). Marching along i, iteration p does
//   step t   on plane p   for all of R1  (X_t from a TMA ring, V_t from a TMA
//            ring; X_{t+1} of R1 kept in shared memory, V_{t+1} in registers)
//   step t+1 on plane p-1 for R2          (neighbours all inside R1)
// and writes X_{t+2}, V_{t+2} of R2 to the OTHER X / V buffers (X and V are
// double-buffered here because neighbouring tiles read X_t / V_t of this
// tile's ring). Both steps use node_math.cuh, so every node update is the same
// IEEE expression as in K1_DIRECT / K1_MARCH (bit-identical), and the stats
// of BOTH steps are accumulated (step t into acc1, step t+1 into acc).
#include <cuda.h>

#include <algorithm>

#include "../kernels.hpp"
#include "node_math.cuh"
#include "stats.cuh"
#include "tma.cuh"

namespace paper {

namespace {

constexpr int kTK = 32, kW = 16, kThreads = kTK * kW;
constexpr int kOK = kTK - 2, kOJ = kW - 2;                  // owned tile 30 x 14
constexpr int kBK = kTK + 2, kBJ = kW + 2;                  // X_t box: R1 + ring (34 x 18)
constexpr int kXComp = kBK * kBJ;
constexpr int kXBoxBytes = kXComp * 3 * 8;                  // 14688
constexpr int kXSlot = 14720;
constexpr int kVBK = kTK + 2, kVBJ = kW;                    // V_t box: R1 (+1 col for alignment) 34 x 16
constexpr int kVComp = kVBK * kVBJ;
constexpr int kVBoxBytes = kVComp * 3 * 8;                  // 13056
constexpr int kYComp = kTK * kW;                            // X_{t+1} of R1: 32 x 16
#ifndef TB2_STAGES
#define TB2_STAGES 3
#endif
#ifndef TB2_VSTAGES
#define TB2_VSTAGES 3
#endif
constexpr int kStages = TB2_STAGES, kVStages = TB2_VSTAGES;
constexpr int kSegPlanes = 64, kMinSegPlanes = 4;

struct __align__(16) Smem {
    unsigned char xst[kStages][kXSlot];
    unsigned char vst[kVStages][kVBoxBytes];
    double y[2][3][kYComp];        // X_{t+1} of R1, two planes
    Vec3 gj1[2][kW][kTK];          // step t: +j springs by plane parity
    Vec3 gj2[2][kW][kTK];          // step t+1
    Vec3 gbj[2][kTK];              // step t tile-border springs (row above R1)
    Vec3 gbk[2][kW];               // step t tile-border springs (column left of R1)
    unsigned long long full[kStages];
    unsigned long long vfull[kVStages];
    WarpStats scratch[kThreads / 32];
};

struct Tb2Params {
    StepArgs a;
    double* x_out;                 // X_{t+2} buffer
    double* v_out;                 // V_{t+2} buffer
    StatsAccum* acc1;              // stats of step t (X_{t+1})
    int tiles_k, tiles_j, seg_planes;
};

__device__ __forceinline__ Vec3 shfl_up1(const Vec3& v) {
    return Vec3{__shfl_up_sync(0xffffffffu, v.x, 1), __shfl_up_sync(0xffffffffu, v.y, 1),
                __shfl_up_sync(0xffffffffu, v.z, 1)};
}

template <bool kUnitMass, bool kPosK>
__global__ void __launch_bounds__(kThreads, 1)
    k1_tb2_kernel(const __grid_constant__ CUtensorMap tmap_x, const __grid_constant__ CUtensorMap tmap_v,
                  const Tb2Params tp) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    Smem& sm = *reinterpret_cast<Smem*>(smem_raw);
    const StepArgs& a = tp.a;
    const SlabGeom& g = a.g;
    const int lane = threadIdx.x, w = threadIdx.y, tid = w * kTK + lane;
    const int tile_k = blockIdx.x % tp.tiles_k, tile_j = blockIdx.x / tp.tiles_k;
    const int kq = tile_k * kOK, jq = tile_j * kOJ;  // owned tile origin
    const int k = kq - 1 + lane, j = jq - 1 + w;     // this thread's R1 node
    const int size = (int)g.size;
    const int pb = 1 + blockIdx.y * tp.seg_planes;
    const int pe = min(size + 1, pb + tp.seg_planes);  // step-(t+1) outputs [pb, pe)
    const int p_first = max(0, pb - 1);                // step-t planes [p_first, pe]
    const int q0 = max(0, p_first - 1);                // X_t planes [q0, qlast]
    const int qlast = min(size + 1, pe + 1);
    const int v_first = max(1, p_first), v_last = min(size, pe);  // V_t planes read

    auto issue_x = [&](int q) {
        const int s = (q - q0) % kStages;
        mbar_expect_tx(&sm.full[s], kXBoxBytes);
        tma_load_4d(sm.xst[s], &tmap_x, kq - 2, jq - 2, 0, q, &sm.full[s]);
    };
    auto issue_v = [&](int p) {  // V_t of slab plane p (V slab plane p-1)
        const int s = (p - v_first) % kVStages;
        mbar_expect_tx(&sm.vfull[s], kVBoxBytes);
        tma_load_4d(sm.vst[s], &tmap_v, kq - 2, jq - 1, 0, p - 1, &sm.vfull[s]);
    };
    if (tid == 0) {
        prefetch_tmap(&tmap_x);
        prefetch_tmap(&tmap_v);
        for (int s = 0; s < kStages; s++) mbar_init(&sm.full[s], 1);
        for (int s = 0; s < kVStages; s++) mbar_init(&sm.vfull[s], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        fence_proxy_async();
        for (int q = q0; q < q0 + kStages && q <= qlast; q++) issue_x(q);
        for (int p = v_first; p < v_first + kVStages && p <= v_last; p++) issue_v(p);
    }
    __syncthreads();

    auto xbox = [&](int q) { return reinterpret_cast<const double*>(sm.xst[(q - q0) % kStages]); };
    auto xwait = [&](int q) { mbar_wait(&sm.full[(q - q0) % kStages], (unsigned)(((q - q0) / kStages) & 1)); };
    const int xo_own = (w + 1) * kBK + (lane + 1);
    auto ldx = [&](const double* b, int off) { return Vec3{b[off], b[off + kXComp], b[off + 2 * kXComp]}; };

    const bool valid = k >= 0 && k < g.n2 && j >= 0 && j < g.n1;
    const bool interior = k >= 1 && k < g.n2 - 1 && j >= 1 && j < g.n1 - 1;
    const bool owned = valid && lane >= 1 && lane <= kOK && w >= 1 && w <= kOJ;
    const int64_t cs = g.comp_stride(), ps = g.plane_stride();
    const int64_t off = owned ? (int64_t)j * g.ld + k : 0;

    // prologue: X_t(p_first) own, and the step-t -i spring of plane p_first
    Vec3 carry1{0.0, 0.0, 0.0}, xc1;
    xwait(p_first);
    xc1 = ldx(xbox(p_first), xo_own);
    if (p_first >= 1) {
        xwait(p_first - 1);
        carry1 = spring_force<kPosK>(ldx(xbox(p_first - 1), xo_own), xc1, a.K, a.L);
    }
    Vec3 carry2{0.0, 0.0, 0.0};
    Vec3 vhold{0.0, 0.0, 0.0};
    NodeStats st1, st2;
    st1.zero();
    st2.zero();
    __syncthreads();
    if (tid == 0 && p_first >= 1 && q0 + kStages <= qlast) {
        fence_proxy_async();
        issue_x(q0 + kStages);  // X_t(p_first - 1) is no longer needed
    }

    for (int p = p_first; p <= pe; p++) {
        const int par = p & 1;
        const bool upd1 = p >= 1 && p <= size;  // step t updates plane p
        const bool has_next = p + 1 <= qlast;
        if (has_next) xwait(p + 1);
        const double* Xc = xbox(p);
        const double* Xn = has_next ? xbox(p + 1) : Xc;
        // ---- step t, phase A: "+" springs
        Vec3 gpi1{0.0, 0.0, 0.0}, gpj1{0.0, 0.0, 0.0}, gpk1{0.0, 0.0, 0.0};
        const Vec3 xn1 = ldx(Xn, xo_own);
        if (has_next) gpi1 = spring_force<kPosK>(xc1, xn1, a.K, a.L);
        if (upd1) {
            gpk1 = spring_force<kPosK>(xc1, ldx(Xc, xo_own + 1), a.K, a.L);
            gpj1 = spring_force<kPosK>(xc1, ldx(Xc, xo_own + kBK), a.K, a.L);
            sm.gj1[par][w][lane] = gpj1;
            if (w == 0) {
                sm.gbj[par][lane] = spring_force<kPosK>(ldx(Xc, lane + 1), ldx(Xc, kBK + lane + 1), a.K, a.L);
            } else if (w == 1 && lane < kW) {
                const int r = (lane + 1) * kBK;
                sm.gbk[par][lane] = spring_force<kPosK>(ldx(Xc, r), ldx(Xc, r + 1), a.K, a.L);
            }
        }
        const Vec3 up1 = shfl_up1(gpk1);
        __syncthreads();  // A: X_t(p) is read for the last time above
        if (tid == 0 && p + kStages <= qlast) {
            fence_proxy_async();
            issue_x(p + kStages);
        }
        // ---- step t, phase B: forces -> V_{t+1}, X_{t+1} of R1 plane p
        Vec3 x1 = xc1, v1{0.0, 0.0, 0.0};
        if (upd1) {
            const int vs = (p - v_first) % kVStages;
            mbar_wait(&sm.vfull[vs], (unsigned)(((p - v_first) / kVStages) & 1));
            if (interior) {
                const Vec3 gmj = neg(w == 0 ? sm.gbj[par][lane] : sm.gj1[par][w - 1][lane]);
                const Vec3 gmk = neg(lane == 0 ? sm.gbk[par][w] : up1);
                const Vec3 F = sum_forces(neg(carry1), gpi1, gmj, gpj1, gmk, gpk1);
                const double* vb = reinterpret_cast<const double*>(sm.vst[vs]) + w * kVBK + (lane + 1);
                v1 = Vec3{vb[0], vb[kVComp], vb[2 * kVComp]};
                kick_drift<kUnitMass>(F, a.M, a.dt, v1, xc1, x1);
            }
            if (owned && p >= pb && p < pe) {
                st1.add_position(x1);
                if (interior) st1.add_velocity(v1);
            }
        }
        sm.y[par][0][tid] = x1.x;
        sm.y[par][1][tid] = x1.y;
        sm.y[par][2][tid] = x1.z;
        carry1 = gpi1;
        xc1 = xn1;
        __syncthreads();  // B: X_{t+1}(p) visible; V_t(p) slot free
        if (tid == 0 && upd1 && p + kVStages <= v_last) {
            fence_proxy_async();
            issue_v(p + kVStages);
        }
        // ---- step t+1 on plane q = p-1, phase C: "+" springs inside R1
        const int q = p - 1;
        Vec3 gpi2{0.0, 0.0, 0.0}, gpj2{0.0, 0.0, 0.0}, gpk2{0.0, 0.0, 0.0};
        const bool do_c = q >= pb - 1 && q >= 0;
        const bool out2 = q >= pb && q < pe;
        Vec3 x2c{0.0, 0.0, 0.0};
        if (do_c) {
            const double* yq = sm.y[q & 1][0];
            const double* yp = sm.y[par][0];
            x2c = Vec3{yq[tid], yq[tid + kYComp], yq[tid + 2 * kYComp]};
            gpi2 = spring_force<kPosK>(x2c, Vec3{yp[tid], yp[tid + kYComp], yp[tid + 2 * kYComp]}, a.K, a.L);
            if (out2) {
                const int tk = lane < kTK - 1 ? tid + 1 : tid;
                const int tj = w < kW - 1 ? tid + kTK : tid;
                gpk2 = spring_force<kPosK>(x2c, Vec3{yq[tk], yq[tk + kYComp], yq[tk + 2 * kYComp]}, a.K, a.L);
                gpj2 = spring_force<kPosK>(x2c, Vec3{yq[tj], yq[tj + kYComp], yq[tj + 2 * kYComp]}, a.K, a.L);
                sm.gj2[par][w][lane] = gpj2;
            }
        }
        const Vec3 up2 = shfl_up1(gpk2);
        __syncthreads();  // C
        // ---- step t+1, phase D: update R2 nodes of plane q, write X_{t+2}, V_{t+2}
        if (out2 && owned) {
            if (interior) {
                const Vec3 gmj = neg(sm.gj2[par][w - 1][lane]);
                const Vec3 F = sum_forces(neg(carry2), gpi2, gmj, gpj2, neg(up2), gpk2);
                Vec3 v2 = vhold, x2;
                kick_drift<kUnitMass>(F, a.M, a.dt, v2, x2c, x2);
                double* xo = tp.x_out + (int64_t)q * ps + off;
                double* vo = tp.v_out + (int64_t)(q - 1) * ps + off;
                xo[0] = x2.x;
                xo[cs] = x2.y;
                xo[2 * cs] = x2.z;
                vo[0] = v2.x;
                vo[cs] = v2.y;
                vo[2 * cs] = v2.z;
                st2.add_position(x2);
                st2.add_velocity(v2);
            } else {
                st2.add_position(x2c);  // fixed face node
            }
        }
        if (do_c) carry2 = gpi2;
        vhold = v1;
    }
    block_accumulate(st1, sm.scratch, tp.acc1);
    __syncthreads();
    block_accumulate(st2, sm.scratch, a.acc);
}

}  // namespace

cudaError_t launch_k1_tb2(const StepArgs& a, double* x_out, double* v_out, StatsAccum* acc1, bool unit_mass,
                          cudaStream_t stream) {
    if (a.g.size <= 0) return cudaSuccess;
    if (!a.tmap_x_cur || !a.tmap_v || a.lo_dst || a.hi_dst) return cudaErrorInvalidValue;
    Tb2Params tp;
    tp.a = a;
    tp.x_out = x_out;
    tp.v_out = v_out;
    tp.acc1 = acc1;
    tp.tiles_k = (int)((a.g.n2 + kOK - 1) / kOK);
    tp.tiles_j = (int)((a.g.n1 + kOJ - 1) / kOJ);
    const int tiles = tp.tiles_k * tp.tiles_j;
    const int want_ctas = 4 * 148;
    int nseg = (int)((a.g.size + kSegPlanes - 1) / kSegPlanes);
    nseg = std::max(nseg, std::min((int)a.g.size, (want_ctas + tiles - 1) / tiles));
    tp.seg_planes = (int)((a.g.size + nseg - 1) / nseg);
    if (tp.seg_planes < kMinSegPlanes) tp.seg_planes = (int)std::min<int64_t>(kMinSegPlanes, a.g.size);
    nseg = (int)((a.g.size + tp.seg_planes - 1) / tp.seg_planes);
    dim3 grid((unsigned)tiles, (unsigned)nseg), block(kTK, kW);
    const size_t smem = sizeof(Smem);
    const CUtensorMap& mx = *static_cast<const CUtensorMap*>(a.tmap_x_cur);
    const CUtensorMap& mv = *static_cast<const CUtensorMap*>(a.tmap_v);
    auto launch = [&](auto kernel) {
        cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        kernel<<<grid, block, smem, stream>>>(mx, mv, tp);
    };
    const bool pos_k = a.K > 0.0;
    if (unit_mass)
        pos_k ? launch(k1_tb2_kernel<true, true>) : launch(k1_tb2_kernel<true, false>);
    else
        pos_k ? launch(k1_tb2_kernel<false, true>) : launch(k1_tb2_kernel<false, false>);
    return cudaGetLastError();
}

}  // namespace paper
