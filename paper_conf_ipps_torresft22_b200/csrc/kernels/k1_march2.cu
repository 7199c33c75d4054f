// k1_march2.cu -- SOMIER_K1_MARCH2: K1_MARCH with two rows per warp.
//
// Same arithmetic (node_math.cuh; bit-identical) and the same TMA ring, but a
// CTA owns a 32 (k) x 16 (j) tile and warp w handles the ADJACENT rows 2w and
// 2w+1. The -j spring of row 2w+1 is then the +j spring of row 2w, already in
// the thread's registers; only row 2w's -j crosses warps (shared memory). Per
// plane, the fixed costs -- mbarrier wait, CTA barrier, stage rotation, the
// tile-border springs, pointer updates -- are paid once per 64 node-updates
// per warp instead of 32, and the two rows' springs give each thread twice the
// independent fp64 work to hide latency with. K1 is energy-bound under the
// 1 kW cap, so fewer issued instructions per node is the lever.
#include <cuda.h>

#include <algorithm>

#include "../kernels.hpp"
#include "node_math.cuh"
#include "signal.cuh"
#include "stats.cuh"
#include "tma.cuh"

namespace paper {

namespace {

constexpr int kTK = 32;                 // tile width along k (one warp)
constexpr int kW = 8;                   // warps per CTA
constexpr int kTJ = 2 * kW;             // tile height along j: two rows per warp
constexpr int kThreads = kTK * kW;
constexpr int kBK = kTK + 4;            // X box columns k0-2 .. k0+33
constexpr int kBJ = kTJ + 2;            // X box rows j0-1 .. j0+16
constexpr int kCol0 = 2;
constexpr int kXBoxBytes = kBK * kBJ * 3 * 8;     // 15552
constexpr int kVBoxBytes = kTK * kTJ * 3 * 8;     // 12288
constexpr int kXSlot = 15616;                     // 128-byte aligned
// Two TMA rings: X (needed one plane ahead, by phase 1) and V (needed by
// phase 2 only). Measured at 512^3 (tools/variants.sh): X3+V3 5.95e10,
// X4+V2 5.82e10 (faster in burst, slower once the power cap engages), X5+V1
// 4.72e10 (V latency exposed). Two CTAs per SM must fit in 228 KB.
#ifndef K1M2_STAGES
#define K1M2_STAGES 3
#endif
#ifndef K1M2_VSTAGES
#define K1M2_VSTAGES 3
#endif
#ifndef K1M2_UNROLL
#define K1M2_UNROLL 1
#endif
constexpr int kM2Unroll = K1M2_UNROLL;  // plane-loop unroll (removes the loop-carried register moves)
constexpr int kStages = K1M2_STAGES;
constexpr int kVStages = K1M2_VSTAGES;
#ifndef K1M2_SEG
#define K1M2_SEG 64
#endif
constexpr int kSegPlanes = K1M2_SEG;    // planes per CTA segment along i
constexpr int kMinSegPlanes = 4;
constexpr int kXComp = kBJ * kBK, kVComp = kTJ * kTK;

struct __align__(16) Smem {
    unsigned char xst[kStages][kXSlot];
    unsigned char vst[kVStages][kVBoxBytes];
    Vec3 gj[2][kW][kTK];   // +j springs of each warp's second row, by plane parity
    Vec3 gbj[2][kTK];      // tile-border springs (j0-1 -> j0)
    Vec3 gbk[2][kTJ];      // tile-border springs (k0-1 -> k0), per row
    unsigned long long full[kStages];
    unsigned long long vfull[kVStages];
    WarpStats scratch[kThreads / 32];
};

struct March2Params {
    StepArgs a;
    int tiles_k;
    int tiles_j;
    int seg_planes;
};

__device__ __forceinline__ Vec3 shfl_up1(const Vec3& v) {
    return Vec3{__shfl_up_sync(0xffffffffu, v.x, 1), __shfl_up_sync(0xffffffffu, v.y, 1),
                __shfl_up_sync(0xffffffffu, v.z, 1)};
}

__device__ __forceinline__ Vec3 ld3(const double* p) { return Vec3{p[0], p[kXComp], p[2 * kXComp]}; }

#ifndef K1M2_HINTS
#define K1M2_HINTS 0  // bit 0: V loads evict-first, bit 1: output stores evict-first, bit 2: X loads evict-last
#endif

__device__ __forceinline__ void st_out(double* p, double v, uint64_t pol) {
    if (K1M2_HINTS & 2)
        st_hint(p, v, pol);
    else
        *p = v;
}

template <bool kUnitMass, bool kPosK, bool kFma>
__device__ __forceinline__ void update_node(bool interior, bool valid, bool write_fixed, const Vec3& F, const double* vb,
                                            const Vec3& xc, double* vo, double* xo, int64_t cs, double* lo_dst,
                                            double* hi_dst, int64_t off, const StepArgs& a, NodeStats& st,
                                            uint64_t pol) {
    if (interior) {
        Vec3 v{vb[0], vb[kVComp], vb[2 * kVComp]};
        Vec3 xn;
        kick_drift<kUnitMass, kFma>(F, a.M, a.dt, v, xc, xn);
        st_out(vo, v.x, pol);
        st_out(vo + cs, v.y, pol);
        st_out(vo + 2 * cs, v.z, pol);
        st_out(xo, xn.x, pol);
        st_out(xo + cs, xn.y, pol);
        st_out(xo + 2 * cs, xn.z, pol);
        if (lo_dst) {
            lo_dst[off] = xn.x;
            lo_dst[off + cs] = xn.y;
            lo_dst[off + 2 * cs] = xn.z;
        }
        if (hi_dst) {
            hi_dst[off] = xn.x;
            hi_dst[off + cs] = xn.y;
            hi_dst[off + 2 * cs] = xn.z;
        }
        st.add_position(xn);
        st.add_velocity(v);
    } else if (valid) {
        st.add_position(xc);
        if (write_fixed) {
            xo[0] = xc.x;
            xo[cs] = xc.y;
            xo[2 * cs] = xc.z;
        }
    }
}

template <bool kUnitMass, bool kPosK, bool kFma>
__global__ void __launch_bounds__(kThreads, 2)
    k1_march2_kernel(const __grid_constant__ CUtensorMap tmap_x, const __grid_constant__ CUtensorMap tmap_v,
                     const March2Params mp) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    Smem& sm = *reinterpret_cast<Smem*>(smem_raw);
    const StepArgs& a = mp.a;
    const SlabGeom& g = a.g;
    const int lane = threadIdx.x;
    const int w = threadIdx.y;
    const int tid = w * kTK + lane;
#ifndef K1M2_RASTER
#define K1M2_RASTER 0
#endif
    // CTA -> tile order (L2 reuse of the halo rows / columns between tiles that
    // run at the same time): 0 = k fastest, 1 = j fastest, G > 1 = bands of G
    // k-tiles walked down j
    int tile_k, tile_j;
    if (K1M2_RASTER == 0) {
        tile_k = blockIdx.x % mp.tiles_k;
        tile_j = blockIdx.x / mp.tiles_k;
    } else if (K1M2_RASTER == 1) {
        tile_j = blockIdx.x % mp.tiles_j;
        tile_k = blockIdx.x / mp.tiles_j;
    } else {
        const int G = K1M2_RASTER;
        const int band = blockIdx.x / (G * mp.tiles_j);
        const int gw = min(G, mp.tiles_k - band * G);
        const int r = blockIdx.x - band * G * mp.tiles_j;
        tile_k = band * G + r % gw;
        tile_j = r / gw;
    }
    const int k0 = tile_k * kTK, j0 = tile_j * kTJ;
    const int k = k0 + lane;
    const int jA = j0 + 2 * w, jB = jA + 1;
    const int ck = lane + kCol0;
    const int rA = 2 * w + 1;  // box row of row A (row B: rA + 1)
    const int pb = 1 + blockIdx.y * mp.seg_planes;
    const int pe = min((int)g.size + 1, pb + mp.seg_planes);
    const int q0 = pb - 1;
    const int qlast = pe;

    auto issue = [&](int q) {  // X of plane q
        const int s = (q - q0) % kStages;
        mbar_expect_tx(&sm.full[s], kXBoxBytes);
        if (K1M2_HINTS & 4)
            tma_load_4d_hint(sm.xst[s], &tmap_x, k0 - kCol0, j0 - 1, 0, q, &sm.full[s], policy_evict_last());
        else
            tma_load_4d(sm.xst[s], &tmap_x, k0 - kCol0, j0 - 1, 0, q, &sm.full[s]);
    };
    auto issue_v = [&](int p) {  // V of output plane p (V slab plane p-1)
        const int s = (p - pb) % kVStages;
        mbar_expect_tx(&sm.vfull[s], kVBoxBytes);
        if (K1M2_HINTS & 1)
            tma_load_4d_hint(sm.vst[s], &tmap_v, k0, j0, 0, p - 1, &sm.vfull[s], policy_evict_first());
        else
            tma_load_4d(sm.vst[s], &tmap_v, k0, j0, 0, p - 1, &sm.vfull[s]);
    };
    if (tid == 0) {
        prefetch_tmap(&tmap_x);
        prefetch_tmap(&tmap_v);
        for (int s = 0; s < kStages; s++) mbar_init(&sm.full[s], 1);
        for (int s = 0; s < kVStages; s++) mbar_init(&sm.vfull[s], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    // PDL: everything above overlapped the previous kernel on the stream; from
    // here on global memory is touched (it read the X buffer this step writes,
    // and wrote the X_t / V this step reads). A no-op without PDL.
    asm volatile("griddepcontrol.wait;" ::: "memory");
    const LaunchSlots slots = launch_slots(a, 1, blockIdx.x == 0 && blockIdx.y == 0, tid);
    // Every CTA is resident once all have passed this point, so the next
    // step's CTAs can only take slots freed by finished CTAs of this one.
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    if (tid == 0) {
        fence_proxy_async();
        for (int q = q0; q < q0 + kStages && q <= qlast; q++) issue(q);
        for (int p = pb; p < pb + kVStages && p < pe; p++) issue_v(p);
    }
    __syncthreads();

    const bool kin = k >= 1 && k < g.n2 - 1, kval = k < g.n2;
    const bool validA = kval && jA < g.n1, validB = kval && jB < g.n1;
    const bool intA = kin && jA >= 1 && jA < g.n1 - 1, intB = kin && jB >= 1 && jB < g.n1 - 1;
    const int64_t cs = g.comp_stride(), ps = g.plane_stride();
    const int64_t offA = (int64_t)jA * g.ld + k, offB = offA + g.ld;
    const int xA = rA * kBK + ck, xB = xA + kBK;
    const int vA = (2 * w) * kTK + lane, vB = vA + kTK;
    auto stage_x = [&](int s) { return reinterpret_cast<const double*>(sm.xst[s]); };

    // prologue: +i springs of plane pb-1 (the -i springs of plane pb)
    {
        const int s0 = 0, s1 = 1;
        mbar_wait(&sm.full[s0], 0);
        mbar_wait(&sm.full[s1], 0);
    }
    Vec3 carryA = spring_force<kPosK, kFma>(ld3(stage_x(0) + xA), ld3(stage_x(1) + xA), a.K, a.L);
    Vec3 carryB = spring_force<kPosK, kFma>(ld3(stage_x(0) + xB), ld3(stage_x(1) + xB), a.K, a.L);
    Vec3 xcA = ld3(stage_x(1) + xA), xcB = ld3(stage_x(1) + xB);
    __syncthreads();
    if (tid == 0 && q0 + kStages <= qlast) {
        fence_proxy_async();
        issue(q0 + kStages);
    }

    double* xo = a.x_nxt + (int64_t)pb * ps + offA;
    double* vo = a.v + (int64_t)(pb - 1) * ps + offA;
    int s_cur = 1, s_nxt = 2 % kStages;
    unsigned ph_nxt = (2 / kStages) & 1;
    const uint64_t pol_st = (K1M2_HINTS & 2) ? policy_evict_first() : 0;
    NodeStats st;
    st.zero();
#pragma unroll(kM2Unroll)
    for (int p = pb; p < pe; p++) {
        const int par = p & 1;
        mbar_wait(&sm.full[s_nxt], ph_nxt);
        const double* Xc = stage_x(s_cur);
        const double* Xn = stage_x(s_nxt);
        // ---- phase 1: "+" springs of both rows (+j of row A uses row B's position)
        const Vec3 gpkA = spring_force<kPosK, kFma>(xcA, ld3(Xc + xA + 1), a.K, a.L);
        const Vec3 gpkB = spring_force<kPosK, kFma>(xcB, ld3(Xc + xB + 1), a.K, a.L);
        const Vec3 gpjA = spring_force<kPosK, kFma>(xcA, xcB, a.K, a.L);
        const Vec3 gpjB = spring_force<kPosK, kFma>(xcB, ld3(Xc + xB + kBK), a.K, a.L);
        sm.gj[par][w][lane] = gpjB;
        const Vec3 niA = ld3(Xn + xA), niB = ld3(Xn + xB);
        const Vec3 gpiA = spring_force<kPosK, kFma>(xcA, niA, a.K, a.L);
        const Vec3 gpiB = spring_force<kPosK, kFma>(xcB, niB, a.K, a.L);
        if (w == 0) {
            sm.gbj[par][lane] = spring_force<kPosK, kFma>(ld3(Xc + ck), ld3(Xc + kBK + ck), a.K, a.L);
        } else if (w == 1 && lane < kTJ) {
            const double* b = Xc + (lane + 1) * kBK + kCol0;
            sm.gbk[par][lane] = spring_force<kPosK, kFma>(ld3(b - 1), ld3(b), a.K, a.L);
        }
        const Vec3 upA = shfl_up1(gpkA), upB = shfl_up1(gpkB);
        __syncthreads();
        // X stage of plane p and V slot of plane p-1 are free now
        if (tid == 0) {
            fence_proxy_async();
            if (p + kStages <= qlast) issue(p + kStages);
            if (p > pb && p - 1 + kVStages < pe) issue_v(p - 1 + kVStages);
        }
        // ---- phase 2
        const int vs = (p - pb) % kVStages;
        mbar_wait(&sm.vfull[vs], (unsigned)(((p - pb) / kVStages) & 1));
        const double* Vb = reinterpret_cast<const double*>(sm.vst[vs]);
        {
            const Vec3 gmj = neg(w == 0 ? sm.gbj[par][lane] : sm.gj[par][w - 1][lane]);
            const Vec3 gmk = neg(lane == 0 ? sm.gbk[par][2 * w] : upA);
            const Vec3 F = sum_forces(neg(carryA), gpiA, gmj, gpjA, gmk, gpkA);
            update_node<kUnitMass, kPosK, kFma>(intA, validA, a.write_fixed, F, Vb + vA, xcA, vo, xo, cs,
                                          (p == 1) ? a.lo_dst : nullptr, (p == g.size) ? a.hi_dst : nullptr, offA,
                                          a, st, pol_st);
        }
        {
            const Vec3 gmk = neg(lane == 0 ? sm.gbk[par][2 * w + 1] : upB);
            const Vec3 F = sum_forces(neg(carryB), gpiB, neg(gpjA), gpjB, gmk, gpkB);
            update_node<kUnitMass, kPosK, kFma>(intB, validB, a.write_fixed, F, Vb + vB, xcB, vo + g.ld, xo + g.ld, cs,
                                          (p == 1) ? a.lo_dst : nullptr, (p == g.size) ? a.hi_dst : nullptr, offB,
                                          a, st, pol_st);
        }
        carryA = gpiA;
        carryB = gpiB;
        xcA = niA;
        xcB = niB;
        xo += ps;
        vo += ps;
        s_cur = s_nxt;
        s_nxt = (s_nxt + 1 == kStages) ? 0 : s_nxt + 1;
        ph_nxt ^= (s_nxt == 0) ? 1u : 0u;
    }
    block_accumulate(st, sm.scratch, slots.fin);
    finish_launch(a, slots.t, 1, blockIdx.y == 0, blockIdx.y == gridDim.y - 1);
}

}  // namespace

cudaError_t launch_k1_march2(const StepArgs& a, bool unit_mass, cudaStream_t stream) {
    if (a.g.size <= 0) return cudaSuccess;
    if (!a.tmap_x_cur || !a.tmap_v2) return cudaErrorInvalidValue;
    March2Params mp;
    mp.a = a;
    mp.tiles_k = (int)((a.g.n2 + kTK - 1) / kTK);
    mp.tiles_j = (int)((a.g.n1 + kTJ - 1) / kTJ);
    const int tiles_j = (int)((a.g.n1 + kTJ - 1) / kTJ);
    const int tiles = mp.tiles_k * tiles_j;
#ifndef K1M2_WAVES
#define K1M2_WAVES 4
#endif
    const int want_ctas = K1M2_WAVES * 148 * 2;  // waves of 2 CTAs per SM
    int nseg = (int)((a.g.size + kSegPlanes - 1) / kSegPlanes);
    // Small grids (few tiles): if some segment count fits every CTA in ONE
    // wave of resident CTAs, take the one minimising (planes per segment + ~3
    // planes of fill / segment-start work); otherwise enough segments for
    // K1M2_WAVES waves (dynamic CTA scheduling then hides the tail). Measured
    // (tools/grid_ab.sh): 128^3 3.53e10 -> 4.03e10 node-updates/s; applying
    // the same cost model across waves at 256^3 was 0.6% slower.
    const int slots = 148 * 2;
    int one_wave = 0;
    double best = 1e300;
    for (int s = nseg; (int64_t)tiles * s <= slots && s <= (int)a.g.size; s++) {
        const int64_t seg = (a.g.size + s - 1) / s;
        if (seg < kMinSegPlanes) break;
        if ((double)(seg + 3) < best) {
            best = (double)(seg + 3);
            one_wave = s;
        }
    }
    if (one_wave > 0)
        nseg = one_wave;
    else
        nseg = std::max(nseg, std::min((int)a.g.size, (want_ctas + tiles - 1) / tiles));
    mp.seg_planes = (int)((a.g.size + nseg - 1) / nseg);
    if (mp.seg_planes < kMinSegPlanes) mp.seg_planes = (int)std::min<int64_t>(kMinSegPlanes, a.g.size);
    nseg = (int)((a.g.size + mp.seg_planes - 1) / mp.seg_planes);
    dim3 grid((unsigned)tiles, (unsigned)nseg);
    dim3 block(kTK, kW);
    mp.a.lo_ctas = mp.a.hi_ctas = grid.x;  // the first / last segment's CTAs
    const size_t smem = sizeof(Smem);
    const CUtensorMap& mx = *static_cast<const CUtensorMap*>(a.tmap_x2_cur);
    const CUtensorMap& mv = *static_cast<const CUtensorMap*>(a.tmap_v2);
    auto launch = [&](auto kernel) {
        cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = grid;
        cfg.blockDim = block;
        cfg.dynamicSmemBytes = smem;
        cfg.stream = stream;
        cudaLaunchAttribute attr[1];
        attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
        attr[0].val.programmaticStreamSerializationAllowed = 1;
        cfg.attrs = attr;
        cfg.numAttrs = a.pdl ? 1 : 0;
        cudaLaunchKernelEx(&cfg, kernel, mx, mv, mp);
    };
    const bool pos_k = a.K > 0.0;
    dispatch_bools([&](auto um, auto pk, auto fm) {
        launch(k1_march2_kernel<decltype(um)::value, decltype(pk)::value, decltype(fm)::value>);
    }, unit_mass, pos_k, a.fma != 0);
    return cudaGetLastError();
}

}  // namespace paper
