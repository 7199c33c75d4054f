// k1_march.cu -- SOMIER_K1_MARCH: the fast fused Somier step.
//
// Same arithmetic as K1_DIRECT (node_math.cuh; bit-identical), organised for
// the B200 memory system:
//   * a CTA owns a 32 (k) x 8 (j) column tile and MARCHES along i over a
//     segment of planes; one warp per row, one lane per k;
//   * TMA (cp.async.bulk.tensor, 4-D fp64 tensor maps) streams each plane's
//     X tile with its halo ring (a 36 x 10 x 3 box) and the matching
//     V tile into a kStages-deep shared-memory ring signalled by mbarriers;
//   * each spring is evaluated ONCE (bit-exact antisymmetry):
//     a node computes its +i, +j, +k springs; -i comes from the previous plane
//     (register carry), -k from lane-1 (warp shuffle), -j from row-1 (shared
//     memory). Only the tile-border springs (32 along j, 8 along k per plane)
//     are evaluated twice, by warps 0 and 1;
//   * forces -> accelerations -> velocities -> positions run in registers;
//     V and X_{t+1} are written once with coalesced 256-byte warp stores, and
//     boundary planes are also stored into the neighbour chunk's halo slot
//     (fused exchange, NVLink P2P / IPC when remote);
//   * the exact int128 centre sums and max v.v accumulate in registers for the
//     whole march and are reduced once per CTA.
// Algorithmic DRAM traffic: 24 B (X_t) + 24 B (V in) + 24 B (V out) + 24 B (X_{t+1})
// per interior node-update; the halo ring and the segment overlap re-read X
// planes from L2, not DRAM.
#include <cuda.h>

#include <algorithm>

#include "../kernels.hpp"
#include "node_math.cuh"
#include "signal.cuh"
#include "stats.cuh"

namespace paper {

namespace {

constexpr int kTK = 32;                 // tile width along k (one warp)
constexpr int kTJ = 8;                  // tile height along j (warps per CTA)
constexpr int kThreads = kTK * kTJ;
// X box with its halo ring: columns k0-2 .. k0+33 (the TMA box must start on a
// 16-byte boundary along the contiguous axis -- an odd fp64 start coordinate
// faults, measured with tools/tma_probe -- so the left halo is 2 columns wide,
// of which only k0-1 is used), rows j0-1 .. j0+8.
constexpr int kBK = kTK + 4;            // 36
constexpr int kBJ = kTJ + 2;            // 10
constexpr int kCol0 = 2;                // box column of k0
constexpr int kXBoxBytes = kBK * kBJ * 3 * 8;   // 8640
constexpr int kVBoxBytes = kTK * kTJ * 3 * 8;   // 6144
constexpr int kXSlot = 8704;                    // 128-byte aligned slots
constexpr int kStageBytes = kXSlot + kVBoxBytes;  // 14848
#ifndef K1_STAGES
#define K1_STAGES 4
#endif
#ifndef K1_SEG
#define K1_SEG 64
#endif
constexpr int kStages = K1_STAGES;              // TMA ring depth (planes)
constexpr int kSegPlanes = K1_SEG;              // max planes per CTA march (segment)
constexpr int kMinSegPlanes = 4;                // min planes per segment (small grids)

struct __align__(16) Smem {
    unsigned char stage[kStages][kStageBytes];
    Vec3 gj[2][kTJ][kTK];       // +j springs of each row, by plane parity
    Vec3 gbj[2][kTK];           // tile-border springs (j0-1 -> j0), per column
    Vec3 gbk[2][kTJ];           // tile-border springs (k0-1 -> k0), per row
    unsigned long long full[kStages];
    WarpStats scratch[kThreads / 32];
};

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(unsigned long long* bar, unsigned count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}

__device__ __forceinline__ void mbar_expect_tx(unsigned long long* bar, unsigned bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}

__device__ __forceinline__ void mbar_wait(unsigned long long* bar, unsigned parity) {
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra WAIT_%=;\n}" ::"r"(smem_u32(bar)),
        "r"(parity)
        : "memory");
}

__device__ __forceinline__ void tma_load_4d(void* dst, const CUtensorMap* map, int c0, int c1, int c2, int c3,
                                            unsigned long long* bar) {
    asm volatile(
        "cp.async.bulk.tensor.4d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
        " [%0], [%1, {%2, %3, %4, %5}], [%6];" ::"r"(smem_u32(dst)),
        "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(c2), "r"(c3), "r"(smem_u32(bar))
        : "memory");
}

struct MarchParams {
    StepArgs a;
    int tiles_k;
    int seg_planes;
};

__device__ __forceinline__ Vec3 shfl_up(const Vec3& v) {
    return Vec3{__shfl_up_sync(0xffffffffu, v.x, 1), __shfl_up_sync(0xffffffffu, v.y, 1),
                __shfl_up_sync(0xffffffffu, v.z, 1)};
}

// Occupancy / unroll knobs (tools/variants.sh). Measured on 512^3 (r01): 2 CTAs
// per SM (<= 128 registers, no spills) with the plane loop unrolled by 2 beats
// 3 CTAs per SM (80 registers, spills, index rematerialisation): under the
// 1 kW power cap the kernel is energy-bound, so fewer issued instructions win.
#ifndef K1_MIN_BLOCKS
#define K1_MIN_BLOCKS 2
#endif
#ifndef K1_UNROLL
#define K1_UNROLL 2
#endif
constexpr int kUnroll = K1_UNROLL;

template <bool kUnitMass, bool kPosK, bool kFma>
__global__ void __launch_bounds__(kThreads, K1_MIN_BLOCKS)
    k1_march_kernel(const __grid_constant__ CUtensorMap tmap_x, const __grid_constant__ CUtensorMap tmap_v,
                    const MarchParams mp) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    Smem& sm = *reinterpret_cast<Smem*>(smem_raw);
    const StepArgs& a = mp.a;
    const SlabGeom& g = a.g;
    const int lane = threadIdx.x;   // k within the tile
    const int w = threadIdx.y;      // j within the tile
    const int tid = w * kTK + lane;
    const int tile_k = blockIdx.x % mp.tiles_k;
    const int tile_j = blockIdx.x / mp.tiles_k;
    const int k0 = tile_k * kTK, j0 = tile_j * kTJ;
    const int k = k0 + lane, j = j0 + w;
    const int ck = lane + kCol0, rj = w + 1;  // the node's column / row in the X box
    // output planes [pb, pe) in slab numbering (owned planes are 1..size)
    const int pb = 1 + blockIdx.y * mp.seg_planes;
    const int pe = min((int)g.size + 1, pb + mp.seg_planes);
    const int q0 = pb - 1;  // first loaded plane
    const int qlast = pe;   // last loaded plane

    const LaunchSlots slots = launch_slots(a, 1, blockIdx.x == 0 && blockIdx.y == 0, tid);

    auto issue = [&](int q) {  // TMA for plane q into its stage (thread 0 only)
        const int s = (q - q0) % kStages;
        unsigned char* st = sm.stage[s];
        const bool with_v = q >= pb + 1;  // V of output plane q-1 rides with X(q)
        mbar_expect_tx(&sm.full[s], kXBoxBytes + (with_v ? kVBoxBytes : 0));
        tma_load_4d(st, &tmap_x, k0 - kCol0, j0 - 1, 0, q, &sm.full[s]);  // OOB -> zeros
        if (with_v) tma_load_4d(st + kXSlot, &tmap_v, k0, j0, 0, q - 2, &sm.full[s]);
    };
    auto wait = [&](int q) {
        const int s = (q - q0) % kStages;
        mbar_wait(&sm.full[s], (unsigned)(((q - q0) / kStages) & 1));
    };

    if (tid == 0) {
        asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmap_x)) : "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmap_v)) : "memory");
        for (int s = 0; s < kStages; s++) mbar_init(&sm.full[s], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        for (int q = q0; q < q0 + kStages && q <= qlast; q++) issue(q);
    }
    __syncthreads();

    const bool valid = j < g.n1 && k < g.n2;
    const bool interior = j >= 1 && j < g.n1 - 1 && k >= 1 && k < g.n2 - 1;
    const int64_t cs = g.comp_stride(), ps = g.plane_stride();
    const int64_t off = (int64_t)j * g.ld + k;
    // per-thread offsets (in doubles) inside a stage: own node of the X box, V box
    constexpr int kXComp = kBJ * kBK, kVComp = kTJ * kTK;
    const int xo_own = rj * kBK + ck;
    const int vo_own = w * kTK + lane;
    auto stage_x = [&](int s) { return reinterpret_cast<const double*>(smem_raw + s * kStageBytes); };
    auto ld3 = [&](const double* p) { return Vec3{p[0], p[kXComp], p[2 * kXComp]}; };

    // prologue: the -i spring of plane pb is the +i spring of plane pb-1 (negated)
    wait(q0);
    wait(pb);
    Vec3 carry = spring_force<kPosK, kFma>(ld3(stage_x(0) + xo_own), ld3(stage_x(1) + xo_own), a.K, a.L);
    Vec3 xc = ld3(stage_x(1) + xo_own);
    __syncthreads();
    if (tid == 0 && q0 + kStages <= qlast) {
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        issue(q0 + kStages);
    }

    double* xo = a.x_nxt + (int64_t)pb * ps + off;      // X_{t+1} of this node, plane pb
    double* vo = a.v + (int64_t)(pb - 1) * ps + off;    // V of this node, plane pb
    int s_cur = 1, s_nxt = 2 % kStages;                 // stages of planes p and p+1
    unsigned ph_nxt = (2 / kStages) & 1;                // mbarrier parity of plane p+1
    NodeStats st;
    st.zero();
#pragma unroll(kUnroll)
    for (int p = pb; p < pe; p++) {
        const int par = p & 1;
        mbar_wait(&sm.full[s_nxt], ph_nxt);
        const double* Xc = stage_x(s_cur);
        const double* Xn = stage_x(s_nxt);
        const double* me = Xc + xo_own;
        // ---- phase 1: the three "+" springs of every node, plus tile borders
        const Vec3 gpk = spring_force<kPosK, kFma>(xc, ld3(me + 1), a.K, a.L);
        const Vec3 xni = ld3(Xn + xo_own);
        const Vec3 gpi = spring_force<kPosK, kFma>(xc, xni, a.K, a.L);
        const Vec3 gpj = spring_force<kPosK, kFma>(xc, ld3(me + kBK), a.K, a.L);
        sm.gj[par][w][lane] = gpj;
        if (w == 0) {
            sm.gbj[par][lane] = spring_force<kPosK, kFma>(ld3(Xc + ck), ld3(Xc + kBK + ck), a.K, a.L);
        } else if (w == 1 && lane < kTJ) {
            const double* b = Xc + (lane + 1) * kBK + kCol0;
            sm.gbk[par][lane] = spring_force<kPosK, kFma>(ld3(b - 1), ld3(b), a.K, a.L);
        }
        const Vec3 up = shfl_up(gpk);
        __syncthreads();
        // stage of plane p is free: refill it with plane p + kStages
        if (tid == 0 && p + kStages <= qlast) {
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            issue(p + kStages);
        }
        // ---- phase 2: gather the "-" springs, sum, integrate, store
        const Vec3 gmi = neg(carry);
        const Vec3 gmj = neg(w == 0 ? sm.gbj[par][lane] : sm.gj[par][w - 1][lane]);
        const Vec3 gmk = neg(lane == 0 ? sm.gbk[par][w] : up);
        carry = gpi;
        if (interior) {
            const Vec3 F = sum_forces(gmi, gpi, gmj, gpj, gmk, gpk);
            const double* Vb = reinterpret_cast<const double*>(smem_raw + s_nxt * kStageBytes + kXSlot) + vo_own;
            Vec3 v{Vb[0], Vb[kVComp], Vb[2 * kVComp]};
            Vec3 xn;
            kick_drift<kUnitMass, kFma>(F, a.M, a.dt, v, xc, xn);
            vo[0] = v.x;
            vo[cs] = v.y;
            vo[2 * cs] = v.z;
            xo[0] = xn.x;
            xo[cs] = xn.y;
            xo[2 * cs] = xn.z;
            if (p == 1 && a.lo_dst) {
                a.lo_dst[off] = xn.x;
                a.lo_dst[off + cs] = xn.y;
                a.lo_dst[off + 2 * cs] = xn.z;
            }
            if (p == g.size && a.hi_dst) {
                a.hi_dst[off] = xn.x;
                a.hi_dst[off + cs] = xn.y;
                a.hi_dst[off + 2 * cs] = xn.z;
            }
            st.add_position(xn);
            st.add_velocity(v);
        } else if (valid) {
            st.add_position(xc);  // fixed face node: X_{t+1} == X_t, V == 0
            if (a.write_fixed) {
                xo[0] = xc.x;
                xo[cs] = xc.y;
                xo[2 * cs] = xc.z;
            }
        }
        xc = xni;
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

cudaError_t launch_k1_march(const StepArgs& a, bool unit_mass, cudaStream_t stream) {
    if (a.g.size <= 0) return cudaSuccess;
    if (!a.tmap_x_cur || !a.tmap_v) return cudaErrorInvalidValue;
    MarchParams mp;
    mp.a = a;
    mp.tiles_k = (int)((a.g.n2 + kTK - 1) / kTK);
    const int tiles_j = (int)((a.g.n1 + kTJ - 1) / kTJ);
    // Segments of <= kSegPlanes planes; on small grids shorter segments so that
    // the grid still holds ~4 waves of CTAs (148 SMs x 2 CTAs): each segment
    // costs one extra plane of X (L2) and one pipeline fill.
    const int tiles = mp.tiles_k * tiles_j;
    const int want_ctas = 4 * 148 * K1_MIN_BLOCKS;
    int nseg = (int)((a.g.size + kSegPlanes - 1) / kSegPlanes);
    nseg = std::max(nseg, std::min((int)a.g.size, (want_ctas + tiles - 1) / tiles));
    mp.seg_planes = (int)((a.g.size + nseg - 1) / nseg);
    if (mp.seg_planes < kMinSegPlanes) mp.seg_planes = (int)std::min<int64_t>(kMinSegPlanes, a.g.size);
    nseg = (int)((a.g.size + mp.seg_planes - 1) / mp.seg_planes);
    dim3 grid((unsigned)(mp.tiles_k * tiles_j), (unsigned)nseg);
    dim3 block(kTK, kTJ);
    mp.a.lo_ctas = mp.a.hi_ctas = grid.x;  // the first / last segment's CTAs
    const size_t smem = sizeof(Smem);
    const CUtensorMap& mx = *static_cast<const CUtensorMap*>(a.tmap_x_cur);
    const CUtensorMap& mv = *static_cast<const CUtensorMap*>(a.tmap_v);
    auto launch = [&](auto kernel) {
        cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        kernel<<<grid, block, smem, stream>>>(mx, mv, mp);
    };
    const bool pos_k = a.K > 0.0;
    dispatch_bools([&](auto um, auto pk, auto fm) {
        launch(k1_march_kernel<decltype(um)::value, decltype(pk)::value, decltype(fm)::value>);
    }, unit_mass, pos_k, a.fma != 0);
    return cudaGetLastError();
}

}  // namespace paper
