// k1_tb2.cu -- SOMIER_K1_TB2: TWO time steps per pass over HBM (2.5-D
// temporal blocking), for a chunk without neighbour chunks (one slab per
// device, no halo exchange).
//
// Why: K1 is energy-bound under the 1 kW cap and HBM traffic is most of its
// energy (tools/power_probe.py). Doing steps t and t+1 in one
// pass halves the bytes per node-update (96 B -> 48 B) at the price of
// recomputing step t on a one-node ring around each tile.
//
// Layout of the work (v2): a CTA = kTB2Warps warps; warp w owns the two
// ADJACENT rows 2w, 2w+1 of the ring-extended region R1 (32 k x 2*kTB2Warps j)
// of an owned tile R2 (lanes 1..30, rows 1..2*kTB2Warps-2). Marching along i,
// iteration p does
//   S1: step t   on plane p   for all of R1  (X_t from a TMA ring, V_t from a
//       TMA ring; X_{t+1} of R1 goes to a two-plane shared-memory ring, V_{t+1}
//       stays in registers for one iteration)
//   S2: step t+1 on plane p-1 for R2         (neighbours all inside R1)
// and writes X_{t+2}, V_{t+2} of R2 to the OTHER X / V buffers (X and V are
// double-buffered here because neighbouring tiles read X_t / V_t of this
// tile's ring). As in K1_MARCH2 each spring is evaluated once per step (+i, +j,
// +k per node; -i from a register carry, -k from a lane shuffle, -j from the
// paired row or shared memory), two CTA barriers per plane. Both steps use
// node_math.cuh, so every node update is the same IEEE expression as in
// K1_DIRECT / K1_MARCH2 (bit-identical). The stats ("centers", PAPER.md:330,
// 354) of BOTH steps are accumulated over the owned nodes of the output planes:
// step t+1's from S2's results, step t's from the S1 results S2 reads anyway
// (X_{t+1} of plane q from the shared ring, V_{t+1} from the register carry).
#include <cuda.h>

#include <algorithm>
#include <climits>
#include <cmath>
#include <cstdlib>
#include <type_traits>

#include "../kernels.hpp"
#include "node_math.cuh"
#include "signal.cuh"
#include "stats.cuh"
#include "tma.cuh"

namespace paper {

namespace {

constexpr int kTK = 32, kW = kTB2Warps, kThreads = kTK * kW;
constexpr int kRows = 2 * kW;                               // R1 rows
constexpr int kOK = kTK - 2, kOJ = kRows - 2;               // owned tile R2
// Tiles cover the INTERIOR k columns [1, n2-2] (30 per tile: 512^3 = 17
// tiles exactly); the fixed k-face columns are ring nodes of the edge tiles
// and their (constant) stats are precomputed into the static stats slot. A
// tile's first owned column kq = 1 + 30 t is odd, so the X box starts at
// kq - 3 (an fp64 box must start on an even column): box column = R1 lane + 2.
constexpr int kBK = kTK + 4, kBJ = kRows + 2;               // X_t box: R1 + ring (+1 alignment column each side)
constexpr int kXComp = kBK * kBJ;
constexpr int kXBoxBytes = kXComp * 3 * 8;
constexpr int kXSlot = (kXBoxBytes + 127) / 128 * 128;
constexpr int kVBK = kTK + 2, kVBJ = kRows;                 // V_t box: R1 from kq - 3 (R1 lane l: column l + 2)
constexpr int kVComp = kVBK * kVBJ;
constexpr int kVBoxBytes = kVComp * 3 * 8;
constexpr int kVSlot = (kVBoxBytes + 127) / 128 * 128;
constexpr int kYComp = kRows * kTK;                         // X_{t+1} of one R1 plane, per component
#ifndef TB2_STAGES
#define TB2_STAGES 3
#endif
#ifndef TB2_VSTAGES
#define TB2_VSTAGES 2
#endif
constexpr int kStages = TB2_STAGES, kVStages = TB2_VSTAGES;
// Step t+1's stats are accumulated in S1 right after its kick-drift, into
// thread-private shared-memory slots (measured fastest of the placements,
// DESIGN.md §6). TB2_MID_STATS=0 skips them -- an A/B of their cost only (the
// stats of every second step, round 1's kernel), not a product configuration.
#ifndef TB2_MID_STATS
#define TB2_MID_STATS 1
#endif
constexpr int kMinSegPlanes = 4, kMaxSegPlanes = 256;
static_assert(kRows <= 32, "the -k border springs are computed by one warp, one row per lane");

struct __align__(16) Smem {
    unsigned char xst[kStages][kXSlot];
    unsigned char vst[kVStages][kVSlot];
    double y[2][3][kYComp];        // X_{t+1} of R1, planes by parity
    Vec3 g1j[kW][kTK];             // S1: +j spring of each warp's second row
    Vec3 g2j[kW][kTK];             // S2: same
    Vec3 gbj[kTK];                 // S1 tile-border springs (row above R1 -> R1 row 0)
    Vec3 gbk[kRows];               // S1 tile-border springs (column left of R1 -> R1 lane 0)
    unsigned long long full[kStages];
    unsigned long long vfull[kVStages];
    WarpStats scratch[kW];
    // step t+1's stats accumulators, thread-private (registers are full):
    // [0..2] = sum bits(hd) of x, y, z; [3..5] = sum bits(ld); [6] = max v.v
    unsigned long long acc1[7][kThreads];
};

struct Tb2Params {
    StepArgs a;                    // a.x_cur / a.v: X_t, V_t slabs (through the tensor maps); a.lo_dst /
                                   // a.hi_dst: the neighbours' X halo planes (see below)
    double* x_out;                 // X_{t+2} (X_{t+1} in one-step mode) buffer, raw slab
    double* v_out;                 // V_{t+2} buffer, raw slab
    double* lo_vdst;               // left neighbour's V halo plane in ITS out buffer, or null
    double* hi_vdst;               // right neighbour's V halo plane in ITS out buffer, or null
    int x_base, v_base;            // global i of raw plane 0 of the X / V slabs (start - 2, start - 1)
    int lo_end, hi_begin;          // planes q < lo_end go to lo_dst + (q - start), q >= hi_begin to hi_dst + (q - hi_begin)
    int stats_lo, stats_hi;        // output planes [stats_lo, stats_hi) contribute to the stats
    int64_t cs, ps;                // component / plane stride in doubles (precomputed: the kernel
                                   // reads them from the parameter bank instead of re-multiplying)
    int tiles_k, tiles_j, seg_planes;
};

__device__ __forceinline__ Vec3 shfl_up1(const Vec3& v) {
    return Vec3{__shfl_up_sync(0xffffffffu, v.x, 1), __shfl_up_sync(0xffffffffu, v.y, 1),
                __shfl_up_sync(0xffffffffu, v.z, 1)};
}

__device__ __forceinline__ void stb3(double* p, int64_t cs, const Vec3& v) {
    p[0] = v.x;
    p[cs] = v.y;
    p[2 * cs] = v.z;
}

__device__ __forceinline__ Vec3 ldb(const double* b, int off, int comp) {
    return Vec3{b[off], b[off + comp], b[off + 2 * comp]};
}


// kTwo: two steps per launch (else one: S1 only, its X_{t+1}, V_{t+1} written
// for R2 -- the odd step of a TB2 handle, with the same halo layout).
template <bool kUnitMass, bool kPosK, bool kTwo, bool kFma>
__global__ void __launch_bounds__(kThreads, 1)
    k1_tb2_kernel(const __grid_constant__ CUtensorMap tmap_x, const __grid_constant__ CUtensorMap tmap_v,
                  const Tb2Params tp) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    Smem& sm = *reinterpret_cast<Smem*>(smem_raw);
    const StepArgs& a = tp.a;
    const SlabGeom& g = a.g;
    const int lane = threadIdx.x, w = threadIdx.y, tid = w * kTK + lane;
    const int tile_k = blockIdx.x % tp.tiles_k, tile_j = blockIdx.x / tp.tiles_k;
    const int kq = 1 + tile_k * kOK, jq = tile_j * kOJ;  // owned tile origin (interior k columns)
    const int rA = 2 * w, rB = rA + 1;               // R1 rows of this thread
    const int k = kq - 1 + lane, jA = jq - 1 + rA, jB = jA + 1;
    // planes are global i; the chunk owns [start, start + size), its X slab
    // holds [start - 2, start + size + 2), its V slab [start - 1, start + size + 1)
    const int start = (int)g.start, size = (int)g.size, ilast = (int)g.n0 - 2;  // updated planes: [1, ilast]
    const int pb = start + blockIdx.y * tp.seg_planes;
    const int pe = min(start + size, pb + tp.seg_planes);  // S2 (step t+1) output planes [pb, pe)
    const int ps0 = pb - 1;                                // S1 (step t) planes [ps0, pe]
    const int q0 = max(0, ps0 - 1);                        // X_t planes [q0, qlast]
    const int qlast = min(ilast + 1, pe + 1);
    const int v_first = max(1, ps0), v_last = min(ilast, pe);  // V_t planes read (S1 on non-fixed planes)
    const LaunchSlots slots = launch_slots(a, kTwo ? 2 : 1, blockIdx.x == 0 && blockIdx.y == 0, tid);

    auto issue_x = [&](int q) {
        const int s = (q - q0) % kStages;
        mbar_expect_tx(&sm.full[s], kXBoxBytes);
        tma_load_4d(sm.xst[s], &tmap_x, kq - 3, jq - 2, 0, q - tp.x_base, &sm.full[s]);
    };
    auto issue_v = [&](int p) {  // V_t of plane p
        const int s = (p - v_first) % kVStages;
        mbar_expect_tx(&sm.vfull[s], kVBoxBytes);
        tma_load_4d(sm.vst[s], &tmap_v, kq - 3, jq - 1, 0, p - tp.v_base, &sm.vfull[s]);
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

    const int xA = (rA + 1) * kBK + (lane + 2), xB = xA + kBK;   // own X box offsets
    const int vA = rA * kVBK + (lane + 2), vB = vA + kVBK;        // own V box offsets
    const int yA = rA * kTK + lane, yB = yA + kTK;                // own X_{t+1} ring offsets
    const int yAk = lane < kTK - 1 ? yA + 1 : yA;                 // +k neighbour (lane 31 is ring: unused)
    const int yBk = lane < kTK - 1 ? yB + 1 : yB;
    const int yBj = w < kW - 1 ? yB + kTK : yB;                   // +j neighbour of row B (last row is ring)
    const bool kin = k >= 1 && k < g.n2 - 1;
    const bool intA = kin && jA >= 1 && jA < g.n1 - 1, intB = kin && jB >= 1 && jB < g.n1 - 1;
    const bool kown = lane >= 1 && lane <= kOK && k <= g.n2 - 2;   // interior k columns only
    const bool ownA = kown && rA >= 1 && jA < g.n1;               // rows 1 .. kRows-2
    const bool ownB = kown && rB <= kRows - 2 && jB < g.n1;
    const int64_t cs = tp.cs, ps = tp.ps;
    const int64_t offA = ownA ? (int64_t)jA * g.ld + k : 0, offB = ownB ? (int64_t)jB * g.ld + k : 0;

    // Tile-border springs of S1 (row above R1 -> R1 row 0: gbj; column left of
    // R1 -> R1 lane 0: gbk) of plane p. They are computed one iteration ahead,
    // after barrier #2, by the two warps whose S2 phase has a ring row and so
    // one row less to update (warp 0: row 0, warp kW-1: row kRows-1) -- keeping
    // the S1 spring phase before barrier #1 equal across warps. Written in
    // phase C of iteration p-1 (or the prologue), read after barrier #1 of
    // iteration p, rewritten after barrier #2 of iteration p.
    auto border_springs = [&](int p) {
        const double* Xb = xbox(p);
        if (w == 0) {
            sm.gbj[lane] = spring_force<kPosK, kFma>(ldb(Xb, lane + 2, kXComp), ldb(Xb, kBK + lane + 2, kXComp), a.K, a.L);
        } else if (w == kW - 1 && lane < kRows) {
            const int r = (lane + 1) * kBK;
            sm.gbk[lane] = spring_force<kPosK, kFma>(ldb(Xb, r + 1, kXComp), ldb(Xb, r + 2, kXComp), a.K, a.L);
        }
    };

    // prologue: X_t(ps0) own, the step-t -i spring of plane ps0, border springs of ps0
    Vec3 carry1A{0.0, 0.0, 0.0}, carry1B{0.0, 0.0, 0.0};
    xwait(ps0);
    Vec3 xcA = ldb(xbox(ps0), xA, kXComp), xcB = ldb(xbox(ps0), xB, kXComp);
    if (ps0 >= 1) {
        border_springs(ps0);  // ps0 <= ilast always
        xwait(ps0 - 1);
        carry1A = spring_force<kPosK, kFma>(ldb(xbox(ps0 - 1), xA, kXComp), xcA, a.K, a.L);
        carry1B = spring_force<kPosK, kFma>(ldb(xbox(ps0 - 1), xB, kXComp), xcB, a.K, a.L);
        __syncthreads();
        if (tid == 0 && q0 + kStages <= qlast) {
            fence_proxy_async();
            issue_x(q0 + kStages);  // X_t(ps0 - 1) is no longer needed
        }
    }
    Vec3 carry2A{0.0, 0.0, 0.0}, carry2B{0.0, 0.0, 0.0};
    Vec3 v1pA{0.0, 0.0, 0.0}, v1pB{0.0, 0.0, 0.0};  // V_{t+1} of plane p-1
    NodeStats st;  // stats of the launch's last step (t+2, or t+1 in one-step mode); step t+1's: sm.acc1
    st.zero();
#pragma unroll
    for (int c = 0; c < 7; c++) sm.acc1[c][tid] = 0ull;
    const int border_last = min(pe, ilast);  // planes whose border springs S1 needs
    // X_{t+2} (X_{t+1}), V of an S2 output node: own slab, and the neighbours'
    // halo planes (2 planes of X, 1 of V per face: what their next launch reads)
    auto store_out = [&](int q, int64_t off, const Vec3& x2, const Vec3& v2) {
        stb3(tp.x_out + (int64_t)(q - tp.x_base) * ps + off, cs, x2);
        stb3(tp.v_out + (int64_t)(q - tp.v_base) * ps + off, cs, v2);
        if (q < tp.lo_end) {
            stb3(a.lo_dst + (int64_t)(q - start) * ps + off, cs, x2);
            if (q == start) stb3(tp.lo_vdst + off, cs, v2);
        }
        if (q >= tp.hi_begin) {
            stb3(a.hi_dst + (int64_t)(q - tp.hi_begin) * ps + off, cs, x2);
            if (q == start + size - 1) stb3(tp.hi_vdst + off, cs, v2);
        }
    };

    // Step t+1's stats of an output plane from S1's registers (X_{t+1},
    // V_{t+1}); read-modify-write of the thread's shared-memory accumulators.
    // Counted rows are shifted by one against R2: a tile counts R1 rows
    // 0 .. kRows-3 (global [jq - 1, jq + kOJ - 1)), which partition the j axis
    // as R2's rows do (the launcher sizes tiles_j so the last row is covered) --
    // so a whole warp (the last) skips, and no addend is selected per node: the
    // threads of ring / k-face / out-of-grid COLUMNS (kown false) accumulate
    // anyway and drop their sums at the end, and rows outside the grid add
    // x = 0, v = 0 (the TMA zero fill, never updated), neutral once counted in
    // n (set at the end: calls x 2).
    auto acc1_update = [&](const Vec3& xa, const Vec3& xb, const Vec3& va, const Vec3& vb) {
        if (w == kW - 1) return;  // warp-uniform
        auto coord = [&](int c, double a, double b) {
            double hda, lda, hdb, ldb_;
            split_q(a, hda, lda);
            split_q(b, hdb, ldb_);
            sm.acc1[c][tid] += (unsigned long long)__double_as_longlong(hda) +
                               (unsigned long long)__double_as_longlong(hdb);
            sm.acc1[3 + c][tid] += (unsigned long long)__double_as_longlong(lda) +
                                   (unsigned long long)__double_as_longlong(ldb_);
        };
        coord(0, xa.x, xb.x);
        coord(1, xa.y, xb.y);
        coord(2, xa.z, xb.z);
        const double v2a = dot_self(va), v2b = dot_self(vb);
        double vm = __longlong_as_double((long long)sm.acc1[6][tid]);
        vm = (v2a > vm || v2a != v2a) ? v2a : vm;
        vm = (v2b > vm || v2b != v2b) ? v2b : vm;
        sm.acc1[6][tid] = (unsigned long long)__double_as_longlong(vm);
    };

    // the last step's stats of one node (hasv: an interior node, v enters vmax)
    auto st_add = [&](const Vec3& x, const Vec3& v, bool hasv) {
        st.add_position(x);
        if (hasv) st.add_velocity(v);
    };

    // One plane of the march. kFull: a steady-state plane (p+1 exists, p is
    // updated by S1, q = p-1 is an S2 output plane): no conditions, no
    // zero-initialised partial results. kPar: p & 1 when known (0/1), else -1.
    auto body = [&](auto full_c, auto par_c, int p) {
        constexpr bool kFull = decltype(full_c)::value;
        constexpr int kPar = decltype(par_c)::value;
        const int par = kPar >= 0 ? kPar : (p & 1);
        const bool upd1 = kFull || (p >= 1 && p <= ilast);  // S1 updates plane p (else a fixed face plane)
        const bool has_next = kFull || p + 1 <= qlast;
        if (has_next) xwait(p + 1);
        const double* Xc = xbox(p);
        const double* Xn = has_next ? xbox(p + 1) : Xc;
        // ---- S1 "+" springs of plane p
        Vec3 gpi1A, gpi1B, gpj1A, gpj1B, gpk1A, gpk1B;
        const Vec3 niA = ldb(Xn, xA, kXComp), niB = ldb(Xn, xB, kXComp);
        if (has_next) {
            gpi1A = spring_force<kPosK, kFma>(xcA, niA, a.K, a.L);
            gpi1B = spring_force<kPosK, kFma>(xcB, niB, a.K, a.L);
        } else {
            gpi1A = gpi1B = Vec3{0.0, 0.0, 0.0};
        }
        if (upd1) {
            gpk1A = spring_force<kPosK, kFma>(xcA, ldb(Xc, xA + 1, kXComp), a.K, a.L);
            gpk1B = spring_force<kPosK, kFma>(xcB, ldb(Xc, xB + 1, kXComp), a.K, a.L);
            gpj1A = spring_force<kPosK, kFma>(xcA, xcB, a.K, a.L);
            gpj1B = spring_force<kPosK, kFma>(xcB, ldb(Xc, xB + kBK, kXComp), a.K, a.L);
            sm.g1j[w][lane] = gpj1B;
        } else {
            gpk1A = gpk1B = gpj1A = gpj1B = Vec3{0.0, 0.0, 0.0};
        }
        const Vec3 up1A = shfl_up1(gpk1A), up1B = shfl_up1(gpk1B);
        __syncthreads();  // #1: S1 springs visible; X_t(p) read for the last time
        if (tid == 0 && p + kStages <= qlast) {
            fence_proxy_async();
            issue_x(p + kStages);
        }
        // ---- S1 forces -> V_{t+1}, X_{t+1} of R1, plane p
        Vec3 x1A = xcA, x1B = xcB, v1A{0.0, 0.0, 0.0}, v1B{0.0, 0.0, 0.0};
        if (upd1) {
            const int vs = (p - v_first) % kVStages;
            mbar_wait(&sm.vfull[vs], (unsigned)(((p - v_first) / kVStages) & 1));
            const double* Vb = reinterpret_cast<const double*>(sm.vst[vs]);
            if (intA) {
                const Vec3 gmj = neg(w == 0 ? sm.gbj[lane] : sm.g1j[w - 1][lane]);
                const Vec3 gmk = neg(lane == 0 ? sm.gbk[rA] : up1A);
                const Vec3 F = sum_forces(neg(carry1A), gpi1A, gmj, gpj1A, gmk, gpk1A);
                v1A = ldb(Vb, vA, kVComp);
                kick_drift<kUnitMass, kFma>(F, a.M, a.dt, v1A, xcA, x1A);
            }
            if (intB) {
                const Vec3 gmk = neg(lane == 0 ? sm.gbk[rB] : up1B);
                const Vec3 F = sum_forces(neg(carry1B), gpi1B, neg(gpj1A), gpj1B, gmk, gpk1B);
                v1B = ldb(Vb, vB, kVComp);
                kick_drift<kUnitMass, kFma>(F, a.M, a.dt, v1B, xcB, x1B);
            }
        }
        // step t+1's stats right where S1 produced them (plane p, if an output plane of this segment)
        if (kTwo && TB2_MID_STATS && p >= max(pb, tp.stats_lo) && p < min(pe, tp.stats_hi))
            acc1_update(x1A, x1B, v1A, v1B);
        {
            double* y = sm.y[par][0];
            y[yA] = x1A.x;
            y[yA + kYComp] = x1A.y;
            y[yA + 2 * kYComp] = x1A.z;
            y[yB] = x1B.x;
            y[yB + kYComp] = x1B.y;
            y[yB + 2 * kYComp] = x1B.z;
        }
        // ---- S2 "+" springs of plane q = p-1 (its X_{t+1} is in the ring since iteration p-1)
        const int q = p - 1;
        const bool do2 = kFull || q >= ps0;  // q == ps0: only the +i spring (carry of plane pb)
        const bool out2 = kFull || q >= pb;  // an output plane
        Vec3 gpi2A, gpi2B, gpj2A, gpj2B, gpk2A, gpk2B, xqA, xqB;
        gpi2A = gpi2B = gpj2A = gpj2B = gpk2A = gpk2B = xqA = xqB = Vec3{0.0, 0.0, 0.0};
        if (do2) {
            const double* yq = sm.y[par ^ 1][0];
            xqA = ldb(yq, yA, kYComp);
            xqB = ldb(yq, yB, kYComp);
            if (kTwo) {
                gpi2A = spring_force<kPosK, kFma>(xqA, x1A, a.K, a.L);
                gpi2B = spring_force<kPosK, kFma>(xqB, x1B, a.K, a.L);
                if (out2) {
                    gpk2A = spring_force<kPosK, kFma>(xqA, ldb(yq, yAk, kYComp), a.K, a.L);
                    gpk2B = spring_force<kPosK, kFma>(xqB, ldb(yq, yBk, kYComp), a.K, a.L);
                    gpj2A = spring_force<kPosK, kFma>(xqA, xqB, a.K, a.L);
                    gpj2B = spring_force<kPosK, kFma>(xqB, ldb(yq, yBj, kYComp), a.K, a.L);
                    sm.g2j[w][lane] = gpj2B;
                }
            }
        }
        const Vec3 up2A = shfl_up1(gpk2A), up2B = shfl_up1(gpk2B);
        __syncthreads();  // #2: S2 springs and X_{t+1}(p) visible; V_t(p) slot free; gbj/gbk(p) consumed
        if (tid == 0 && upd1 && p + kVStages <= v_last) {
            fence_proxy_async();
            issue_v(p + kVStages);
        }
        // ---- S2 forces -> X_{t+2}, V_{t+2} of R2, plane q (one-step mode: X_{t+1}, V_{t+1} of S1)
        const bool sq = kFull ? (q >= tp.stats_lo && q < tp.stats_hi) : (out2 && q >= tp.stats_lo && q < tp.stats_hi);
        if (out2) {
            if (ownA) {
                if (intA) {
                    Vec3 v2 = v1pA, x2 = xqA;
                    if (kTwo) {
                        const Vec3 gmj = neg(sm.g2j[w > 0 ? w - 1 : 0][lane]);  // w == 0: row 0 is ring, not owned
                        const Vec3 F = sum_forces(neg(carry2A), gpi2A, gmj, gpj2A, neg(up2A), gpk2A);
                        kick_drift<kUnitMass, kFma>(F, a.M, a.dt, v2, xqA, x2);
                    }
                    // stats first: v.v must not overwrite v2's registers before the stores read them
                    if (sq) st_add(x2, v2, true);
                    store_out(q, offA, x2, v2);
                } else if (sq) {
                    st_add(xqA, xqA, false);  // fixed face node
                }
            }
            if (ownB) {
                if (intB) {
                    Vec3 v2 = v1pB, x2 = xqB;
                    if (kTwo) {
                        const Vec3 F = sum_forces(neg(carry2B), gpi2B, neg(gpj2A), gpj2B, neg(up2B), gpk2B);
                        kick_drift<kUnitMass, kFma>(F, a.M, a.dt, v2, xqB, x2);
                    }
                    // stats first: v.v must not overwrite v2's registers before the stores read them
                    if (sq) st_add(x2, v2, true);
                    store_out(q, offB, x2, v2);
                } else if (sq) {
                    st_add(xqB, xqB, false);
                }
            }
        }
        // border springs of the next plane (X_t(p+1) is resident until barrier #1 of iteration p+1)
        if (p + 1 <= border_last) border_springs(p + 1);
        carry1A = gpi1A;
        carry1B = gpi1B;
        xcA = niA;
        xcB = niB;
        carry2A = gpi2A;
        carry2B = gpi2B;
        v1pA = v1A;
        v1pB = v1B;
    };
    using F0 = std::integral_constant<bool, false>;
    using F1 = std::integral_constant<bool, true>;
    using PN = std::integral_constant<int, -1>;
    using P0 = std::integral_constant<int, 0>;
    using P1 = std::integral_constant<int, 1>;
    // steady planes: p >= pb+1 (q = p-1 is an output plane, p > ps0), p <= min(ilast, pe) (updated, p+1 exists)
    const int lo = pb + 1, hi = min(ilast, pe);
    int p = ps0;
    for (; p < lo && p <= pe; p++) body(F0{}, PN{}, p);
    if (p <= hi && (p & 1)) body(F1{}, P1{}, p++);
    for (; p + 1 <= hi; p += 2) {
        body(F1{}, P0{}, p);
        body(F1{}, P1{}, p + 1);
    }
    if (p <= hi) body(F1{}, P0{}, p++);
    for (; p <= pe; p++) body(F0{}, PN{}, p);
    block_accumulate(st, sm.scratch, slots.fin);
    if (kTwo && TB2_MID_STATS) {
#ifndef STATS_FP64_ACC
        NodeStats st1;
        for (int c = 0; c < 3; c++) {
            st1.hb[c] = sm.acc1[c][tid];
            st1.lb[c] = sm.acc1[3 + c][tid];
        }
        st1.vmax2 = __longlong_as_double((long long)sm.acc1[6][tid]);
        {
            const int calls = max(0, min(pe, tp.stats_hi) - max(pb, tp.stats_lo));
            st1.n = (unsigned)(calls * 2);
            if (!kown || w == kW - 1) st1.zero();
        }
        __syncthreads();  // scratch reuse
        block_accumulate(st1, sm.scratch, slots.mid);
#else
#error "K1_TB2 keeps step t+1's stats as bit-pattern sums (no STATS_FP64_ACC variant)"
#endif
    }
    // lo side: stores planes start, start+1 into the left neighbour or reads
    // planes below start; hi side: the mirror image (launch_k1_tb2 counts them)
    finish_launch(a, slots.t, kTwo ? 2 : 1, pb <= start + 1, pe >= start + size - 1);
}

}  // namespace

cudaError_t launch_k1_tb2(const StepArgs& a, const Tb2Out& o, bool unit_mass, cudaStream_t stream) {
    if (a.g.size <= 0) return cudaSuccess;
    if (!a.tmap_x_cur || !a.tmap_v || !o.x_out || !o.v_out) return cudaErrorInvalidValue;
    if (!a.step_word && (!a.acc || (o.two && !a.acc_mid))) return cudaErrorInvalidValue;  // both steps' stats slots
    if ((a.lo_dst && (!o.lo_vdst || a.g.size < 2)) || (a.hi_dst && (!o.hi_vdst || a.g.size < 2)))
        return cudaErrorInvalidValue;  // a neighbour's two halo planes come from one chunk
    Tb2Params tp;
    tp.a = a;
    tp.x_out = o.x_out;
    tp.v_out = o.v_out;
    tp.lo_vdst = o.lo_vdst;
    tp.hi_vdst = o.hi_vdst;
    tp.x_base = (int)a.g.start - 2;
    tp.v_base = (int)a.g.start - 1;
    tp.lo_end = a.lo_dst ? (int)a.g.start + 2 : INT_MIN;
    tp.hi_begin = a.hi_dst ? (int)(a.g.start + a.g.size) - 2 : INT_MAX;
    tp.cs = a.g.comp_stride();
    tp.ps = a.g.plane_stride();
    tp.stats_lo = o.stats_lo;
    tp.stats_hi = o.stats_hi;
    if (o.stats_lo == 0 && o.stats_hi == 0) {  // default: the chunk's own planes
        tp.stats_lo = (int)a.g.start;
        tp.stats_hi = (int)(a.g.start + a.g.size);
    }
    tp.tiles_k = (int)((a.g.n2 - 2 + kOK - 1) / kOK);
    // R2 rows [jq, jq + kOJ) cover [0, n1); step t+1's stats rows [jq - 1,
    // jq + kOJ - 1) must too (one more tile when n1 is a multiple of kOJ)
    tp.tiles_j = (int)((a.g.n1 + kOJ) / kOJ);
    const int tiles = tp.tiles_k * tp.tiles_j;
    // Segments per tile column: one CTA per SM (384 threads x 168 registers),
    // so the grid runs in waves of `sms` CTAs. Each segment pays ~3 planes of
    // extra work (step t on its first and last planes, the X/V pipeline fill);
    // a partial last wave leaves SMs idle. Pick the count minimising
    // waves x (segment + 3), segments of at most 256 planes (measured, DESIGN.md
    // §6: 256^3 4 segments 6.92e10 vs 6 of the old 64-plane rule 6.23e10;
    // 512^3 5 vs 8: 7.30 vs 7.19e10; 1024^3 7 vs 16: 7.00 vs 6.88e10; one
    // segment of 1022 planes 6.51e10).
    static int sms_cache[64] = {0};
    int dev = 0;
    cudaGetDevice(&dev);
    int& sms = sms_cache[dev & 63];
    if (!sms) {
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        if (sms <= 0) sms = 148;
    }
    const int64_t size = a.g.size;
    int nseg = 0;
    double best = 0.0;
    for (int c = 1; c <= std::min<int64_t>(size, 64); c++) {
        const int64_t seg = (size + c - 1) / c;
        if (seg < kMinSegPlanes && c > 1) break;
        if (seg > kMaxSegPlanes) continue;  // long segments drift apart: halo rows fall out of L2
        const double waves = std::ceil((double)tiles * c / sms);
        const double cost = waves * (double)(seg + 3);
        if (nseg == 0 || cost < best - 1e-9) {
            best = cost;
            nseg = c;
        }
    }
    if (nseg == 0) nseg = (int)((size + kMaxSegPlanes - 1) / kMaxSegPlanes);
    static const int env_nseg = [] {  // experiment hook: segments per tile column
        const char* e = std::getenv("SOMIER_TB2_NSEG");
        return e ? std::atoi(e) : 0;
    }();
    if (env_nseg > 0) nseg = std::min<int>(env_nseg, (int)a.g.size);
    tp.seg_planes = (int)((a.g.size + nseg - 1) / nseg);
    if (tp.seg_planes < kMinSegPlanes) tp.seg_planes = (int)std::min<int64_t>(kMinSegPlanes, a.g.size);
    nseg = (int)((a.g.size + tp.seg_planes - 1) / tp.seg_planes);
    dim3 grid((unsigned)tiles, (unsigned)nseg), block(kTK, kW);
    {  // CTAs of the segments that touch each neighbour (the kernel's lo_side / hi_side)
        unsigned int lo = 0, hi = 0;
        const int start = (int)a.g.start, size = (int)a.g.size;
        for (int sg = 0; sg < nseg; sg++) {
            const int pb = start + sg * tp.seg_planes, pe = std::min(start + size, pb + tp.seg_planes);
            lo += pb <= start + 1 ? 1u : 0u;
            hi += pe >= start + size - 1 ? 1u : 0u;
        }
        tp.a.lo_ctas = lo * (unsigned)tiles;
        tp.a.hi_ctas = hi * (unsigned)tiles;
    }
    const size_t smem = sizeof(Smem);
    const CUtensorMap& mx = *static_cast<const CUtensorMap*>(a.tmap_x_cur);
    const CUtensorMap& mv = *static_cast<const CUtensorMap*>(a.tmap_v);
    auto launch = [&](auto kernel) {
        cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        kernel<<<grid, block, smem, stream>>>(mx, mv, tp);
    };
    const bool pos_k = a.K > 0.0;
    dispatch_bools([&](auto um, auto pk, auto two, auto fm) {
        launch(k1_tb2_kernel<decltype(um)::value, decltype(pk)::value, decltype(two)::value, decltype(fm)::value>);
    }, unit_mass, pos_k, o.two, a.fma != 0);
    return cudaGetLastError();
}

}  // namespace paper
