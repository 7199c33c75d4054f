// somier.cpp -- the Somier driver behind include/somier.h: per-chunk slabs on
// the devices of a spread, the step loop with the fused halo exchange, exact
// stats combination, map-to / map-from copies, and CUDA IPC for one process per
// GPU. PAPER.md §V (319-344) for the method; §III-B (79-243) for the clauses
// whose semantics the calls follow (see include/somier.h).
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <map>
#include <new>
#include <string>
#include <vector>

#include "driver_util.hpp"
#include "guard.hpp"
#include "kernels.hpp"
#include "nccl_api.hpp"
#include "trace.hpp"
#include "somier.h"
#include "spread_impl.hpp"
#include "status.hpp"

using paper::set_last_error;

namespace {

constexpr uint64_t kIpcMagic = 0x534f4d4945524950ull;  // "SOMIERIP"
constexpr uint32_t kIpcVersion = 4;

using PFN_waitValue64 = CUresult (*)(CUstream, CUdeviceptr, cuuint64_t, unsigned int);
using PFN_writeValue64 = CUresult (*)(CUstream, CUdeviceptr, cuuint64_t, unsigned int);
using PFN_encodeTiled = CUresult (*)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                     const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                     CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

struct DevCtx {
    int device = -1;
    cudaStream_t own = nullptr;   // created by the library
    cudaStream_t stream = nullptr;  // in use (own or user-provided)
    // CU_STREAM_WAIT_VALUE_FLUSH when the device supports it: remote (peer)
    // halo stores that reached the device before the flag are made visible to
    // the kernels after the wait
    unsigned int wait_flush = 0;
};

// One chunk = one `target spread` iteration block (omp_spread_start/size).
struct Chunk {
    int64_t index = 0, start = 0, size = 0;
    int pos = 0, device = 0;
    bool local = false;
    // local allocation: [x0 | x1 | v0 | (v1, K1_TB2 only) | acc[kStatsRing + 2] | flags[2] | counter | step word]
    // acc: [0, kStatsRing) per-step stats history (state s in ring_slot(s)),
    // [kStatsRing] the fixed nodes no launch visits (end planes held as halos,
    // K1_TB2's k-face columns), [kStatsRing + 1] unused. The step word is the
    // device copy of the step counter the kernels take their ring slots from.
    // X slabs: planes [start-1, start+size+1) (one halo plane per face), V
    // slabs [start, start+size); on a K1_TB2 handle one more halo plane per
    // face each (X [start-2, start+size+2), V [start-1, start+size+1)) and V
    // double-buffered. xs()/vs() are the one-halo views every other path uses.
    void* base = nullptr;
    size_t bytes = 0;
    size_t off_x[2] = {0, 0}, off_v = 0, off_v1 = 0, off_acc = 0, off_flags = 0, off_counter = 0;
    size_t xbytes = 0;  // one X buffer (without a guard zone)
    paper::GuardLayout guard;  // SOMIER_GUARD zones (guard.hpp; none by default)
    int64_t view_off = 0;  // doubles from a raw slab to its one-halo view (one plane on K1_TB2 handles)
    // remote view (IPC-opened), for non-local neighbours
    void* remote_base = nullptr;
    // TMA descriptors of the local slabs, by X / V buffer: K1_MARCH, K1_MARCH2, K1_TB2 box shapes
    alignas(64) CUtensorMap tmap_x[2];
    alignas(64) CUtensorMap tmap_v[2];
    alignas(64) CUtensorMap tmap_x2[2];
    alignas(64) CUtensorMap tmap_v2[2];
    alignas(64) CUtensorMap tmap_xt[2];
    alignas(64) CUtensorMap tmap_vt[2];

    void* mem() const { return local ? base : remote_base; }
    double* x(int parity) const { return (double*)((char*)mem() + off_x[parity]); }
    double* v(int b = 0) const { return (double*)((char*)mem() + (b ? off_v1 : off_v)); }
    double* xs(int parity) const { return x(parity) + view_off; }
    double* vs(int b = 0) const { return v(b) + view_off; }
    paper::StatsAccum* acc() const { return (paper::StatsAccum*)((char*)mem() + off_acc); }
    unsigned long long* flags() const { return (unsigned long long*)((char*)mem() + off_flags); }
    unsigned int* counter() const { return (unsigned int*)((char*)mem() + off_counter); }
    unsigned long long* step_word() const { return (unsigned long long*)((char*)mem() + off_counter + 8); }
    unsigned int* side_counter() const { return (unsigned int*)((char*)mem() + off_counter + 16); }  // [2]
    paper::StatsAccum* acc_static() const { return acc() + paper::kStatsRing; }
};

struct IpcChunkRecord {
    int64_t index;
    uint64_t bytes, off_x0, off_x1, off_v, off_v1, off_acc, off_flags, off_counter;
    cudaIpcMemHandle_t handle;
};

struct IpcHeader {
    uint64_t magic;
    uint32_t version;
    int32_t device_pos;
    int64_t n[3];
    int64_t nchunks;
    int64_t chunk;
    uint64_t layout;  // FNV-1a of every chunk's (device_pos, start, size): catches unequal irregular tables
    int64_t nrecords;
    int32_t tb2;      // slab layout: K1_TB2 (deep halo, V double-buffered) or one-step
    int32_t pad;
};

uint64_t spread_layout_hash(const spread_s& s) {
    uint64_t h = 1469598103934665603ull;
    auto mix = [&](int64_t v) {
        for (int b = 0; b < 8; b++) {
            h ^= (uint64_t)((v >> (8 * b)) & 0xff);
            h *= 1099511628211ull;
        }
    };
    for (int64_t c = 0; c < s.nchunks; c++) {
        const paper::ChunkInfo ci = s.chunk_info(c);
        mix(ci.pos);
        mix(ci.start);
        mix(ci.size);
    }
    return h;
}

size_t round_up(size_t v, size_t a) { return (v + a - 1) / a * a; }


}  // namespace

struct somier_s {
    somier_params p{};
    spread_s spread;
    paper::SlabGeom geom{};  // start/size filled per chunk
    int64_t ld = 0;
    int64_t step = 0;
    int64_t hist_first = 0;  // oldest state whose stats are in the history ring (last init / load)
    int64_t launches = 0;
    int xbuf = 0;      // X buffer holding X_t (flips once per launch)
    int vbuf = 0;      // V buffer holding V_t (flips once per K1_TB2 launch; 1-step kernels update in place)
    bool tb2 = false;  // K1_TB2 mode (two steps per launch, deep-halo slabs)
    bool multi_process = false;
    int local_pos = -1;
    std::vector<Chunk> chunks;
    std::vector<DevCtx> devs;  // indexed by list position
    std::string sticky;        // first asynchronous CUDA error
    PFN_waitValue64 wait_value64 = nullptr;
    PFN_writeValue64 write_value64 = nullptr;
    PFN_encodeTiled encode_tiled = nullptr;
    bool connected = true;
    // CUDA graph of an (even, odd) step pair, when every chunk is on one stream
    bool graph_ok = false;
    bool pdl = false;
    int graph_pos = -1;
    cudaGraphExec_t graph_exec = nullptr;
    cudaGraphExec_t tb2_graph[4] = {nullptr, nullptr, nullptr, nullptr};  // by (X buffer parity, step parity)
    // somier_set_timing: per launch, events before the neighbour-flag waits,
    // after them (= kernel start) and after the kernel
    struct TimingRec {
        int device;
        cudaEvent_t a, b, c;
    };
    bool timing = false;
    std::vector<TimingRec> trecs;
    std::vector<paper::ncclComm> comms;  // SOMIER_EXCHANGE_NCCL: per list position (local ones)

    bool unit_mass() const { return p.mass == 1.0; }
    paper::K1Variant variant() const {
        return paper::k1_variant(p.kernel);
    }
    paper::SlabGeom geom_of(const Chunk& c) const {
        paper::SlabGeom g = geom;
        g.start = c.start;
        g.size = c.size;
        return g;
    }
    cudaStream_t stream_of(const Chunk& c) const { return devs[c.pos].stream; }
    // Neighbour chunks on another stream (other device or other process) need
    // the flag protocol; same-stream neighbours are ordered by the stream.
    bool needs_flags(const Chunk& a, const Chunk& b) const {
        if (p.exchange == SOMIER_EXCHANGE_NCCL) return false;  // the NCCL ops order the streams
        if (!a.local || !b.local) return true;
        return a.pos != b.pos;
    }
};

namespace {

spread_status cuda_fail(somier_t h, cudaError_t e, const char* what) {
    std::string msg = std::string(what) + ": " + cudaGetErrorString(e);
    if (h && h->sticky.empty()) h->sticky = msg;
    set_last_error("%s", msg.c_str());
    return e == cudaErrorMemoryAllocation ? SPREAD_ENOMEM : SPREAD_ECUDA;
}

#define CUDA_TRY(h, call)                                         \
    do {                                                          \
        cudaError_t e_ = (call);                                  \
        if (e_ != cudaSuccess) return cuda_fail((h), e_, #call);  \
    } while (0)

// somier_set_timing instrumentation: events around one launch's waits and kernel
spread_status timing_begin(somier_t h, int device, cudaStream_t st, somier_s::TimingRec* r) {
    r->device = device;
    r->a = r->b = r->c = nullptr;
    CUDA_TRY(h, cudaEventCreate(&r->a));
    CUDA_TRY(h, cudaEventCreate(&r->b));
    CUDA_TRY(h, cudaEventCreate(&r->c));
    CUDA_TRY(h, cudaEventRecord(r->a, st));
    return SPREAD_OK;
}

// SOMIER_EXCHANGE_COPY: publish the neighbours' flags once everything before
// on the stream (the kernel, the halo copies) is done
spread_status signal_after(somier_t h, cudaStream_t st, unsigned long long* lo, unsigned long long* hi,
                           unsigned long long value) {
    for (unsigned long long* f : {lo, hi}) {
        if (!f) continue;
        CUresult r = h->write_value64((CUstream)st, (CUdeviceptr)f, (cuuint64_t)value, CU_STREAM_WRITE_VALUE_DEFAULT);
        if (r != CUDA_SUCCESS) PAPER_FAIL(SPREAD_ECUDA, "somier_step: cuStreamWriteValue64 failed (%d)", (int)r);
    }
    return SPREAD_OK;
}

spread_status check_params(const somier_params* p) {
    if (!p) PAPER_FAIL(SPREAD_EINVAL, "somier: params is NULL");
    for (int d = 0; d < 3; d++)
        if (p->n[d] < 3) PAPER_FAIL(SPREAD_EINVAL, "somier: n[%d] = %lld < 3", d, (long long)p->n[d]);
    const double vals[] = {p->spacing, p->rest_len, p->k_spring, p->mass, p->dt, p->amplitude};
    for (double v : vals)
        if (!std::isfinite(v)) PAPER_FAIL(SPREAD_EINVAL, "somier: non-finite parameter");
    if (!(p->mass > 0)) PAPER_FAIL(SPREAD_EINVAL, "somier: mass must be > 0");
    if (!(p->dt > 0)) PAPER_FAIL(SPREAD_EINVAL, "somier: dt must be > 0");
    if (p->kernel < SOMIER_K1_AUTO || p->kernel > SOMIER_K1_TB2)
        PAPER_FAIL(SPREAD_EINVAL, "somier: unknown kernel %d", p->kernel);
    if (p->exchange != SOMIER_EXCHANGE_FUSED && p->exchange != SOMIER_EXCHANGE_COPY &&
        p->exchange != SOMIER_EXCHANGE_NCCL)
        PAPER_FAIL(SPREAD_EINVAL, "somier: unknown exchange %d", p->exchange);
    if (p->math != SOMIER_MATH_EXACT && p->math != SOMIER_MATH_FMA)
        PAPER_FAIL(SPREAD_EINVAL, "somier: unknown math mode %d", p->math);
    if (p->reserved != 0) PAPER_FAIL(SPREAD_EINVAL, "somier: reserved must be 0");
    const int64_t n0 = p->n[0], n1 = p->n[1], n2 = p->n[2];
    if (n1 > 65535LL * 8 || n0 > 65535 + 2)
        PAPER_FAIL(SPREAD_EINVAL, "somier: grid too large for the launch geometry");
    // the branch-free sqrt / division of the spring law (kernels/node_math.cuh)
    // are correctly rounded for |K|, |L| in [2^-100, 2^100] (or 0)
    auto in_domain = [](double v) { return v == 0.0 || (std::fabs(v) >= 0x1p-100 && std::fabs(v) <= 0x1p100); };
    if (!in_domain(p->k_spring) || !in_domain(p->rest_len))
        PAPER_FAIL(SPREAD_EINVAL, "somier: k_spring and rest_len must be 0 or of magnitude in [2^-100, 2^100]");
    // the fused exact centre sums (kernels/stats.cuh) need |x| < 2^18; keep a
    // factor-2 margin over the initial extent of the lattice
    const double extent = (double)(std::max(n0, std::max(n1, n2)) - 1) / 2.0 * std::fabs(p->spacing) +
                          std::fabs(p->amplitude);
    if (!(extent < 131072.0))
        PAPER_FAIL(SPREAD_EINVAL, "somier: lattice extent %.3g too large for exact centre sums (< 2^17)", extent);
    return SPREAD_OK;
}

spread_status load_driver_entry(somier_t h) {
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    cudaError_t e = cudaGetDriverEntryPoint("cuStreamWaitValue64", &fn, cudaEnableDefault, &q);
    if (e != cudaSuccess || q != cudaDriverEntryPointSuccess || !fn)
        PAPER_FAIL(SPREAD_ECUDA, "somier: cuStreamWaitValue64 unavailable (%s)", cudaGetErrorString(e));
    h->wait_value64 = (PFN_waitValue64)fn;
    fn = nullptr;
    e = cudaGetDriverEntryPoint("cuStreamWriteValue64", &fn, cudaEnableDefault, &q);
    if (e != cudaSuccess || q != cudaDriverEntryPointSuccess || !fn)
        PAPER_FAIL(SPREAD_ECUDA, "somier: cuStreamWriteValue64 unavailable (%s)", cudaGetErrorString(e));
    h->write_value64 = (PFN_writeValue64)fn;
    fn = nullptr;
    e = cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q);
    if (e != cudaSuccess || q != cudaDriverEntryPointSuccess || !fn)
        PAPER_FAIL(SPREAD_ECUDA, "somier: cuTensorMapEncodeTiled unavailable (%s)", cudaGetErrorString(e));
    h->encode_tiled = (PFN_encodeTiled)fn;
    return SPREAD_OK;
}

void free_all(somier_t h) {
    if (!h) return;
    for (size_t q = 0; q < h->comms.size(); q++)
        if (h->comms[q]) {
            cudaSetDevice(h->devs[q].device);
            paper::nccl_lib().CommDestroy(h->comms[q]);
            h->comms[q] = nullptr;
        }
    for (auto& c : h->chunks) {
        if (c.remote_base) {
            cudaSetDevice(h->devs[h->local_pos >= 0 ? h->local_pos : 0].device);
            cudaIpcCloseMemHandle(c.remote_base);
            c.remote_base = nullptr;
        }
    }
    for (auto& c : h->chunks) {
        if (c.local && c.base) {
            cudaSetDevice(c.device);
            cudaFree(c.base);
            c.base = nullptr;
        }
    }
    for (auto& d : h->devs) {
        if (d.own) {
            cudaSetDevice(d.device);
            cudaStreamDestroy(d.own);
            d.own = nullptr;
        }
    }
}

// Recompute the stats slots of a chunk from its resident state: the history
// ring is cleared (the stats of earlier states are gone) and ring_slot(step)
// receives the stats of the current state; the static slot the fixed end
// planes the chunk holds as halos (global i = 0 and i = n0-1) and, on K1_TB2
// handles, the fixed k-face columns of its owned planes (which the kernel's
// tiles do not own) -- those are then left out of the per-step slots.
spread_status reset_stats(somier_t h, Chunk& c) {
    cudaStream_t s = h->stream_of(c);
    paper::SlabGeom g = h->geom_of(c);
    CUDA_TRY(h, cudaMemsetAsync(c.acc(), 0, (paper::kStatsRing + 2) * sizeof(paper::StatsAccum), s));
    const int cur = h->xbuf;
    paper::StatsAccum* last = c.acc() + paper::ring_slot((unsigned long long)h->step);
    CUDA_TRY(h, paper::launch_stats(c.xs(cur), c.vs(h->vbuf), g, 1, c.size, last, s, h->tb2));
    if (c.start == 1) CUDA_TRY(h, paper::launch_stats(c.xs(cur), nullptr, g, 0, 1, c.acc_static(), s));
    if (c.start + c.size == h->p.n[0] - 1)
        CUDA_TRY(h, paper::launch_stats(c.xs(cur), nullptr, g, c.size + 1, 1, c.acc_static(), s));
    if (h->tb2) {
        // K1_TB2 does not own the fixed k-face columns of its planes: their
        // constant positions are counted here once, in the static slot
        CUDA_TRY(h, paper::launch_kface_stats(c.xs(cur), g, 1, c.size, c.acc_static(), s));
    }
    h->hist_first = h->step;
    return SPREAD_OK;
}

spread_status allocate_chunk(somier_t h, Chunk& c) {
    const paper::SlabGeom g = h->geom_of(c);
    const size_t plane = (size_t)g.plane_stride() * sizeof(double);
    const int64_t deep = h->tb2 ? 1 : 0;  // K1_TB2: one more halo plane per face (X and V)
    const size_t xb = round_up(plane * (size_t)(c.size + 2 + 2 * deep), 4096);
    const size_t vb = round_up(plane * (size_t)(c.size + 2 * deep), 4096);
    c.view_off = deep * g.plane_stride();
    c.xbytes = xb;
    // [guard] X_0 [guard] X_1 [guard] V ([guard] V') [guard] stats ring + flags + counters [guard]
    const size_t accb = (paper::kStatsRing + 2) * sizeof(paper::StatsAccum);
    std::vector<std::pair<size_t, const char*>> regions = {{xb, "X_0"}, {xb, "X_1"}, {vb, "V"}};
    if (h->tb2) regions.push_back({vb, "V'"});
    regions.push_back({accb + 2 * sizeof(unsigned long long) + 64, "stats"});
    c.guard.plan(paper::guard_bytes(plane), regions);  // no zones unless SOMIER_GUARD is set
    c.off_x[0] = c.guard.off[0];
    c.off_x[1] = c.guard.off[1];
    c.off_v = c.guard.off[2];
    c.off_v1 = h->tb2 ? c.guard.off[3] : c.off_v;
    c.off_acc = c.guard.off.back();
    c.off_flags = c.off_acc + accb;
    c.off_counter = c.off_flags + 2 * sizeof(unsigned long long);  // counter (4 B, padded to 8), step word, side counters[2]
    c.bytes = c.guard.bytes;
    CUDA_TRY(h, cudaSetDevice(c.device));
    CUDA_TRY(h, cudaMalloc(&c.base, c.bytes));
    cudaStream_t s = h->stream_of(c);
    CUDA_TRY(h, cudaMemsetAsync(c.base, 0, c.bytes, s));
    CUDA_TRY(h, paper::guard_fill(c.guard, c.base, s));
    paper::InitArgs ia;
    ia.x0 = c.x(0);
    ia.x1 = c.x(1);
    ia.g = g;
    if (deep) {  // all planes of the deep slab: [start-2, start+size+2) (those outside the grid are never read)
        ia.g.start -= 1;
        ia.g.size += 2;
    }
    ia.spacing = h->p.spacing;
    ia.amplitude = h->p.amplitude;
    ia.seed = h->p.seed;
    CUDA_TRY(h, paper::launch_init(ia, s));
    for (int b = 0; b < 2; b++) {
        const struct {
            CUtensorMap* map;
            double* base;
            int64_t planes;
            uint32_t bk, bj;
        } maps[6] = {{&c.tmap_x[b], c.xs(b), c.size + 2, paper::kXBoxK, paper::kXBoxJ},
                     {&c.tmap_v[b], c.vs(b), c.size, paper::kVBoxK, paper::kVBoxJ},
                     {&c.tmap_x2[b], c.xs(b), c.size + 2, paper::kXBoxK, paper::kX2BoxJ},
                     {&c.tmap_v2[b], c.vs(b), c.size, paper::kVBoxK, paper::kV2BoxJ},
                     {&c.tmap_xt[b], c.x(b), c.size + 2 + 2 * deep, paper::kTB2XBoxK, paper::kTB2XBoxJ},
                     {&c.tmap_vt[b], c.v(b), c.size + 2 * deep, paper::kTB2VBoxK, paper::kTB2VBoxJ}};
        for (const auto& m : maps) {
            spread_status st = paper::encode_slab_tmap(m.map, g, m.base, m.planes, m.bk, m.bj);
            if (st != SPREAD_OK) return st;
        }
    }
    return reset_stats(h, c);
}

spread_status sync_all(somier_t h) {
    for (auto& d : h->devs) {
        if (!d.stream) continue;
        cudaError_t e = cudaSetDevice(d.device);
        if (e == cudaSuccess) e = cudaStreamSynchronize(d.stream);
        if (e != cudaSuccess) return cuda_fail(h, e, "somier_sync");
    }
    if (!h->sticky.empty()) PAPER_FAIL(SPREAD_ECUDA, "%s", h->sticky.c_str());
    for (size_t ci = 0; ci < h->chunks.size(); ci++) {  // SOMIER_GUARD zones (guard.hpp)
        const Chunk& c = h->chunks[ci];
        if (!c.local || !c.guard.G) continue;
        std::string msg;
        cudaError_t e = cudaSetDevice(c.device);
        if (e != cudaSuccess) return cuda_fail(h, e, "somier guard check");
        const std::string what = "chunk " + std::to_string(ci);
        if (!paper::guard_check(c.guard, c.base, what.c_str(), msg, e)) {
            if (e != cudaSuccess) return cuda_fail(h, e, "somier guard check");
            if (h->sticky.empty()) h->sticky = msg;
            PAPER_FAIL(SPREAD_ECUDA, "%s", msg.c_str());
        }
    }
    return SPREAD_OK;
}

spread_status init_common(spread_t s, const somier_params* p, int local_pos, int cuda_device, somier_t* out,
                          const int* cuda_devices = nullptr) {
    if (!out) PAPER_FAIL(SPREAD_EINVAL, "somier_init: out is NULL");
    *out = nullptr;
    if (!s) PAPER_FAIL(SPREAD_EINVAL, "somier_init: spread is NULL");
    if (s->dynamic)
        PAPER_FAIL(SPREAD_ENOTSUP, "somier_init: resident chunks are bound to their devices; the dynamic schedule "
                   "applies to the host-streamed mode (somier_stream_create)");
    spread_status st = check_params(p);
    if (st != SPREAD_OK) return st;
    // Coherence of the spread with the loop it is applied to (the paper leaves
    // this to the programmer): for(i=1; i<n0-1; i++).
    if (s->range_start != 1 || s->range_len != p->n[0] - 2)
        PAPER_FAIL(SPREAD_EINVAL, "somier_init: spread range (%lld:%lld) must be range(1:%lld), the i-loop [1, n0-1)",
                   (long long)s->range_start, (long long)s->range_len, (long long)(p->n[0] - 2));
    int ndev = 0;
    cudaError_t e = cudaGetDeviceCount(&ndev);
    if (e != cudaSuccess) PAPER_FAIL(SPREAD_ENODEV, "somier_init: no CUDA device (%s)", cudaGetErrorString(e));
    const int npos = (int)s->devices.size();
    if (local_pos >= npos) PAPER_FAIL(SPREAD_EINVAL, "somier_init_local: position %d outside the list", local_pos);
    for (int q = 0; q < npos; q++) {
        if (local_pos >= 0 && q != local_pos) continue;
        const int dev = cuda_devices ? cuda_devices[q]
                                     : (q == local_pos && cuda_device >= 0) ? cuda_device : s->devices[q];
        if (dev < 0 || dev >= ndev)
            PAPER_FAIL(SPREAD_ENODEV, "somier_init: device %d not present (%d visible)", dev, ndev);
    }

    somier_s* h = new (std::nothrow) somier_s;
    if (!h) PAPER_FAIL(SPREAD_ENOMEM, "somier_init: out of host memory");
    h->p = *p;
    h->spread = *s;
    h->multi_process = local_pos >= 0;
    h->local_pos = local_pos;
    h->ld = (int64_t)round_up((size_t)p->n[2], 32);
    h->geom = paper::SlabGeom{p->n[0], p->n[1], p->n[2], h->ld, 0, 0};
    h->devs.resize(npos);
    for (int q = 0; q < npos; q++) h->devs[q].device = cuda_devices ? cuda_devices[q] : s->devices[q];
    if (local_pos >= 0 && cuda_device >= 0) h->devs[local_pos].device = cuda_device;
    h->chunks.resize(s->nchunks);
    for (int64_t c = 0; c < s->nchunks; c++) {
        paper::ChunkInfo ci = s->chunk_info(c);
        Chunk& ch = h->chunks[c];
        ch.index = c;
        ch.start = ci.start;
        ch.size = ci.size;
        ch.pos = ci.pos;
        ch.device = h->devs[ci.pos].device;
        ch.local = (local_pos < 0) || (ci.pos == local_pos);
    }
    // K1_TB2 (two steps per launch, deep-halo slabs) runs any spread whose
    // chunks hold >= 2 planes each when there are several (a neighbour's two
    // halo planes come from one chunk). AUTO takes it where it was measured
    // faster than K1_MARCH2 -- chunks of >= kTb2AutoMinNodes nodes (TB2
    // +14..27% from 160^3 up, -2% at 128^3) -- and each device
    // has room for its deeper slabs and second V buffer (96 instead of 72 B/node).
    constexpr double kTb2AutoMinNodes = 3.0e6;
    h->tb2 = false;
    if (p->kernel == SOMIER_K1_TB2 || p->kernel == SOMIER_K1_AUTO) {
        int64_t min_size = INT64_MAX;
        for (auto& c : h->chunks) min_size = std::min(min_size, c.size);
        const bool layout_ok = s->nchunks == 1 || min_size >= 2;
        h->tb2 = layout_ok && (p->kernel == SOMIER_K1_TB2 ||
                               (double)min_size * (double)p->n[1] * (double)p->n[2] >= kTb2AutoMinNodes);
        if (h->tb2 && p->kernel == SOMIER_K1_AUTO) {
            const size_t plane = (size_t)3 * (size_t)p->n[1] * (size_t)h->ld * sizeof(double);
            std::map<int, size_t> need;
            for (auto& c : h->chunks)
                if (c.local) need[c.device] += 2 * plane * (size_t)(c.size + 4) + 2 * plane * (size_t)(c.size + 2);
            for (auto& kv : need) {
                size_t free_b = 0, total_b = 0;
                if (cudaSetDevice(kv.first) != cudaSuccess || cudaMemGetInfo(&free_b, &total_b) != cudaSuccess ||
                    free_b < kv.second + ((size_t)1 << 30))
                    h->tb2 = false;
                cudaGetLastError();
            }
        }
    }
    st = load_driver_entry(h);
    if (st != SPREAD_OK) {
        delete h;
        return st;
    }
    auto fail = [&](spread_status code) {
        std::string msg = paper::last_error();
        free_all(h);
        delete h;
        set_last_error("%s", msg.c_str());
        return code;
    };
    // streams for every list position that owns a local chunk
    for (auto& c : h->chunks) {
        if (!c.local) continue;
        DevCtx& d = h->devs[c.pos];
        if (d.own) continue;
        if ((e = cudaSetDevice(d.device)) != cudaSuccess ||
            (e = cudaStreamCreateWithFlags(&d.own, cudaStreamNonBlocking)) != cudaSuccess) {
            cuda_fail(h, e, "somier_init: stream");
            return fail(SPREAD_ECUDA);
        }
        d.stream = d.own;
        int can_flush = 0;
        if (cudaDeviceGetAttribute(&can_flush, cudaDevAttrCanFlushRemoteWrites, d.device) == cudaSuccess && can_flush)
            d.wait_flush = CU_STREAM_WAIT_VALUE_FLUSH;
        cudaGetLastError();
    }
    // peer access between devices holding neighbouring local chunks
    for (size_t c = 0; c + 1 < h->chunks.size(); c++) {
        const Chunk& a = h->chunks[c];
        const Chunk& b = h->chunks[c + 1];
        if (!a.local || !b.local || a.device == b.device) continue;
        for (int dir = 0; dir < 2; dir++) {
            int from = dir ? b.device : a.device, to = dir ? a.device : b.device;
            int can = 0;
            cudaDeviceCanAccessPeer(&can, from, to);
            if (!can) {
                set_last_error("somier_init: device %d cannot access device %d (no P2P)", from, to);
                return fail(SPREAD_ENOTSUP);
            }
            cudaSetDevice(from);
            e = cudaDeviceEnablePeerAccess(to, 0);
            if (e == cudaErrorPeerAccessAlreadyEnabled) {
                cudaGetLastError();
            } else if (e != cudaSuccess) {
                cuda_fail(h, e, "somier_init: cudaDeviceEnablePeerAccess");
                return fail(SPREAD_ECUDA);
            }
        }
    }
    for (auto& c : h->chunks) {
        if (!c.local) continue;
        st = allocate_chunk(h, c);
        if (st != SPREAD_OK) return fail(st);
    }
    st = sync_all(h);
    if (st != SPREAD_OK) return fail(st);
    // neighbours owned by other processes must be connected before stepping
    for (size_t c = 0; c < h->chunks.size(); c++) {
        if (!h->chunks[c].local) continue;
        if ((c > 0 && !h->chunks[c - 1].local) || (c + 1 < h->chunks.size() && !h->chunks[c + 1].local))
            h->connected = false;
    }
    // SOMIER_EXCHANGE_NCCL: one rank per list position
    h->comms.assign(h->devs.size(), nullptr);
    if (p->exchange == SOMIER_EXCHANGE_NCCL) {
        const paper::NcclLib& L = paper::nccl_lib();
        if (!L.ok) {
            set_last_error("somier_init: NCCL unavailable (%s)", L.error.c_str());
            return fail(SPREAD_ENOTSUP);
        }
        if (local_pos < 0) {
            std::vector<int> devl;
            for (auto& d : h->devs) devl.push_back(d.device);
            std::vector<int> sorted = devl;
            std::sort(sorted.begin(), sorted.end());
            if (std::adjacent_find(sorted.begin(), sorted.end()) != sorted.end()) {
                set_last_error("somier_init: the NCCL exchange needs one CUDA device per list position "
                               "(NCCL places one rank per GPU)");
                return fail(SPREAD_ENOTSUP);
            }
            const int r = L.CommInitAll(h->comms.data(), (int)devl.size(), devl.data());
            if (r != 0) {
                set_last_error("somier_init: ncclCommInitAll: %s", L.GetErrorString(r));
                return fail(SPREAD_ENCCL);
            }
        } else {
            h->connected = false;  // somier_nccl_connect
        }
    }
    // graph replay needs a single stream and no flag protocol (SOMIER_NO_GRAPH=1 disables it)
    {
        int pos = -1;
        bool one = true;
        for (auto& c : h->chunks) {
            if (!c.local) {
                one = false;
                break;
            }
            if (pos < 0) pos = c.pos;
            if (c.pos != pos) one = false;
        }
        const char* ng = std::getenv("SOMIER_NO_GRAPH");
        h->graph_ok = one && pos >= 0 && !(ng && ng[0] == '1') && p->exchange != SOMIER_EXCHANGE_NCCL;
        h->graph_pos = pos;
        // PDL between consecutive K1 launches only where nothing else sits
        // between them on the stream (one stream, no flag waits); SOMIER_NO_PDL=1
        // disables it
        const char* np = std::getenv("SOMIER_NO_PDL");
        h->pdl = one && pos >= 0 && !(np && np[0] == '1');
    }
    *out = h;
    return SPREAD_OK;
}

int64_t owned_nodes(const somier_s* h, const Chunk& c) {
    int64_t planes = c.size + (c.start == 1 ? 1 : 0) + (c.start + c.size == h->p.n[0] - 1 ? 1 : 0);
    return planes * h->p.n[1] * h->p.n[2];
}

// in_domain: the state's bound on max |x| is inside the exact-stats domain
// (stats_layout.hpp, xbound_ok); else the sums need not be the exact centre
// sums and the centre is reported as NaN (the sums are still exported).
void finish_stats(const somier_params* p, __int128 sums[3], unsigned long long vmax2, int64_t nodes, int64_t step,
                  somier_stats_t* out, bool in_domain = true) {
    const double N = (double)(p->n[0] * p->n[1] * p->n[2]);
    for (int c = 0; c < 3; c++) {
        out->sum_lo[c] = (uint64_t)(unsigned __int128)sums[c];
        out->sum_hi[c] = (int64_t)(sums[c] >> 64);
        out->centre[c] = in_domain ? std::ldexp((double)sums[c], -60) / N : std::nan("");
    }
    double v2;
    std::memcpy(&v2, &vmax2, sizeof v2);
    out->vmax2_bits = vmax2;
    out->vmax = std::sqrt(v2);
    out->nodes = nodes;
    out->step = step;
}

// cudaMemcpy3D between a slab (planes of 3 component blocks, row pitch ld) and
// a host grid of one component (n0 x n1 x n2, dense).
cudaError_t copy_planes(somier_t h, double* slab, int comp, int64_t slab_plane, double* host, int64_t host_plane,
                        int64_t nplanes, cudaMemcpyKind kind, cudaStream_t s) {
    return paper::copy_slab_planes(h->geom, slab, comp, slab_plane, host, host_plane, nplanes, kind, s);
}

}  // namespace

namespace paper {

spread_status check_somier_params(const somier_params* p) { return check_params(p); }

void finish_somier_stats(const somier_params* p, const __int128 sums[3], unsigned long long vmax2, int64_t nodes,
                         int64_t step, somier_stats_t* out, bool in_domain) {
    __int128 s[3] = {sums[0], sums[1], sums[2]};
    finish_stats(p, s, vmax2, nodes, step, out, in_domain);
}

spread_status encode_slab_tmap(CUtensorMap* map, const SlabGeom& g, double* base, int64_t planes, uint32_t box_k,
                               uint32_t box_j) {
    static PFN_encodeTiled encode = nullptr;
    if (!encode) {
        void* fn = nullptr;
        cudaDriverEntryPointQueryResult q;
        cudaError_t e = cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q);
        if (e != cudaSuccess || q != cudaDriverEntryPointSuccess || !fn)
            PAPER_FAIL(SPREAD_ECUDA, "somier: cuTensorMapEncodeTiled unavailable (%s)", cudaGetErrorString(e));
        encode = (PFN_encodeTiled)fn;
    }
    const cuuint64_t dims[4] = {(cuuint64_t)g.n2, (cuuint64_t)g.n1, 3, (cuuint64_t)planes};
    const cuuint64_t strides[3] = {(cuuint64_t)g.ld * 8, (cuuint64_t)(g.n1 * g.ld) * 8,
                                   (cuuint64_t)(3 * g.n1 * g.ld) * 8};
    const cuuint32_t box[4] = {box_k, box_j, 3, 1};
    const cuuint32_t estr[4] = {1, 1, 1, 1};
    // L2 promotion: 256 B by default; SOMIER_TMA_PROMO=0/64/128/256 for experiments
    CUtensorMapL2promotion promo = CU_TENSOR_MAP_L2_PROMOTION_L2_256B;
    if (const char* e = std::getenv("SOMIER_TMA_PROMO")) {
        const int v = std::atoi(e);
        promo = v == 0 ? CU_TENSOR_MAP_L2_PROMOTION_NONE
                       : v == 64 ? CU_TENSOR_MAP_L2_PROMOTION_L2_64B
                                 : v == 128 ? CU_TENSOR_MAP_L2_PROMOTION_L2_128B : CU_TENSOR_MAP_L2_PROMOTION_L2_256B;
    }
    CUresult r = encode(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 4, base, dims, strides, box, estr,
                        CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, promo,
                        CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) PAPER_FAIL(SPREAD_ECUDA, "somier: cuTensorMapEncodeTiled failed (%d)", (int)r);
    return SPREAD_OK;
}

cudaError_t copy_slab_planes(const SlabGeom& g, double* slab, int comp, int64_t slab_plane, double* host,
                             int64_t host_plane, int64_t nplanes, cudaMemcpyKind kind, cudaStream_t s) {
    const int64_t n1 = g.n1, n2 = g.n2;
    cudaMemcpy3DParms m;
    std::memset(&m, 0, sizeof m);
    cudaPitchedPtr sp = make_cudaPitchedPtr(slab + comp * n1 * g.ld, (size_t)g.ld * sizeof(double), (size_t)n2,
                                            (size_t)(3 * n1));
    cudaPitchedPtr hp = make_cudaPitchedPtr(host, (size_t)n2 * sizeof(double), (size_t)n2, (size_t)n1);
    if (kind == cudaMemcpyDeviceToHost) {
        m.srcPtr = sp;
        m.srcPos = make_cudaPos(0, 0, (size_t)slab_plane);
        m.dstPtr = hp;
        m.dstPos = make_cudaPos(0, 0, (size_t)host_plane);
    } else {
        m.srcPtr = hp;
        m.srcPos = make_cudaPos(0, 0, (size_t)host_plane);
        m.dstPtr = sp;
        m.dstPos = make_cudaPos(0, 0, (size_t)slab_plane);
    }
    m.extent = make_cudaExtent((size_t)n2 * sizeof(double), (size_t)n1, (size_t)nplanes);
    m.kind = kind;
    return cudaMemcpy3DAsync(&m, s);
}

}  // namespace paper

extern "C" {

}  // extern "C"

namespace {

// SOMIER_EXCHANGE_NCCL: after the launches of one step (one-step kernels) or
// one two-step launch (K1_TB2), every chunk boundary exchanges its planes by
// ncclSend / ncclRecv in one group: message U (the lower chunk's top planes ->
// the upper chunk's bottom halo) then message D (the upper chunk's bottom
// planes -> the lower chunk's top halo), in boundary order on every rank, so
// the k-th send from a rank to a peer matches that peer's k-th receive from it
// (same-position boundaries are self send/recv). xo / vo: the buffers of the
// new state (K1_TB2: raw deep-halo slabs; one-step: the one-halo X views, V
// unused).
spread_status nccl_exchange(somier_t h, bool tb2, int xo, int vo) {
    const paper::NcclLib& L = paper::nccl_lib();
    const int64_t ps = h->geom.plane_stride();
    const size_t pb = (size_t)ps * sizeof(double);
    const int64_t nch = (int64_t)h->chunks.size();
    std::string err;
    auto ck = [&](int r, const char* what) {
        if (r != 0 && err.empty()) err = std::string(what) + ": " + L.GetErrorString(r);
    };
    ck(L.GroupStart(), "ncclGroupStart");
    for (int64_t b = 0; b + 1 < nch; b++) {
        Chunk& lo = h->chunks[(size_t)b];
        Chunk& hi = h->chunks[(size_t)b + 1];
        struct Msg {
            double* src;
            double* dst;
            size_t bytes;
        };
        // U: lo -> hi, D: hi -> lo (X planes, then the V plane on K1_TB2 handles)
        Msg U[2], D[2];
        int nm = 1;
        if (tb2) {
            U[0] = {lo.x(xo) + lo.size * ps, hi.x(xo), 2 * pb};
            U[1] = {lo.v(vo) + lo.size * ps, hi.v(vo), pb};
            D[0] = {hi.x(xo) + 2 * ps, lo.x(xo) + (lo.size + 2) * ps, 2 * pb};
            D[1] = {hi.v(vo) + ps, lo.v(vo) + (lo.size + 1) * ps, pb};
            nm = 2;
        } else {
            U[0] = {lo.xs(xo) + lo.size * ps, hi.xs(xo), pb};
            D[0] = {hi.xs(xo) + ps, lo.xs(xo) + (lo.size + 1) * ps, pb};
        }
        const paper::ncclComm clo = h->comms[(size_t)lo.pos], chi = h->comms[(size_t)hi.pos];
        for (int m = 0; m < nm; m++) {
            if (lo.local) ck(L.Send(U[m].src, U[m].bytes, paper::kNcclUint8, hi.pos, clo, h->stream_of(lo)), "ncclSend");
            if (hi.local) ck(L.Recv(U[m].dst, U[m].bytes, paper::kNcclUint8, lo.pos, chi, h->stream_of(hi)), "ncclRecv");
        }
        for (int m = 0; m < nm; m++) {
            if (hi.local) ck(L.Send(D[m].src, D[m].bytes, paper::kNcclUint8, lo.pos, chi, h->stream_of(hi)), "ncclSend");
            if (lo.local) ck(L.Recv(D[m].dst, D[m].bytes, paper::kNcclUint8, hi.pos, clo, h->stream_of(lo)), "ncclRecv");
        }
    }
    ck(L.GroupEnd(), "ncclGroupEnd");
    if (!err.empty()) {
        if (h->sticky.empty()) h->sticky = err;
        PAPER_FAIL(SPREAD_ENCCL, "somier_step: %s", err.c_str());
    }
    return SPREAD_OK;
}

spread_status enqueue_steps(somier_t h, int64_t nsteps);
spread_status enqueue_tb2(somier_t h, bool two);
}

extern "C" {

spread_status somier_init(spread_t s, const somier_params* p, somier_t* out) {
    return init_common(s, p, -1, -1, out);
}

spread_status somier_init_on(spread_t s, const somier_params* p, const int* cuda_devices, somier_t* out) {
    if (!cuda_devices) return init_common(s, p, -1, -1, out);
    return init_common(s, p, -1, -1, out, cuda_devices);
}

spread_status somier_init_local(spread_t s, const somier_params* p, int device_pos, int cuda_device,
                                somier_t* out) {
    if (device_pos < 0) PAPER_FAIL(SPREAD_EINVAL, "somier_init_local: negative device position");
    return init_common(s, p, device_pos, cuda_device, out);
}

spread_status somier_ipc_export(somier_t h, void* buf, size_t cap, size_t* len) {
    if (!h) PAPER_FAIL(SPREAD_EINVAL, "somier_ipc_export: NULL handle");
    std::vector<IpcChunkRecord> recs;
    for (auto& c : h->chunks) {
        if (!c.local) continue;
        IpcChunkRecord r;
        std::memset(&r, 0, sizeof r);
        r.index = c.index;
        r.bytes = c.bytes;
        r.off_x0 = c.off_x[0];
        r.off_x1 = c.off_x[1];
        r.off_v = c.off_v;
        r.off_v1 = c.off_v1;
        r.off_acc = c.off_acc;
        r.off_flags = c.off_flags;
        r.off_counter = c.off_counter;
        CUDA_TRY(h, cudaSetDevice(c.device));
        CUDA_TRY(h, cudaIpcGetMemHandle(&r.handle, c.base));
        recs.push_back(r);
    }
    IpcHeader hd;
    std::memset(&hd, 0, sizeof hd);
    hd.magic = kIpcMagic;
    hd.version = kIpcVersion;
    hd.device_pos = h->local_pos;
    for (int d = 0; d < 3; d++) hd.n[d] = h->p.n[d];
    hd.nchunks = (int64_t)h->chunks.size();
    hd.chunk = h->spread.chunk;
    hd.layout = spread_layout_hash(h->spread);
    hd.nrecords = (int64_t)recs.size();
    hd.tb2 = h->tb2 ? 1 : 0;
    const size_t need = sizeof hd + recs.size() * sizeof(IpcChunkRecord);
    if (len) *len = need;
    if (!buf) return SPREAD_OK;
    if (cap < need) PAPER_FAIL(SPREAD_EINVAL, "somier_ipc_export: buffer of %zu bytes < %zu", cap, need);
    std::memcpy(buf, &hd, sizeof hd);
    if (!recs.empty()) std::memcpy((char*)buf + sizeof hd, recs.data(), recs.size() * sizeof(IpcChunkRecord));
    return SPREAD_OK;
}

spread_status somier_ipc_connect(somier_t h, const void* const* blobs, const size_t* lens, int nblobs) {
    if (!h) PAPER_FAIL(SPREAD_EINVAL, "somier_ipc_connect: NULL handle");
    if (!h->multi_process) PAPER_FAIL(SPREAD_ESTATE, "somier_ipc_connect: handle is not multi-process");
    if (nblobs < 0 || (nblobs > 0 && (!blobs || !lens))) PAPER_FAIL(SPREAD_EINVAL, "somier_ipc_connect: bad blob list");
    std::map<int64_t, IpcChunkRecord> remote;
    for (int b = 0; b < nblobs; b++) {
        if (!blobs[b] || lens[b] < sizeof(IpcHeader)) PAPER_FAIL(SPREAD_EINVAL, "somier_ipc_connect: blob %d too short", b);
        IpcHeader hd;
        std::memcpy(&hd, blobs[b], sizeof hd);
        if (hd.magic != kIpcMagic || hd.version != kIpcVersion)
            PAPER_FAIL(SPREAD_EINVAL, "somier_ipc_connect: blob %d is not a somier IPC blob", b);
        if (hd.n[0] != h->p.n[0] || hd.n[1] != h->p.n[1] || hd.n[2] != h->p.n[2] ||
            hd.nchunks != (int64_t)h->chunks.size() || hd.chunk != h->spread.chunk ||
            hd.layout != spread_layout_hash(h->spread))
            PAPER_FAIL(SPREAD_EINVAL, "somier_ipc_connect: blob %d describes another grid or spread", b);
        if (hd.tb2 != (h->tb2 ? 1 : 0))
            PAPER_FAIL(SPREAD_EINVAL, "somier_ipc_connect: blob %d uses the other K1 slab layout (K1_TB2 vs one-step): "
                       "the processes resolved the kernel differently; pass the same explicit kernel", b);
        if (lens[b] != sizeof hd + (size_t)hd.nrecords * sizeof(IpcChunkRecord))
            PAPER_FAIL(SPREAD_EINVAL, "somier_ipc_connect: blob %d has a bad length", b);
        if (hd.device_pos == h->local_pos) continue;
        for (int64_t r = 0; r < hd.nrecords; r++) {
            IpcChunkRecord rec;
            std::memcpy(&rec, (const char*)blobs[b] + sizeof hd + r * sizeof rec, sizeof rec);
            if (rec.index < 0 || rec.index >= (int64_t)h->chunks.size())
                PAPER_FAIL(SPREAD_EINVAL, "somier_ipc_connect: chunk index out of range");
            remote[rec.index] = rec;
        }
    }
    CUDA_TRY(h, cudaSetDevice(h->devs[h->local_pos].device));
    for (size_t c = 0; c < h->chunks.size(); c++) {
        Chunk& me = h->chunks[c];
        if (!me.local) continue;
        for (int side = -1; side <= 1; side += 2) {
            int64_t nb = (int64_t)c + side;
            if (nb < 0 || nb >= (int64_t)h->chunks.size()) continue;
            Chunk& o = h->chunks[nb];
            if (o.local || o.remote_base) continue;
            auto it = remote.find(nb);
            if (it == remote.end())
                PAPER_FAIL(SPREAD_EINVAL, "somier_ipc_connect: no process exported neighbour chunk %lld", (long long)nb);
            const IpcChunkRecord& rec = it->second;
            void* ptr = nullptr;
            CUDA_TRY(h, cudaIpcOpenMemHandle(&ptr, rec.handle, cudaIpcMemLazyEnablePeerAccess));
            o.remote_base = ptr;
            o.bytes = rec.bytes;
            o.off_x[0] = rec.off_x0;
            o.off_x[1] = rec.off_x1;
            o.off_v = rec.off_v;
            o.off_v1 = rec.off_v1;
            o.view_off = h->tb2 ? h->geom.plane_stride() : 0;
            o.off_acc = rec.off_acc;
            o.off_flags = rec.off_flags;
            o.off_counter = rec.off_counter;
        }
    }
    // the NCCL exchange does not use the neighbours' memory: it still needs its communicator
    h->connected = h->p.exchange != SOMIER_EXCHANGE_NCCL || h->comms[(size_t)h->local_pos] != nullptr;
    return SPREAD_OK;
}

spread_status somier_step(somier_t h, int64_t nsteps) {
    PAPER_NVTX("somier_step");
    if (!h) PAPER_FAIL(SPREAD_EINVAL, "somier_step: NULL handle");
    if (nsteps < 0) PAPER_FAIL(SPREAD_EINVAL, "somier_step: nsteps < 0");
    if (!h->connected) PAPER_FAIL(SPREAD_ESTATE, "somier_step: remote neighbour chunks not connected (somier_ipc_connect)");
    if (!h->sticky.empty()) PAPER_FAIL(SPREAD_ECUDA, "%s", h->sticky.c_str());
    if (h->tb2) {
        // K1_TB2: pairs of steps; a leftover single step runs the same kernel
        // in one-step mode (same slab layout and halo protocol). On one stream
        // without flags, two consecutive pairs (four steps) are captured once
        // per (buffer parity, step parity) -- everything a launch depends on --
        // and replayed as a CUDA graph; the handle's first pair runs eagerly
        // (lazy host-side state is set up outside any capture).
        if (h->graph_ok && !h->timing && nsteps >= 4) {
            if (h->launches == 0) {
                spread_status st = enqueue_tb2(h, true);
                if (st != SPREAD_OK) return st;
                nsteps -= 2;
            }
            DevCtx& d = h->devs[h->graph_pos];
            int64_t nloc = 0;
            for (auto& c : h->chunks) nloc += c.local ? 1 : 0;
            while (nsteps >= 4) {
                cudaGraphExec_t& ge = h->tb2_graph[(h->xbuf & 1) * 2 + (int)(h->step & 1)];
                CUDA_TRY(h, cudaSetDevice(d.device));
                if (!ge) {
                    const int64_t s0 = h->step, l0 = h->launches;
                    const int xb0 = h->xbuf, vb0 = h->vbuf;
                    CUDA_TRY(h, cudaStreamBeginCapture(d.stream, cudaStreamCaptureModeThreadLocal));
                    spread_status st = enqueue_tb2(h, true);
                    if (st == SPREAD_OK) st = enqueue_tb2(h, true);
                    h->step = s0;
                    h->launches = l0;
                    h->xbuf = xb0;
                    h->vbuf = vb0;
                    cudaGraph_t g = nullptr;
                    cudaError_t e = cudaStreamEndCapture(d.stream, &g);
                    if (st != SPREAD_OK) return st;
                    if (e != cudaSuccess) return cuda_fail(h, e, "somier_step: graph capture");
                    e = cudaGraphInstantiate(&ge, g, 0);
                    cudaGraphDestroy(g);
                    if (e != cudaSuccess) return cuda_fail(h, e, "somier_step: graph instantiate");
                    CUDA_TRY(h, cudaSetDevice(d.device));
                }
                CUDA_TRY(h, cudaGraphLaunch(ge, d.stream));
                h->step += 4;
                h->launches += 2 * nloc;
                nsteps -= 4;
            }
        }
        for (; nsteps >= 2; nsteps -= 2) {
            spread_status st = enqueue_tb2(h, true);
            if (st != SPREAD_OK) return st;
        }
        return nsteps ? enqueue_tb2(h, false) : SPREAD_OK;
    }
    // All chunks on one stream (no cross-stream flags): the launches of two
    // consecutive steps depend only on the buffer parity, so a CUDA graph of an
    // (even, odd) step pair is captured once and replayed.
    if (h->graph_ok && !h->timing && nsteps >= 2) {
        if (h->step & 1) {
            spread_status st = enqueue_steps(h, 1);
            if (st != SPREAD_OK) return st;
            nsteps--;
        }
        DevCtx& d = h->devs[h->graph_pos];
        if (!h->graph_exec && nsteps >= 2) {
            CUDA_TRY(h, cudaSetDevice(d.device));
            CUDA_TRY(h, cudaStreamBeginCapture(d.stream, cudaStreamCaptureModeThreadLocal));
            const int64_t s0 = h->step, l0 = h->launches;
            spread_status st = enqueue_steps(h, 2);
            h->step = s0;
            h->launches = l0;
            cudaGraph_t g = nullptr;
            cudaError_t e = cudaStreamEndCapture(d.stream, &g);
            if (st != SPREAD_OK) return st;
            if (e != cudaSuccess) return cuda_fail(h, e, "somier_step: graph capture");
            e = cudaGraphInstantiate(&h->graph_exec, g, 0);
            cudaGraphDestroy(g);
            if (e != cudaSuccess) return cuda_fail(h, e, "somier_step: graph instantiate");
        }
        if (h->graph_exec) {
            CUDA_TRY(h, cudaSetDevice(d.device));
            int64_t nloc = 0;
            for (auto& c : h->chunks) nloc += c.local ? 1 : 0;
            for (; nsteps >= 2; nsteps -= 2) {
                CUDA_TRY(h, cudaGraphLaunch(h->graph_exec, d.stream));
                h->step += 2;
                h->launches += 2 * nloc;
            }
        }
    }
    return enqueue_steps(h, nsteps);
}

}  // extern "C"

namespace {

spread_status enqueue_steps(somier_t h, int64_t nsteps) {
    const int64_t nch = (int64_t)h->chunks.size();
    int cur_dev = -1;
    for (int64_t s = 0; s < nsteps; s++) {
        const int64_t t = h->step;
        const int cur = h->xbuf, nxt = cur ^ 1;       // X buffers
        const int vb = h->vbuf;  // V buffer
        for (int64_t c = 0; c < nch; c++) {
            Chunk& me = h->chunks[c];
            if (!me.local) continue;
            if (me.device != cur_dev) {
                CUDA_TRY(h, cudaSetDevice(me.device));
                cur_dev = me.device;
            }
            cudaStream_t st = h->stream_of(me);
            const Chunk* left = c > 0 ? &h->chunks[c - 1] : nullptr;
            const Chunk* right = c + 1 < nch ? &h->chunks[c + 1] : nullptr;
            const bool fl = left && h->needs_flags(me, *left);
            const bool fr = right && h->needs_flags(me, *right);
            somier_s::TimingRec tr{};
            if (h->timing) {
                spread_status ts = timing_begin(h, me.device, st, &tr);
                if (ts != SPREAD_OK) return ts;
            }
            // wait until the neighbours finished step t-1 (their halo stores into
            // my X_t are visible, and they no longer read the halo buffer I am
            // about to write): flags[0] = from_left, flags[1] = from_right.
            if (t > 0 && fl) {
                CUresult r = h->wait_value64((CUstream)st, (CUdeviceptr)&me.flags()[0], (cuuint64_t)t,
                                             CU_STREAM_WAIT_VALUE_GEQ | h->devs[me.pos].wait_flush);
                if (r != CUDA_SUCCESS) PAPER_FAIL(SPREAD_ECUDA, "somier_step: cuStreamWaitValue64 failed (%d)", (int)r);
            }
            if (t > 0 && fr) {
                CUresult r = h->wait_value64((CUstream)st, (CUdeviceptr)&me.flags()[1], (cuuint64_t)t,
                                             CU_STREAM_WAIT_VALUE_GEQ | h->devs[me.pos].wait_flush);
                if (r != CUDA_SUCCESS) PAPER_FAIL(SPREAD_ECUDA, "somier_step: cuStreamWaitValue64 failed (%d)", (int)r);
            }
            paper::StepArgs a;
            std::memset(&a, 0, sizeof a);
            a.fma = h->p.math == SOMIER_MATH_FMA ? 1 : 0;
            a.x_cur = me.xs(cur);
            a.x_nxt = me.xs(nxt);
            a.v = me.vs(vb);
            const bool fused = h->p.exchange == SOMIER_EXCHANGE_FUSED;
            a.lo_dst = left && fused ? left->xs(nxt) + (left->size + 1) * h->geom.plane_stride() : nullptr;
            a.hi_dst = right && fused ? right->xs(nxt) : nullptr;
            a.g = h->geom_of(me);
            a.K = h->p.k_spring;
            a.L = h->p.rest_len;
            a.M = h->p.mass;
            a.dt = h->p.dt;
            a.step_word = me.step_word();  // the kernel takes its ring slots from the device step counter
            a.acc_ring = me.acc();
            a.signal_lo = fl && fused ? &left->flags()[1] : nullptr;
            a.signal_hi = fr && fused ? &right->flags()[0] : nullptr;
            a.signal_value = (unsigned long long)(t + 1);
            a.done_counter = me.counter();
            a.side_counter = me.side_counter();
            a.tmap_x_cur = &me.tmap_x[cur];
            a.tmap_v = &me.tmap_v[vb];
            a.tmap_x2_cur = &me.tmap_x2[cur];
            a.tmap_v2 = &me.tmap_v2[vb];
            a.pdl = h->pdl && !h->timing ? 1 : 0;
            if (h->timing) CUDA_TRY(h, cudaEventRecord(tr.b, st));
            CUDA_TRY(h, paper::launch_k1(h->variant(), a, h->unit_mass(), st));
            if (h->p.exchange == SOMIER_EXCHANGE_COPY) {
                // SOMIER_EXCHANGE_COPY: the boundary planes of X_{t+1} into the
                // neighbours' halo planes after the kernel, then their flags
                const int64_t ps = h->geom.plane_stride();
                const size_t pb = (size_t)ps * sizeof(double);
                if (left)
                    CUDA_TRY(h, cudaMemcpyAsync(left->xs(nxt) + (left->size + 1) * ps, me.xs(nxt) + ps, pb,
                                                cudaMemcpyDeviceToDevice, st));
                if (right)
                    CUDA_TRY(h, cudaMemcpyAsync(right->xs(nxt), me.xs(nxt) + me.size * ps, pb,
                                                cudaMemcpyDeviceToDevice, st));
                spread_status ss = signal_after(h, st, fl ? &left->flags()[1] : nullptr,
                                                fr ? &right->flags()[0] : nullptr, (unsigned long long)(t + 1));
                if (ss != SPREAD_OK) return ss;
            }
            if (h->timing) {
                CUDA_TRY(h, cudaEventRecord(tr.c, st));
                h->trecs.push_back(tr);
            }
            h->launches++;
        }
        if (h->p.exchange == SOMIER_EXCHANGE_NCCL) {
            spread_status ns = nccl_exchange(h, false, nxt, 0);
            if (ns != SPREAD_OK) return ns;
        }
        h->step++;
        h->xbuf ^= 1;
    }
    return SPREAD_OK;
}

// K1_TB2: steps t, t+1 (two) or step t in one launch per local chunk. The
// launch reads X_t / V_t (buffers xbuf / vbuf) with their deep halos and
// writes the other buffers, its boundary planes also into the neighbours'
// other buffers; flags as in enqueue_steps (the neighbours finished the launch
// that produced step t: my halo planes of X_t / V_t are written, and they no
// longer read their buffers I write into). Stats of both steps go to the
// history ring (slots from the device step word).
spread_status enqueue_tb2(somier_t h, bool two) {
    const int64_t nch = (int64_t)h->chunks.size();
    const int64_t t = h->step, t_end = t + (two ? 2 : 1);
    const int cur = h->xbuf, vb = h->vbuf;
    const int64_t ps = h->geom.plane_stride();
    int cur_dev = -1;
    for (int64_t c = 0; c < nch; c++) {
        Chunk& me = h->chunks[c];
        if (!me.local) continue;
        if (me.device != cur_dev) {
            CUDA_TRY(h, cudaSetDevice(me.device));
            cur_dev = me.device;
        }
        cudaStream_t st = h->stream_of(me);
        const Chunk* left = c > 0 ? &h->chunks[c - 1] : nullptr;
        const Chunk* right = c + 1 < nch ? &h->chunks[c + 1] : nullptr;
        const bool fl = left && h->needs_flags(me, *left);
        const bool fr = right && h->needs_flags(me, *right);
        somier_s::TimingRec tr{};
        if (h->timing) {
            spread_status ts = timing_begin(h, me.device, st, &tr);
            if (ts != SPREAD_OK) return ts;
        }
        for (int side = 0; side < 2; side++) {
            if (t == 0 || !(side ? fr : fl)) continue;
            CUresult r = h->wait_value64((CUstream)st, (CUdeviceptr)&me.flags()[side], (cuuint64_t)t,
                                         CU_STREAM_WAIT_VALUE_GEQ | h->devs[me.pos].wait_flush);
            if (r != CUDA_SUCCESS) PAPER_FAIL(SPREAD_ECUDA, "somier_step: cuStreamWaitValue64 failed (%d)", (int)r);
        }
        paper::StepArgs a;
        std::memset(&a, 0, sizeof a);
        a.fma = h->p.math == SOMIER_MATH_FMA ? 1 : 0;
        a.x_cur = me.x(cur);
        a.v = me.v(vb);
        a.g = h->geom_of(me);
        a.K = h->p.k_spring;
        a.L = h->p.rest_len;
        a.M = h->p.mass;
        a.dt = h->p.dt;
        a.step_word = me.step_word();
        a.acc_ring = me.acc();
        a.tmap_x_cur = &me.tmap_xt[cur];
        a.tmap_v = &me.tmap_vt[vb];
        paper::Tb2Out o;
        std::memset(&o, 0, sizeof o);
        o.x_out = me.x(cur ^ 1);
        o.v_out = me.v(vb ^ 1);
        o.two = two;
        // neighbours' deep halo planes in THEIR out buffers: left X planes of
        // global i = start, start+1 (its raw planes size+2, size+3), V plane
        // of i = start (raw size+1); right X planes start+size-2, -1 (raw 0, 1),
        // V plane start+size-1 (raw 0)
        const bool fused = h->p.exchange == SOMIER_EXCHANGE_FUSED;
        if (left && fused) {
            a.lo_dst = left->x(cur ^ 1) + (left->size + 2) * ps;
            o.lo_vdst = left->v(vb ^ 1) + (left->size + 1) * ps;
        }
        if (right && fused) {
            a.hi_dst = right->x(cur ^ 1);
            o.hi_vdst = right->v(vb ^ 1);
        }
        a.signal_lo = fl && fused ? &left->flags()[1] : nullptr;
        a.signal_hi = fr && fused ? &right->flags()[0] : nullptr;
        a.signal_value = (unsigned long long)t_end;
        a.done_counter = me.counter();
        a.side_counter = me.side_counter();
        if (h->timing) CUDA_TRY(h, cudaEventRecord(tr.b, st));
        CUDA_TRY(h, paper::launch_k1_tb2(a, o, h->unit_mass(), st));
        if (h->p.exchange == SOMIER_EXCHANGE_COPY) {
            // SOMIER_EXCHANGE_COPY: the first two X planes and the first V plane
            // of the new state to the left neighbour's deep halo, the last two /
            // last one to the right's (the planes the fused kernel stores), then
            // the flags
            const size_t pb = (size_t)ps * sizeof(double);
            if (left) {
                CUDA_TRY(h, cudaMemcpyAsync(left->x(cur ^ 1) + (left->size + 2) * ps, me.x(cur ^ 1) + 2 * ps, 2 * pb,
                                            cudaMemcpyDeviceToDevice, st));
                CUDA_TRY(h, cudaMemcpyAsync(left->v(vb ^ 1) + (left->size + 1) * ps, me.v(vb ^ 1) + ps, pb,
                                            cudaMemcpyDeviceToDevice, st));
            }
            if (right) {
                CUDA_TRY(h, cudaMemcpyAsync(right->x(cur ^ 1), me.x(cur ^ 1) + me.size * ps, 2 * pb,
                                            cudaMemcpyDeviceToDevice, st));
                CUDA_TRY(h, cudaMemcpyAsync(right->v(vb ^ 1), me.v(vb ^ 1) + me.size * ps, pb,
                                            cudaMemcpyDeviceToDevice, st));
            }
            spread_status ss = signal_after(h, st, fl ? &left->flags()[1] : nullptr, fr ? &right->flags()[0] : nullptr,
                                            (unsigned long long)t_end);
            if (ss != SPREAD_OK) return ss;
        }
        if (h->timing) {
            CUDA_TRY(h, cudaEventRecord(tr.c, st));
            h->trecs.push_back(tr);
        }
        h->launches++;
    }
    if (h->p.exchange == SOMIER_EXCHANGE_NCCL) {
        spread_status ns = nccl_exchange(h, true, cur ^ 1, vb ^ 1);
        if (ns != SPREAD_OK) return ns;
    }
    h->step = t_end;
    h->xbuf ^= 1;
    h->vbuf ^= 1;
    return SPREAD_OK;
}

}  // namespace

extern "C" {

spread_status somier_sync(somier_t h) {
    PAPER_NVTX("somier_sync");
    if (!h) PAPER_FAIL(SPREAD_EINVAL, "somier_sync: NULL handle");
    return sync_all(h);
}

static_assert(SOMIER_STATS_HISTORY == paper::kStatsHistory, "somier.h history depth");

spread_status somier_stats_history(somier_t h, int64_t first_step, int64_t count, somier_stats_t* out) {
    PAPER_NVTX("somier_stats_history");
    if (!h || (count > 0 && !out)) PAPER_FAIL(SPREAD_EINVAL, "somier_stats_history: NULL argument");
    if (count < 0) PAPER_FAIL(SPREAD_EINVAL, "somier_stats_history: count < 0");
    const int64_t lo = std::max(h->hist_first, h->step - (int64_t)paper::kStatsHistory + 1);
    if (count > 0 && (first_step < lo || first_step + count - 1 > h->step))
        PAPER_FAIL(SPREAD_EINVAL, "somier_stats_history: steps [%lld, %lld] outside the history [%lld, %lld]",
                   (long long)first_step, (long long)(first_step + count - 1), (long long)lo, (long long)h->step);
    spread_status st = sync_all(h);
    if (st != SPREAD_OK) return st;
    if (count == 0) return SPREAD_OK;
    std::vector<__int128> sums((size_t)count * 3, 0);
    std::vector<unsigned long long> vmax2((size_t)count, 0ull), xmax((size_t)count, 0ull);
    int64_t nodes = 0;
    std::vector<paper::StatsAccum> acc(paper::kStatsRing + 1);
    for (auto& c : h->chunks) {
        if (!c.local) continue;
        CUDA_TRY(h, cudaSetDevice(c.device));
        CUDA_TRY(h, cudaMemcpy(acc.data(), c.acc(), acc.size() * sizeof(paper::StatsAccum), cudaMemcpyDeviceToHost));
        for (int64_t i = 0; i < count; i++) {
            for (int q : {paper::ring_slot((unsigned long long)(first_step + i)), paper::kStatsRing}) {
                for (int d = 0; d < 3; d++)
                    sums[(size_t)(3 * i + d)] += (__int128)(((unsigned __int128)acc[q].hi[d] << 64) | acc[q].lo[d]);
                vmax2[(size_t)i] = std::max(vmax2[(size_t)i], (unsigned long long)acc[q].vmax2);
                xmax[(size_t)i] = std::max(xmax[(size_t)i], (unsigned long long)acc[q].xmax);
            }
        }
        nodes += owned_nodes(h, c);
    }
    for (int64_t i = 0; i < count; i++)
    {
        double B;
        const unsigned long long b = xmax[(size_t)i];
        std::memcpy(&B, &b, sizeof B);  // the bound's IEEE bits (NaN bits order above inf)
        finish_stats(&h->p, &sums[(size_t)(3 * i)], vmax2[(size_t)i], nodes, first_step + i, &out[i],
                     paper::xbound_ok(B));
    }
    return SPREAD_OK;
}

spread_status somier_stats(somier_t h, somier_stats_t* out) {
    if (!h || !out) PAPER_FAIL(SPREAD_EINVAL, "somier_stats: NULL argument");
    return somier_stats_history(h, h->step, 1, out);
}

spread_status somier_stats_combine(const somier_stats_t* parts, int n, const somier_params* p, somier_stats_t* out) {
    if (!parts || n < 1 || !p || !out) PAPER_FAIL(SPREAD_EINVAL, "somier_stats_combine: bad arguments");
    __int128 sums[3] = {0, 0, 0};
    unsigned long long vmax2 = 0;
    int64_t nodes = 0;
    bool in_domain = true;  // a partial outside the exact-stats domain reports a NaN centre
    for (int i = 0; i < n; i++) {
        if (parts[i].step != parts[0].step)
            PAPER_FAIL(SPREAD_EINVAL, "somier_stats_combine: partials of different steps");
        for (int d = 0; d < 3; d++) in_domain = in_domain && !std::isnan(parts[i].centre[d]);
        for (int d = 0; d < 3; d++)
            sums[d] += (__int128)(((unsigned __int128)(uint64_t)parts[i].sum_hi[d] << 64) | parts[i].sum_lo[d]);
        vmax2 = std::max(vmax2, (unsigned long long)parts[i].vmax2_bits);
        nodes += parts[i].nodes;
    }
    finish_stats(p, sums, vmax2, nodes, parts[0].step, out, in_domain);
    return SPREAD_OK;
}

spread_status somier_read_planes(somier_t h, int64_t i0, int64_t count, double* x, double* y, double* z, double* vx,
                                 double* vy, double* vz) {
    PAPER_NVTX("somier_read_planes");
    if (!h) PAPER_FAIL(SPREAD_EINVAL, "somier_read_planes: NULL handle");
    const int64_t n0 = h->p.n[0];
    if (i0 < 0 || count < 0 || i0 + count > n0)
        PAPER_FAIL(SPREAD_EINVAL, "somier_read_planes: planes [%lld, %lld) outside [0, %lld)", (long long)i0,
                   (long long)(i0 + count), (long long)n0);
    spread_status st = sync_all(h);
    if (st != SPREAD_OK) return st;
    double* X[3] = {x, y, z};
    double* V[3] = {vx, vy, vz};
    const int cur = h->xbuf;
    const size_t plane = (size_t)(h->p.n[1] * h->p.n[2]);
    const int64_t i1 = i0 + count;
    // host grids hold planes [i0, i1): global plane i -> host plane i - i0
    for (auto& c : h->chunks) {
        if (!c.local) continue;
        CUDA_TRY(h, cudaSetDevice(c.device));
        cudaStream_t s = h->stream_of(c);
        // owned planes [start, start+size) plus the fixed end planes held as halos
        struct Span {
            int64_t lo, hi, slab0;  // global planes [lo, hi) <- X slab plane slab0 + (i - lo)
            bool fixed;
        } spans[3] = {{c.start, c.start + c.size, 1, false},
                      {0, c.start == 1 ? 1 : 0, 0, true},
                      {n0 - 1, (c.start + c.size == n0 - 1) ? n0 : n0 - 1, c.size + 1, true}};
        for (const Span& sp : spans) {
            const int64_t lo = std::max(sp.lo, i0), hi = std::min(sp.hi, i1);
            if (lo >= hi) continue;
            for (int d = 0; d < 3; d++) {
                if (X[d])
                    CUDA_TRY(h, copy_planes(h, c.xs(cur), d, sp.slab0 + (lo - sp.lo), X[d], lo - i0, hi - lo,
                                            cudaMemcpyDeviceToHost, s));
                if (V[d]) {
                    if (sp.fixed)  // fixed end planes have zero velocity
                        std::memset(V[d] + (size_t)(lo - i0) * plane, 0, (size_t)(hi - lo) * plane * sizeof(double));
                    else
                        CUDA_TRY(h, copy_planes(h, c.vs(h->vbuf), d, lo - c.start, V[d], lo - i0, hi - lo,
                                                cudaMemcpyDeviceToHost, s));
                }
            }
        }
    }
    return sync_all(h);
}

spread_status somier_read(somier_t h, double* x, double* y, double* z, double* vx, double* vy, double* vz) {
    if (!h) PAPER_FAIL(SPREAD_EINVAL, "somier_read: NULL handle");
    return somier_read_planes(h, 0, h->p.n[0], x, y, z, vx, vy, vz);
}

spread_status somier_load(somier_t h, const double* x, const double* y, const double* z, const double* vx,
                          const double* vy, const double* vz) {
    PAPER_NVTX("somier_load");
    if (!h) PAPER_FAIL(SPREAD_EINVAL, "somier_load: NULL handle");
    if (!x || !y || !z || !vx || !vy || !vz) PAPER_FAIL(SPREAD_EINVAL, "somier_load: NULL grid");
    if (!h->sticky.empty()) PAPER_FAIL(SPREAD_ECUDA, "%s", h->sticky.c_str());
    const double* X[3] = {x, y, z};
    const double* V[3] = {vx, vy, vz};
    const int cur = h->xbuf;
    for (auto& c : h->chunks) {
        if (!c.local) continue;
        CUDA_TRY(h, cudaSetDevice(c.device));
        cudaStream_t s = h->stream_of(c);
        for (int d = 0; d < 3; d++) {
            CUDA_TRY(h, copy_planes(h, c.xs(cur), d, 0, const_cast<double*>(X[d]), c.start - 1, c.size + 2,
                                    cudaMemcpyHostToDevice, s));
            CUDA_TRY(h, copy_planes(h, c.vs(h->vbuf), d, 0, const_cast<double*>(V[d]), c.start, c.size,
                                    cudaMemcpyHostToDevice, s));
            if (h->tb2) {
                // the deep halo: X planes start-2, start+size+1 and V planes
                // start-1, start+size where they are grid planes that move
                const int64_t n0 = h->p.n[0];
                if (c.start - 2 >= 0)
                    CUDA_TRY(h, copy_planes(h, c.x(cur), d, 0, const_cast<double*>(X[d]), c.start - 2, 1,
                                            cudaMemcpyHostToDevice, s));
                if (c.start + c.size + 1 <= n0 - 1)
                    CUDA_TRY(h, copy_planes(h, c.x(cur), d, c.size + 3, const_cast<double*>(X[d]),
                                            c.start + c.size + 1, 1, cudaMemcpyHostToDevice, s));
                if (c.start - 1 >= 1)
                    CUDA_TRY(h, copy_planes(h, c.v(h->vbuf), d, 0, const_cast<double*>(V[d]), c.start - 1, 1,
                                            cudaMemcpyHostToDevice, s));
                if (c.start + c.size <= n0 - 2)
                    CUDA_TRY(h, copy_planes(h, c.v(h->vbuf), d, c.size + 1, const_cast<double*>(V[d]),
                                            c.start + c.size, 1, cudaMemcpyHostToDevice, s));
            }
        }
        // the X_{t+1} buffer must hold the same fixed nodes (never written by a step)
        CUDA_TRY(h, cudaMemcpyAsync(c.x(cur ^ 1), c.x(cur), c.xbytes, cudaMemcpyDeviceToDevice, s));
        spread_status st = reset_stats(h, c);
        if (st != SPREAD_OK) return st;
    }
    // The copy above replaces the chunk's whole X_{t+1} buffer, halo planes
    // included, which the neighbours' next step stores into from THEIR streams
    // (their flag waits are already satisfied): order every other position's
    // stream after this position's load. Other processes cannot be ordered
    // from here: multi-process loads complete before returning (the caller's
    // barrier then orders them, include/somier.h).
    if (h->multi_process) return sync_all(h);
    std::vector<cudaEvent_t> evs;
    spread_status st = SPREAD_OK;
    for (size_t q = 0; q < h->devs.size() && st == SPREAD_OK; q++) {
        DevCtx& d = h->devs[q];
        if (!d.stream) continue;
        cudaEvent_t ev = nullptr;
        cudaError_t e = cudaSetDevice(d.device);
        if (e == cudaSuccess) e = cudaEventCreateWithFlags(&ev, cudaEventDisableTiming);
        if (e == cudaSuccess) evs.push_back(ev);
        if (e == cudaSuccess) e = cudaEventRecord(ev, d.stream);
        if (e != cudaSuccess) st = cuda_fail(h, e, "somier_load: event");
    }
    for (size_t q = 0, i = 0; q < h->devs.size() && st == SPREAD_OK; q++) {
        DevCtx& d = h->devs[q];
        if (!d.stream) continue;
        cudaError_t e = cudaSetDevice(d.device);
        for (size_t r = 0; r < evs.size() && e == cudaSuccess; r++)
            if (r != i) e = cudaStreamWaitEvent(d.stream, evs[r], 0);
        if (e != cudaSuccess) st = cuda_fail(h, e, "somier_load: stream wait");
        i++;
    }
    for (cudaEvent_t ev : evs) cudaEventDestroy(ev);
    return st;
}

spread_status somier_set_stream(somier_t h, int device_pos, void* stream) {
    if (!h) PAPER_FAIL(SPREAD_EINVAL, "somier_set_stream: NULL handle");
    if (device_pos < 0 || device_pos >= (int)h->devs.size() || !h->devs[device_pos].own)
        PAPER_FAIL(SPREAD_EINVAL, "somier_set_stream: no local chunk at list position %d", device_pos);
    DevCtx& d = h->devs[device_pos];
    cudaStream_t next = stream ? (cudaStream_t)stream : d.own;
    if (next != d.stream) {
        // order the new stream after everything already enqueued on the old one
        cudaEvent_t ev;
        CUDA_TRY(h, cudaSetDevice(d.device));
        CUDA_TRY(h, cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
        CUDA_TRY(h, cudaEventRecord(ev, d.stream));
        CUDA_TRY(h, cudaStreamWaitEvent(next, ev, 0));
        CUDA_TRY(h, cudaEventDestroy(ev));
        d.stream = next;
    }
    return SPREAD_OK;
}

spread_status somier_get_stream(somier_t h, int device_pos, void** stream) {
    if (!h || !stream) PAPER_FAIL(SPREAD_EINVAL, "somier_get_stream: NULL argument");
    if (device_pos < 0 || device_pos >= (int)h->devs.size() || !h->devs[device_pos].own)
        PAPER_FAIL(SPREAD_EINVAL, "somier_get_stream: no local chunk at list position %d", device_pos);
    *stream = (void*)h->devs[device_pos].stream;
    return SPREAD_OK;
}

spread_status somier_step_count(somier_t h, int64_t* steps) {
    if (!h || !steps) PAPER_FAIL(SPREAD_EINVAL, "somier_step_count: NULL argument");
    *steps = h->step;
    return SPREAD_OK;
}

spread_status somier_local_chunks(somier_t h, int64_t* nchunks) {
    if (!h || !nchunks) PAPER_FAIL(SPREAD_EINVAL, "somier_local_chunks: NULL argument");
    int64_t n = 0;
    for (auto& c : h->chunks) n += c.local ? 1 : 0;
    *nchunks = n;
    return SPREAD_OK;
}

spread_status somier_launch_count(somier_t h, int64_t* launches) {
    if (!h || !launches) PAPER_FAIL(SPREAD_EINVAL, "somier_launch_count: NULL argument");
    *launches = h->launches;
    return SPREAD_OK;
}

spread_status somier_kernel_in_use(somier_t h, int32_t* kernel) {
    if (!h || !kernel) PAPER_FAIL(SPREAD_EINVAL, "somier_kernel_in_use: NULL argument");
    if (h->tb2) {
        *kernel = SOMIER_K1_TB2;
        return SPREAD_OK;
    }
    switch (h->variant()) {
        case paper::K1Variant::Direct: *kernel = SOMIER_K1_DIRECT; break;
        case paper::K1Variant::March: *kernel = SOMIER_K1_MARCH; break;
        default: *kernel = SOMIER_K1_MARCH2; break;
    }
    return SPREAD_OK;
}

spread_status somier_device_bytes(somier_t h, int64_t* bytes) {
    if (!h || !bytes) PAPER_FAIL(SPREAD_EINVAL, "somier_device_bytes: NULL argument");
    int64_t b = 0;
    for (auto& c : h->chunks)
        if (c.local) b += (int64_t)c.bytes;
    *bytes = b;
    return SPREAD_OK;
}

spread_status somier_nccl_unique_id(void* id_out) {
    if (!id_out) PAPER_FAIL(SPREAD_EINVAL, "somier_nccl_unique_id: NULL argument");
    const paper::NcclLib& L = paper::nccl_lib();
    if (!L.ok) PAPER_FAIL(SPREAD_ENOTSUP, "somier_nccl_unique_id: NCCL unavailable (%s)", L.error.c_str());
    paper::NcclUniqueId id;
    const int r = L.GetUniqueId(&id);
    if (r != 0) PAPER_FAIL(SPREAD_ENCCL, "ncclGetUniqueId: %s", L.GetErrorString(r));
    std::memcpy(id_out, &id, sizeof id);
    return SPREAD_OK;
}

spread_status somier_nccl_connect(somier_t h, const void* id, int nranks) {
    if (!h || !id) PAPER_FAIL(SPREAD_EINVAL, "somier_nccl_connect: NULL argument");
    if (!h->multi_process || h->p.exchange != SOMIER_EXCHANGE_NCCL)
        PAPER_FAIL(SPREAD_ESTATE, "somier_nccl_connect: not a multi-process handle with the NCCL exchange");
    if (nranks != (int)h->devs.size())
        PAPER_FAIL(SPREAD_EINVAL, "somier_nccl_connect: %d ranks for a list of %d positions", nranks,
                   (int)h->devs.size());
    const paper::NcclLib& L = paper::nccl_lib();
    paper::NcclUniqueId uid;
    std::memcpy(&uid, id, sizeof uid);
    CUDA_TRY(h, cudaSetDevice(h->devs[(size_t)h->local_pos].device));
    const int r = L.CommInitRank(&h->comms[(size_t)h->local_pos], nranks, uid, h->local_pos);
    if (r != 0) PAPER_FAIL(SPREAD_ENCCL, "ncclCommInitRank: %s", L.GetErrorString(r));
    h->connected = true;
    return SPREAD_OK;
}

spread_status somier_set_timing(somier_t h, int on) {
    if (!h) PAPER_FAIL(SPREAD_EINVAL, "somier_set_timing: NULL handle");
    h->timing = on != 0;
    return SPREAD_OK;
}

spread_status somier_take_timing(somier_t h, somier_timing_t* out) {
    if (!h || !out) PAPER_FAIL(SPREAD_EINVAL, "somier_take_timing: NULL argument");
    spread_status st = sync_all(h);
    if (st != SPREAD_OK) return st;
    out->launches = 0;
    out->wait_ms = out->kernel_ms = 0.0;
    out->wait_max_ms = out->kernel_max_ms = 0.0;
    for (auto& r : h->trecs) {
        float w = 0.f, k = 0.f;
        CUDA_TRY(h, cudaSetDevice(r.device));
        CUDA_TRY(h, cudaEventElapsedTime(&w, r.a, r.b));
        CUDA_TRY(h, cudaEventElapsedTime(&k, r.b, r.c));
        out->launches++;
        out->wait_ms += w;
        out->kernel_ms += k;
        out->wait_max_ms = std::max(out->wait_max_ms, (double)w);
        out->kernel_max_ms = std::max(out->kernel_max_ms, (double)k);
    }
    for (auto& r : h->trecs) {
        cudaSetDevice(r.device);
        for (cudaEvent_t e : {r.a, r.b, r.c}) cudaEventDestroy(e);
    }
    h->trecs.clear();
    return SPREAD_OK;
}

spread_status somier_destroy(somier_t h) {
    if (!h) return SPREAD_OK;
    for (auto& d : h->devs)
        if (d.stream) {
            cudaSetDevice(d.device);
            cudaStreamSynchronize(d.stream);
        }
    for (auto& r : h->trecs) {
        cudaSetDevice(r.device);
        for (cudaEvent_t e : {r.a, r.b, r.c}) cudaEventDestroy(e);
    }
    if (h->graph_exec) cudaGraphExecDestroy(h->graph_exec);
    for (auto& ge : h->tb2_graph)
        if (ge) cudaGraphExecDestroy(ge);
    free_all(h);
    delete h;
    return SPREAD_OK;
}

const char* somier_version(void) { return "somier-spread 0.1 (sm_100a)"; }

}  // extern "C"
