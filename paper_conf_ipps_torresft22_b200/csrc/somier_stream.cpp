// somier_stream.cpp -- host-streamed ("out-of-core") Somier: the paper's own
// experiment (§V-A..C, 336-659) on B200. The state stays in host
// memory; each time step maps every chunk of the spread to its device
// (X[start-1 : size+2] and V[start : size]), runs the
// fused K1 on it, and maps X[start : size], V[start : size] back
// (PAPER.md:218-219). With `buffers` >= 2 device slots the H2D of chunk m+1,
// K1 of chunk m and the D2H of chunk m-1 overlap on three streams -- the
// paper's double buffering expressed with CUDA streams and
// events instead of OpenMP tasks and `depend`.
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstring>
#include <new>
#include <string>
#include <thread>
#include <utility>
#include <vector>

#include "driver_util.hpp"
#include "guard.hpp"
#include "kernels.hpp"
#include "somier.h"
#include "spread_impl.hpp"
#include "status.hpp"
#include "trace.hpp"

using paper::set_last_error;

namespace {

struct Slot {
    void* base = nullptr;
    double* x_in = nullptr;   // X_t of the chunk, size+2 planes (halo planes included)
    double* x_out = nullptr;  // X_{t+1}, planes 1..size written by K1
    double* v = nullptr;      // V of the chunk, size planes
    paper::GuardLayout guard; // SOMIER_GUARD zones (guard.hpp; none by default)
    alignas(64) CUtensorMap tmap_x;
    alignas(64) CUtensorMap tmap_v;
    alignas(64) CUtensorMap tmap_x2;
    alignas(64) CUtensorMap tmap_v2;
    cudaEvent_t comp_done = nullptr, d2h_done = nullptr;
    bool used = false;
};

// Per-chunk completion events, by step parity: the chunk-level `depend`
// (PAPER.md:746-767). H2D(c, t+1) depends on D2H(c-1, t), D2H(c, t),
// D2H(c+1, t) (it reads the halo planes and V they wrote); D2H(c, t+1), which
// overwrites X_t[c], depends on H2D(c-1, t) and H2D(c+1, t) (they read its
// edge planes as halos). No other ordering between steps is needed.
// Events are per list position (created on first use on that position's
// device, since an event is recorded on its own device's streams): under the
// dynamic schedule a chunk moves between devices from step to step; *_at
// remembers which position recorded the last one.
struct ChunkEvents {
    std::vector<cudaEvent_t> h2d[2], d2h[2];
    int h2d_at[2] = {-1, -1}, d2h_at[2] = {-1, -1};
    cudaEvent_t last_h2d(int par) const { return h2d_at[par] < 0 ? nullptr : h2d[par][(size_t)h2d_at[par]]; }
    cudaEvent_t last_d2h(int par) const { return d2h_at[par] < 0 ? nullptr : d2h[par][(size_t)d2h_at[par]]; }
};

// record a chunk event of list position pos (the current device) on stream st
cudaError_t record_at(std::vector<cudaEvent_t>& v, int& at, int pos, cudaStream_t st) {
    if (v.size() <= (size_t)pos) v.resize((size_t)pos + 1, nullptr);
    if (!v[(size_t)pos]) {
        cudaError_t e = cudaEventCreateWithFlags(&v[(size_t)pos], cudaEventDisableTiming);
        if (e != cudaSuccess) return e;
    }
    at = pos;
    return cudaEventRecord(v[(size_t)pos], st);
}

cudaError_t wait_ev(cudaStream_t st, cudaEvent_t ev) { return ev ? cudaStreamWaitEvent(st, ev, 0) : cudaSuccess; }

// spread_schedule(dynamic) is a test of the slot ring's next slot: free once
// its previous chunk's map(from) completed
template <class SlotT>
bool slot_free(const SlotT& sl) {
    if (!sl.used) return true;
    const cudaError_t e = cudaEventQuery(sl.d2h_done);
    if (e == cudaErrorNotReady) cudaGetLastError();  // not an error: clear it
    return e == cudaSuccess;
}

// Device buffers of a blocked round trip (somier_stream_run_blocked): the
// chunk's X_t planes [start-s-1, start+size+s+1) and V_t planes
// [start-s, start+size+s) for s steps per trip, plus a second X and V buffer
// the launches ping-pong through. Allocated on first use.
struct DeepSlot {
    void* base = nullptr;
    double *xa = nullptr, *xb = nullptr, *va = nullptr, *vb = nullptr;
    paper::GuardLayout guard;
    int64_t planes = 0;  // X planes per buffer (V: planes - 2)
    cudaEvent_t comp_done = nullptr, d2h_done = nullptr;
    bool used = false;
};

struct Dev {
    int pos = 0, device = 0;
    cudaStream_t s_h2d = nullptr, s_comp = nullptr, s_d2h = nullptr;
    std::vector<Slot> slots;
    std::vector<DeepSlot> deep;
    // StatsAccum[1 + acc_steps]: [0] the fixed nodes no launch visits (end
    // planes, K1_TB2's k-face columns), then one slot per step of the run
    void* acc_base = nullptr;
    int64_t acc_steps = 0;
    std::vector<int64_t> chunks;  // the static round-robin's chunks (generate; slot sizing)
    bool active = false;          // takes chunks (static: has some; dynamic: every position)
    size_t next_slot = 0;         // dynamic schedule: the slot ring's next slot
    int64_t chunks_run = 0;       // chunk tasks this position ran (somier_stream_chunk_counts)
    int64_t delay_ns = 0;         // test hook: extra device time per chunk (somier_stream_set_delay)
    paper::StatsAccum* acc(int64_t t) const { return (paper::StatsAccum*)acc_base + 1 + t; }
    paper::StatsAccum* acc_static() const { return (paper::StatsAccum*)acc_base; }
};

}  // namespace

struct somier_stream_s {
    somier_params p{};
    spread_s spread;
    paper::SlabGeom geom{};
    int buffers = 1;
    int64_t max_chunk = 0;
    int64_t step = 0;
    int64_t launches = 0;
    std::vector<Dev> devs;
    std::vector<ChunkEvents> ev;   // per chunk, created on the chunk's device
    std::string sticky;
};

namespace {

// The position and buffer slot chunk c runs on. Static schedule: its
// round-robin position, slot (c / p) mod buffers. Dynamic schedule
// (PAPER.md:771, 775): the first position -- polled from c's round-robin one --
// whose next slot is free, i.e. whichever device frees a slot first; the host
// thread waits (polling the slots' completion events) while none is free.
template <class SlotT>
std::pair<Dev*, SlotT*> place_chunk(somier_stream_s* h, int64_t c, std::vector<SlotT> Dev::*slots) {
    const paper::ChunkInfo ci = h->spread.chunk_info(c);
    const size_t np = h->devs.size();
    if (!h->spread.dynamic) {
        Dev& d = h->devs[(size_t)ci.pos];
        const size_t m = (size_t)(c / (int64_t)np);  // index of c among its device's chunks
        d.chunks_run++;
        return {&d, &(d.*slots)[m % (d.*slots).size()]};
    }
    for (;;) {
        for (size_t k = 0; k < np; k++) {
            Dev& d = h->devs[((size_t)ci.pos + k) % np];
            auto& v = d.*slots;
            if (v.empty()) continue;
            SlotT& sl = v[d.next_slot % v.size()];
            if (slot_free(sl)) {
                d.next_slot++;
                d.chunks_run++;
                return {&d, &sl};
            }
        }
        std::this_thread::yield();
    }
}

spread_status sfail(somier_stream_t h, cudaError_t e, const char* what) {
    std::string msg = std::string(what) + ": " + cudaGetErrorString(e);
    if (h && h->sticky.empty()) h->sticky = msg;
    set_last_error("%s", msg.c_str());
    return e == cudaErrorMemoryAllocation ? SPREAD_ENOMEM : SPREAD_ECUDA;
}

#define S_TRY(h, call)                                        \
    do {                                                      \
        cudaError_t e_ = (call);                              \
        if (e_ != cudaSuccess) return sfail((h), e_, #call);  \
    } while (0)

size_t round_up(size_t v, size_t a) { return (v + a - 1) / a * a; }

constexpr int64_t kAccSteps = 64;  // initial per-step stats history (grown on demand)

void destroy_all(somier_stream_t h) {
    for (auto& d : h->devs) {
        cudaSetDevice(d.device);
        for (cudaStream_t s : {d.s_h2d, d.s_comp, d.s_d2h})
            if (s) cudaStreamSynchronize(s);
        for (auto& sl : d.slots) {
            for (cudaEvent_t e : {sl.comp_done, sl.d2h_done})
                if (e) cudaEventDestroy(e);
            if (sl.base) cudaFree(sl.base);
        }
        for (auto& sl : d.deep) {
            for (cudaEvent_t e : {sl.comp_done, sl.d2h_done})
                if (e) cudaEventDestroy(e);
            if (sl.base) cudaFree(sl.base);
        }
        if (d.acc_base) cudaFree(d.acc_base);
        for (cudaStream_t s : {d.s_h2d, d.s_comp, d.s_d2h})
            if (s) cudaStreamDestroy(s);
    }
    for (auto& ce : h->ev)
        for (int q = 0; q < 2; q++) {
            for (auto* v : {&ce.h2d[q], &ce.d2h[q]})
                for (cudaEvent_t e : *v)
                    if (e) cudaEventDestroy(e);
        }
    h->ev.clear();
    h->devs.clear();
}

paper::SlabGeom geom_of(const somier_stream_s* h, const paper::ChunkInfo& c) {
    paper::SlabGeom g = h->geom;
    g.start = c.start;
    g.size = c.size;
    return g;
}

spread_status sync_devs(somier_stream_t h) {
    for (auto& d : h->devs) {
        cudaError_t e = cudaSetDevice(d.device);
        for (cudaStream_t s : {d.s_h2d, d.s_comp, d.s_d2h})
            if (e == cudaSuccess) e = cudaStreamSynchronize(s);
        if (e != cudaSuccess) return sfail(h, e, "somier_stream: synchronize");
    }
    if (!h->sticky.empty()) PAPER_FAIL(SPREAD_ECUDA, "%s", h->sticky.c_str());
    for (auto& d : h->devs) {  // SOMIER_GUARD zones (guard.hpp)
        auto check = [&](const paper::GuardLayout& L, const void* base, const char* kind, size_t i) -> spread_status {
            if (!L.G || !base) return SPREAD_OK;
            std::string msg;
            cudaError_t e = cudaSetDevice(d.device);
            const std::string what = std::string(kind) + " " + std::to_string(i) + " of list position " +
                                     std::to_string(d.pos);
            if (e == cudaSuccess && paper::guard_check(L, base, what.c_str(), msg, e)) return SPREAD_OK;
            if (e != cudaSuccess) return sfail(h, e, "somier_stream guard check");
            if (h->sticky.empty()) h->sticky = msg;
            PAPER_FAIL(SPREAD_ECUDA, "%s", msg.c_str());
        };
        for (size_t i = 0; i < d.slots.size(); i++) {
            spread_status st = check(d.slots[i].guard, d.slots[i].base, "slot", i);
            if (st != SPREAD_OK) return st;
        }
        for (size_t i = 0; i < d.deep.size(); i++) {
            spread_status st = check(d.deep[i].guard, d.deep[i].base, "deep slot", i);
            if (st != SPREAD_OK) return st;
        }
    }
    return SPREAD_OK;
}

// Grow every device's per-step stats history to hold `nsteps` steps.
spread_status ensure_acc(somier_stream_t h, int64_t nsteps) {
    for (auto& d : h->devs) {
        if (!d.active || d.acc_steps >= nsteps) continue;
        S_TRY(h, cudaSetDevice(d.device));
        S_TRY(h, cudaDeviceSynchronize());
        S_TRY(h, cudaFree(d.acc_base));
        d.acc_base = nullptr;
        d.acc_steps = 0;
        S_TRY(h, cudaMalloc(&d.acc_base, (1 + (size_t)nsteps) * sizeof(paper::StatsAccum)));
        d.acc_steps = nsteps;
    }
    return SPREAD_OK;
}

// Enqueue step t of a run (0-based within the run): every chunk, in chunk
// order, reads X_t from X, writes X_{t+1} to XN and V in place. `chained`:
// a step of the same run precedes it, so its copies wait on that step's
// per-chunk events instead of a host barrier.
spread_status enqueue_stream_step(somier_stream_t h, double* const X[3], double* const V[3], double* const XN[3],
                                  int64_t t, bool chained) {
    const int64_t n0 = h->p.n[0];
    const int64_t nch = h->spread.nchunks;
    const int par = (int)(t & 1), prev = par ^ 1;
    for (int64_t c = 0; c < nch; c++) {
        const paper::ChunkInfo ci = h->spread.chunk_info(c);
        const auto pl = place_chunk(h, c, &Dev::slots);
        Dev& d = *pl.first;
        Slot& sl = *pl.second;
        const paper::SlabGeom g = geom_of(h, ci);
        const bool first = ci.start == 1, last = ci.start + ci.size == n0 - 1;
        ChunkEvents& ev = h->ev[(size_t)c];
        S_TRY(h, cudaSetDevice(d.device));
        // map(to: X[start-1 : size+2], V[start : size])  -- depend(in: ...)
        if (sl.used) S_TRY(h, cudaStreamWaitEvent(d.s_h2d, sl.d2h_done, 0));
        if (chained)
            for (int64_t nb = std::max<int64_t>(0, c - 1); nb <= std::min<int64_t>(nch - 1, c + 1); nb++)
                S_TRY(h, wait_ev(d.s_h2d, h->ev[(size_t)nb].last_d2h(prev)));
        for (int q = 0; q < 3; q++) {
            S_TRY(h, paper::copy_slab_planes(g, sl.x_in, q, 0, X[q], ci.start - 1, ci.size + 2,
                                             cudaMemcpyHostToDevice, d.s_h2d));
            S_TRY(h, paper::copy_slab_planes(g, sl.v, q, 0, V[q], ci.start, ci.size, cudaMemcpyHostToDevice,
                                             d.s_h2d));
        }
        S_TRY(h, record_at(ev.h2d[par], ev.h2d_at[par], d.pos, d.s_h2d));
        // the fused step (forces, accelerations, velocities, positions, centers)
        S_TRY(h, wait_ev(d.s_comp, ev.last_h2d(par)));
        paper::StatsAccum* acc = d.acc(t);
        if (t == 0) {  // the fixed end planes, once per run (they never move)
            if (first) S_TRY(h, paper::launch_stats(sl.x_in, nullptr, g, 0, 1, d.acc_static(), d.s_comp));
            if (last) S_TRY(h, paper::launch_stats(sl.x_in, nullptr, g, ci.size + 1, 1, d.acc_static(), d.s_comp));
            // max |x| of the input state (the exact-stats domain bound, stats_layout.hpp)
            S_TRY(h, paper::launch_xmax(sl.x_in, g, 1, ci.size, d.acc_static(), d.s_comp));
        }
        paper::StepArgs a;
        std::memset(&a, 0, sizeof a);
        a.fma = h->p.math == SOMIER_MATH_FMA ? 1 : 0;
        a.x_cur = sl.x_in;
        a.x_nxt = sl.x_out;
        a.v = sl.v;
        a.g = g;
        a.K = h->p.k_spring;
        a.L = h->p.rest_len;
        a.M = h->p.mass;
        a.dt = h->p.dt;
        a.acc = acc;
        a.tmap_x_cur = &sl.tmap_x;
        a.tmap_v = &sl.tmap_v;
        a.tmap_x2_cur = &sl.tmap_x2;
        a.tmap_v2 = &sl.tmap_v2;
        a.write_fixed = 1;
        const paper::K1Variant var = paper::k1_variant(h->p.kernel);
        S_TRY(h, paper::launch_delay(d.delay_ns, d.s_comp));
        S_TRY(h, paper::launch_k1(var, a, h->p.mass == 1.0, d.s_comp));
        h->launches++;
        S_TRY(h, cudaEventRecord(sl.comp_done, d.s_comp));
        // map(from: X[start : size], V[start : size]) (+ the fixed end planes);
        // it overwrites X_{t-1}[chunk], whose edge planes the neighbours' H2D of
        // the previous step read as halos
        S_TRY(h, cudaStreamWaitEvent(d.s_d2h, sl.comp_done, 0));
        if (chained) {
            if (c > 0) S_TRY(h, wait_ev(d.s_d2h, h->ev[(size_t)c - 1].last_h2d(prev)));
            if (c + 1 < nch) S_TRY(h, wait_ev(d.s_d2h, h->ev[(size_t)c + 1].last_h2d(prev)));
        }
        for (int q = 0; q < 3; q++) {
            S_TRY(h, paper::copy_slab_planes(g, sl.x_out, q, 1, XN[q], ci.start, ci.size, cudaMemcpyDeviceToHost,
                                             d.s_d2h));
            S_TRY(h, paper::copy_slab_planes(g, sl.v, q, 0, V[q], ci.start, ci.size, cudaMemcpyDeviceToHost,
                                             d.s_d2h));
            if (first)
                S_TRY(h, paper::copy_slab_planes(g, sl.x_in, q, 0, XN[q], 0, 1, cudaMemcpyDeviceToHost, d.s_d2h));
            if (last)
                S_TRY(h, paper::copy_slab_planes(g, sl.x_in, q, ci.size + 1, XN[q], n0 - 1, 1,
                                                 cudaMemcpyDeviceToHost, d.s_d2h));
        }
        S_TRY(h, record_at(ev.d2h[par], ev.d2h_at[par], d.pos, d.s_d2h));
        S_TRY(h, cudaEventRecord(sl.d2h_done, d.s_d2h));
        sl.used = true;
    }
    return SPREAD_OK;
}

// Combine the per-step stats slots of every device (plus its static slot)
// into stats[0 .. n).
spread_status gather_stats(somier_stream_t h, int64_t n, const int64_t* steps, somier_stats_t* stats) {
    std::vector<__int128> sums((size_t)n * 3, 0);
    std::vector<unsigned long long> vmax2((size_t)n, 0);
    unsigned long long xmax0 = 0;  // max |x| bits of the run's input state and the fixed nodes
    std::vector<paper::StatsAccum> acc((size_t)n + 1);
    for (auto& d : h->devs) {
        if (!d.active) continue;
        S_TRY(h, cudaSetDevice(d.device));
        S_TRY(h, cudaMemcpy(acc.data(), d.acc_base, acc.size() * sizeof(paper::StatsAccum), cudaMemcpyDeviceToHost));
        for (int64_t t = 0; t < n; t++)
            for (size_t q : {(size_t)0, (size_t)(t + 1)}) {
                const paper::StatsAccum& a = acc[q];
                for (int k = 0; k < 3; k++)
                    sums[(size_t)(3 * t + k)] += (__int128)(((unsigned __int128)a.hi[k] << 64) | a.lo[k]);
                vmax2[(size_t)t] = std::max(vmax2[(size_t)t], (unsigned long long)a.vmax2);
            }
        xmax0 = std::max(xmax0, (unsigned long long)acc[0].xmax);
    }
    // exact-stats domain: the bound of each state from the input state's max |x|
    // and every step's vmax (stats_layout.hpp)
    double B;
    std::memcpy(&B, &xmax0, sizeof B);
    for (int64_t t = 0; t < n; t++) {
        double v2;
        std::memcpy(&v2, &vmax2[(size_t)t], sizeof v2);
        B = paper::xbound_step(B, v2, h->p.dt);
        paper::finish_somier_stats(&h->p, &sums[(size_t)(3 * t)], vmax2[(size_t)t],
                                   h->p.n[0] * h->p.n[1] * h->p.n[2], steps[t], &stats[t], paper::xbound_ok(B));
    }
    return SPREAD_OK;
}

// The one-step slots and the deep slots of blocked trips never coexist: the
// mode in use holds the device memory (a switch synchronises and reallocates),
// so a blocked run can use the memory the one-step slots would pin.
void release_deep(Dev& d) {
    for (auto& sl : d.deep) {
        if (sl.base) cudaFree(sl.base);
        sl.base = nullptr;
        sl.planes = 0;
        sl.used = false;
    }
}

spread_status ensure_flat(somier_stream_t h) {
    const size_t plane = (size_t)h->geom.plane_stride() * sizeof(double);
    const size_t xb = round_up(plane * (size_t)(h->max_chunk + 2), 4096);
    const size_t vb = round_up(plane * (size_t)h->max_chunk, 4096);
    for (auto& d : h->devs) {
        bool missing = false;
        for (auto& sl : d.slots) missing = missing || !sl.base;
        if (!d.active || !missing) continue;
        S_TRY(h, cudaSetDevice(d.device));
        S_TRY(h, cudaDeviceSynchronize());
        release_deep(d);
        for (auto& sl : d.slots) {
            if (sl.base) continue;
            sl.guard.plan(paper::guard_bytes(plane), {{xb, "X in"}, {xb, "X out"}, {vb, "V"}});
            S_TRY(h, cudaMalloc(&sl.base, sl.guard.bytes));
            sl.x_in = (double*)((char*)sl.base + sl.guard.off[0]);
            sl.x_out = (double*)((char*)sl.base + sl.guard.off[1]);
            sl.v = (double*)((char*)sl.base + sl.guard.off[2]);
            if (sl.guard.G) {  // cudaMemset* on the legacy stream: finished before the handle's streams start
                S_TRY(h, paper::guard_fill(sl.guard, sl.base, 0));
                S_TRY(h, cudaDeviceSynchronize());
            }
            sl.used = false;
            const paper::SlabGeom g = h->geom;
            spread_status st = paper::encode_slab_tmap(&sl.tmap_x, g, sl.x_in, h->max_chunk + 2, paper::kXBoxK,
                                                       paper::kXBoxJ);
            if (st == SPREAD_OK)
                st = paper::encode_slab_tmap(&sl.tmap_v, g, sl.v, h->max_chunk, paper::kVBoxK, paper::kVBoxJ);
            if (st == SPREAD_OK)
                st = paper::encode_slab_tmap(&sl.tmap_x2, g, sl.x_in, h->max_chunk + 2, paper::kXBoxK,
                                             paper::kX2BoxJ);
            if (st == SPREAD_OK)
                st = paper::encode_slab_tmap(&sl.tmap_v2, g, sl.v, h->max_chunk, paper::kVBoxK, paper::kV2BoxJ);
            if (st != SPREAD_OK) return st;
        }
    }
    return SPREAD_OK;
}

// (Re)allocate every device's deep slots for `planes` X planes per buffer.
spread_status ensure_deep(somier_stream_t h, int64_t planes) {
    const size_t plane = (size_t)h->geom.plane_stride() * sizeof(double);
    for (auto& d : h->devs) {
        if (!d.active) continue;
        S_TRY(h, cudaSetDevice(d.device));
        if (!d.deep.empty() && d.deep[0].base && d.deep[0].planes >= planes) continue;
        S_TRY(h, cudaDeviceSynchronize());
        for (auto& sl : d.slots) {  // the one-step slots give their memory up (ensure_flat restores them)
            if (sl.base) cudaFree(sl.base);
            sl.base = nullptr;
            sl.x_in = sl.x_out = sl.v = nullptr;
        }
        for (auto& sl : d.deep)
            if (sl.base) S_TRY(h, cudaFree(sl.base));
        d.deep.resize(d.slots.size());
        const size_t xb = round_up(plane * (size_t)planes, 4096), vb = round_up(plane * (size_t)(planes - 2), 4096);
        for (auto& sl : d.deep) {
            sl.base = nullptr;
            sl.guard.plan(paper::guard_bytes(plane), {{xb, "X a"}, {xb, "X b"}, {vb, "V a"}, {vb, "V b"}});
            S_TRY(h, cudaMalloc(&sl.base, sl.guard.bytes));
            // zeroed once: the fixed face nodes of V are never written by K1_TB2
            S_TRY(h, cudaMemset(sl.base, 0, sl.guard.bytes));
            S_TRY(h, paper::guard_fill(sl.guard, sl.base, 0));
            sl.xa = (double*)((char*)sl.base + sl.guard.off[0]);
            sl.xb = (double*)((char*)sl.base + sl.guard.off[1]);
            sl.va = (double*)((char*)sl.base + sl.guard.off[2]);
            sl.vb = (double*)((char*)sl.base + sl.guard.off[3]);
            sl.planes = planes;
            sl.used = false;
            for (cudaEvent_t* pe : {&sl.comp_done, &sl.d2h_done})
                if (!*pe) S_TRY(h, cudaEventCreateWithFlags(pe, cudaEventDisableTiming));
        }
        // cudaMemset runs on the legacy stream, which the handle's non-blocking
        // streams do not wait for: finish the zeroing before any copy lands
        S_TRY(h, cudaDeviceSynchronize());
    }
    return SPREAD_OK;
}

// Chunks within `depth` planes of chunk c (either way).
void reach_range(const somier_stream_s* h, const paper::ChunkInfo& ci, int64_t depth, int64_t* c_lo, int64_t* c_hi) {
    const int64_t n0 = h->p.n[0];
    *c_lo = h->spread.chunk_of(std::max<int64_t>(1, ci.start - depth));
    *c_hi = h->spread.chunk_of(std::min<int64_t>(n0 - 2, ci.start + ci.size + depth - 1));
}

// Trip k of a blocked run: every chunk maps in X_t planes [start-s, start+size+s)
// and V_t planes [start-s+1, start+size+s-1) (at least one halo plane; clipped
// to the grid), advances s
// steps with ceil(s/2) K1_TB2 launches over regions that shrink by two planes
// per side per launch (the last one is the chunk itself; an odd s ends with a
// one-step launch), and maps X_{t+s}, V_{t+s} of its planes out into (XN, VN).
//   t0: the run's step index of the trip's first step (stats of step t0 + j go
//       to d.acc(t0 + j)); s_prev: the previous trip's depth (its H2D read
//       s_prev planes around each chunk, which this trip's D2H overwrites)
spread_status enqueue_stream_blocked(somier_stream_t h, double* const X[3], double* const V[3], double* const XN[3],
                                     double* const VN[3], int64_t k, int64_t s, int64_t t0, int64_t s_prev,
                                     bool chained) {
    const int64_t n0 = h->p.n[0];
    const int64_t nch = h->spread.nchunks;
    const int64_t ps = h->geom.plane_stride();
    const int par = (int)(k & 1), prev = par ^ 1;
    const int64_t nl = s / 2 + (s & 1);
    for (int64_t c = 0; c < nch; c++) {
        const paper::ChunkInfo ci = h->spread.chunk_info(c);
        const auto pl = place_chunk(h, c, &Dev::deep);
        Dev& d = *pl.first;
        DeepSlot& sl = *pl.second;
        const bool first = ci.start == 1, last = ci.start + ci.size == n0 - 1;
        ChunkEvents& ev = h->ev[(size_t)c];
        int64_t c_lo, c_hi, w_lo, w_hi;
        reach_range(h, ci, s, &c_lo, &c_hi);           // H2D waits: the D2H of the chunks this trip reads
        reach_range(h, ci, std::max(s, s_prev), &w_lo, &w_hi);  // D2H waits: the H2D that read what it overwrites
        // global plane of raw plane 0 of the X / V buffers: one plane of slack
        // beyond the s-plane halo on each side (a one-step launch still reads
        // the deep layout's outer ring plane, whose values it does not use)
        const int64_t x0 = ci.start - s - 1, v0 = ci.start - s;
        S_TRY(h, cudaSetDevice(d.device));
        if (sl.used) S_TRY(h, cudaStreamWaitEvent(d.s_h2d, sl.d2h_done, 0));
        if (chained)
            for (int64_t nb = c_lo; nb <= c_hi; nb++)
                S_TRY(h, wait_ev(d.s_h2d, h->ev[(size_t)nb].last_d2h(prev)));
        const int64_t xlo = std::max<int64_t>(0, ci.start - s), xhi = std::min<int64_t>(n0, ci.start + ci.size + s);
        // V_t is needed one plane less deep than X_t, but at least one plane
        // (a one-step launch reads the ring plane; the first chunk maps the face plane)
        const int64_t vd = std::max<int64_t>(1, s - 1);
        const int64_t vlo = std::max<int64_t>(0, ci.start - vd), vhi = std::min<int64_t>(n0, ci.start + ci.size + vd);
        paper::SlabGeom g = geom_of(h, ci);
        for (int q = 0; q < 3; q++) {
            S_TRY(h, paper::copy_slab_planes(g, sl.xa, q, xlo - x0, X[q], xlo, xhi - xlo, cudaMemcpyHostToDevice,
                                             d.s_h2d));
            S_TRY(h, paper::copy_slab_planes(g, sl.va, q, vlo - v0, V[q], vlo, vhi - vlo,
                                             cudaMemcpyHostToDevice, d.s_h2d));
        }
        S_TRY(h, record_at(ev.h2d[par], ev.h2d_at[par], d.pos, d.s_h2d));
        S_TRY(h, wait_ev(d.s_comp, ev.last_h2d(par)));
        // the fixed face nodes of every output plane (K1_TB2 writes the moving nodes only)
        S_TRY(h, cudaMemcpyAsync(sl.xb + (xlo - x0) * ps, sl.xa + (xlo - x0) * ps,
                                 (size_t)((xhi - xlo) * ps) * sizeof(double), cudaMemcpyDeviceToDevice, d.s_comp));
        if (k == 0) {  // the fixed nodes no launch visits, once per run
            double* xv_one = sl.xa + (ci.start - 1 - x0) * ps;  // one-step view: raw plane 0 = start - 1
            if (first) S_TRY(h, paper::launch_stats(xv_one, nullptr, g, 0, 1, d.acc_static(), d.s_comp));
            if (last) S_TRY(h, paper::launch_stats(xv_one, nullptr, g, ci.size + 1, 1, d.acc_static(), d.s_comp));
            S_TRY(h, paper::launch_kface_stats(xv_one, g, 1, ci.size, d.acc_static(), d.s_comp));
            // max |x| of the input state (the exact-stats domain bound, stats_layout.hpp)
            S_TRY(h, paper::launch_xmax(xv_one, g, 1, ci.size, d.acc_static(), d.s_comp));
        }
        S_TRY(h, paper::launch_delay(d.delay_ns, d.s_comp));
        int64_t remaining = s, done = 0;
        double *xin = sl.xa, *xout = sl.xb, *vin = sl.va, *vout = sl.vb;
        for (int64_t j = 0; j < nl; j++) {
            const bool two = remaining >= 2;
            const int64_t w = remaining - (two ? 2 : 1);  // planes this launch's region extends beyond the chunk
            paper::SlabGeom gj = g;
            gj.start = std::max<int64_t>(1, ci.start - w);
            gj.size = std::min<int64_t>(n0 - 1, ci.start + ci.size + w) - gj.start;
            double* xs = xin + (gj.start - 2 - x0) * ps;       // raw plane 0 = region start - 2
            double* vs = vin + (gj.start - 1 - v0) * ps;        // raw plane 0 = region start - 1
            alignas(64) CUtensorMap mx, mv;
            spread_status st = paper::encode_slab_tmap(&mx, gj, xs, gj.size + 4, paper::kTB2XBoxK, paper::kTB2XBoxJ);
            if (st != SPREAD_OK) return st;
            st = paper::encode_slab_tmap(&mv, gj, vs, gj.size + 2, paper::kTB2VBoxK, paper::kTB2VBoxJ);
            if (st != SPREAD_OK) return st;
            paper::StepArgs a;
            std::memset(&a, 0, sizeof a);
            a.fma = h->p.math == SOMIER_MATH_FMA ? 1 : 0;
            a.x_cur = xs;
            a.v = vs;
            a.g = gj;
            a.K = h->p.k_spring;
            a.L = h->p.rest_len;
            a.M = h->p.mass;
            a.dt = h->p.dt;
            // every launch counts the chunk's own planes only: stats of every step
            a.acc_mid = d.acc(t0 + done);
            a.acc = d.acc(t0 + done + (two ? 1 : 0));
            a.tmap_x_cur = &mx;
            a.tmap_v = &mv;
            paper::Tb2Out o;
            std::memset(&o, 0, sizeof o);
            o.x_out = xout + (gj.start - 2 - x0) * ps;
            o.v_out = vout + (gj.start - 1 - v0) * ps;
            o.two = two;
            o.stats_lo = ci.start;
            o.stats_hi = ci.start + ci.size;
            S_TRY(h, paper::launch_k1_tb2(a, o, h->p.mass == 1.0, d.s_comp));
            h->launches++;
            remaining -= two ? 2 : 1;
            done += two ? 2 : 1;
            std::swap(xin, xout);
            std::swap(vin, vout);
        }
        S_TRY(h, cudaEventRecord(sl.comp_done, d.s_comp));
        S_TRY(h, cudaStreamWaitEvent(d.s_d2h, sl.comp_done, 0));
        if (chained)
            for (int64_t nb = w_lo; nb <= w_hi; nb++)
                if (nb != c) S_TRY(h, wait_ev(d.s_d2h, h->ev[(size_t)nb].last_h2d(prev)));
        // after the last launch the state is in (xin, vin)
        for (int q = 0; q < 3; q++) {
            S_TRY(h, paper::copy_slab_planes(g, xin, q, ci.start - x0, XN[q], ci.start, ci.size,
                                             cudaMemcpyDeviceToHost, d.s_d2h));
            S_TRY(h, paper::copy_slab_planes(g, vin, q, ci.start - v0, VN[q], ci.start, ci.size,
                                             cudaMemcpyDeviceToHost, d.s_d2h));
            if (first) {
                S_TRY(h, paper::copy_slab_planes(g, sl.xa, q, 0 - x0, XN[q], 0, 1, cudaMemcpyDeviceToHost, d.s_d2h));
                S_TRY(h, paper::copy_slab_planes(g, sl.va, q, 0 - v0, VN[q], 0, 1, cudaMemcpyDeviceToHost,
                                                 d.s_d2h));
            }
            if (last) {
                S_TRY(h, paper::copy_slab_planes(g, sl.xa, q, n0 - 1 - x0, XN[q], n0 - 1, 1, cudaMemcpyDeviceToHost,
                                                 d.s_d2h));
                S_TRY(h, paper::copy_slab_planes(g, sl.va, q, n0 - 1 - v0, VN[q], n0 - 1, 1,
                                                 cudaMemcpyDeviceToHost, d.s_d2h));
            }
        }
        S_TRY(h, record_at(ev.d2h[par], ev.d2h_at[par], d.pos, d.s_d2h));
        S_TRY(h, cudaEventRecord(sl.d2h_done, d.s_d2h));
        sl.used = true;
    }
    return SPREAD_OK;
}

// Blocked run: trips of s steps (the last one shorter if s does not divide
// nsteps), alternating (X, V) -> (XN, VN) -> (X, V) ...; stats[t] (if non-NULL)
// receives the statistics after step t. One host barrier at the end.
spread_status stream_run_blocked(somier_stream_t h, double* const X[3], double* const V[3], double* const XN[3],
                                 double* const VN[3], int64_t nsteps, int64_t s, somier_stats_t* stats) {
    PAPER_NVTX("somier_stream_run_blocked");
    if (!h->sticky.empty()) PAPER_FAIL(SPREAD_ECUDA, "%s", h->sticky.c_str());
    const int64_t ntrips = (nsteps + s - 1) / s;
    spread_status st = ensure_acc(h, nsteps);
    if (st != SPREAD_OK) return st;
    st = ensure_deep(h, h->max_chunk + 2 * s + 2);
    if (st != SPREAD_OK) return st;
    for (auto& d : h->devs) {
        if (!d.active) continue;
        S_TRY(h, cudaSetDevice(d.device));
        S_TRY(h, cudaMemsetAsync(d.acc_base, 0, (1 + (size_t)nsteps) * sizeof(paper::StatsAccum), d.s_comp));
    }
    for (int64_t k = 0; k < ntrips; k++) {
        const int64_t sk = std::min<int64_t>(s, nsteps - k * s);
        st = (k & 1) ? enqueue_stream_blocked(h, XN, VN, X, V, k, sk, k * s, s, k > 0)
                     : enqueue_stream_blocked(h, X, V, XN, VN, k, sk, k * s, s, k > 0);
        if (st != SPREAD_OK) return st;
    }
    st = sync_devs(h);
    if (st != SPREAD_OK) return st;
    std::vector<int64_t> steps((size_t)nsteps);
    for (int64_t t = 0; t < nsteps; t++) steps[(size_t)t] = h->step + t + 1;
    h->step += nsteps;
    return stats ? gather_stats(h, nsteps, steps.data(), stats) : SPREAD_OK;
}

// Run nsteps steps from (X, V), alternating X -> XN -> X ...; stats[t] (if
// non-NULL) receives the statistics after step t. One host barrier at the end.
spread_status stream_run(somier_stream_t h, double* const X[3], double* const V[3], double* const XN[3],
                         int64_t nsteps, somier_stats_t* stats) {
    PAPER_NVTX("somier_stream_run");
    if (!h->sticky.empty()) PAPER_FAIL(SPREAD_ECUDA, "%s", h->sticky.c_str());
    spread_status st = ensure_flat(h);
    if (st != SPREAD_OK) return st;
    st = ensure_acc(h, nsteps);
    if (st != SPREAD_OK) return st;
    for (auto& d : h->devs) {
        if (!d.active) continue;
        S_TRY(h, cudaSetDevice(d.device));
        S_TRY(h, cudaMemsetAsync(d.acc_base, 0, (1 + (size_t)nsteps) * sizeof(paper::StatsAccum), d.s_comp));
    }
    for (int64_t t = 0; t < nsteps; t++) {
        st = (t & 1) ? enqueue_stream_step(h, XN, V, X, t, t > 0) : enqueue_stream_step(h, X, V, XN, t, t > 0);
        if (st != SPREAD_OK) return st;
    }
    st = sync_devs(h);
    if (st != SPREAD_OK) return st;
    std::vector<int64_t> steps((size_t)nsteps);
    for (int64_t t = 0; t < nsteps; t++) steps[(size_t)t] = h->step + t + 1;
    h->step += nsteps;
    return stats ? gather_stats(h, nsteps, steps.data(), stats) : SPREAD_OK;
}

}  // namespace

extern "C" {

spread_status somier_stream_create(spread_t s, const somier_params* p, int buffers, somier_stream_t* out) {
    return somier_stream_create_on(s, p, buffers, nullptr, out);
}

spread_status somier_stream_create_on(spread_t s, const somier_params* p, int buffers, const int* cuda_devices,
                                      somier_stream_t* out) {
    if (!out) PAPER_FAIL(SPREAD_EINVAL, "somier_stream_create: out is NULL");
    *out = nullptr;
    if (!s) PAPER_FAIL(SPREAD_EINVAL, "somier_stream_create: spread is NULL");
    spread_status st = paper::check_somier_params(p);
    if (st != SPREAD_OK) return st;
    if (buffers < 1 || buffers > 16) PAPER_FAIL(SPREAD_EINVAL, "somier_stream_create: buffers %d outside [1, 16]", buffers);
    if (s->range_start != 1 || s->range_len != p->n[0] - 2)
        PAPER_FAIL(SPREAD_EINVAL, "somier_stream_create: spread range must be range(1:%lld)", (long long)(p->n[0] - 2));
    int ndev = 0;
    cudaError_t e = cudaGetDeviceCount(&ndev);
    if (e != cudaSuccess) PAPER_FAIL(SPREAD_ENODEV, "somier_stream_create: no CUDA device (%s)", cudaGetErrorString(e));
    for (size_t q = 0; q < s->devices.size(); q++) {
        const int id = cuda_devices ? cuda_devices[q] : s->devices[q];
        if (id < 0 || id >= ndev)
            PAPER_FAIL(SPREAD_ENODEV, "somier_stream_create: device %d not present (%d visible)", id, ndev);
    }

    somier_stream_s* h = new (std::nothrow) somier_stream_s;
    if (!h) PAPER_FAIL(SPREAD_ENOMEM, "somier_stream_create: out of host memory");
    h->p = *p;
    h->spread = *s;
    h->buffers = buffers;
    h->geom = paper::SlabGeom{p->n[0], p->n[1], p->n[2], paper::slab_ld(p->n[2]), 0, 0};
    h->max_chunk = s->max_chunk();
    h->devs.resize(s->devices.size());
    for (size_t q = 0; q < s->devices.size(); q++) {
        h->devs[q].pos = (int)q;
        h->devs[q].device = cuda_devices ? cuda_devices[q] : s->devices[q];
    }
    for (int64_t c = 0; c < s->nchunks; c++) h->devs[s->chunk_info(c).pos].chunks.push_back(c);
    for (auto& d : h->devs) d.active = !d.chunks.empty() || (s->dynamic && s->nchunks > 0);

    auto fail = [&](spread_status code) {
        std::string msg = paper::last_error();
        destroy_all(h);
        delete h;
        set_last_error("%s", msg.c_str());
        return code;
    };
    for (auto& d : h->devs) {
        if (!d.active) continue;
        if ((e = cudaSetDevice(d.device)) != cudaSuccess) return fail(sfail(h, e, "cudaSetDevice"));
        for (cudaStream_t* ps : {&d.s_h2d, &d.s_comp, &d.s_d2h})
            if ((e = cudaStreamCreateWithFlags(ps, cudaStreamNonBlocking)) != cudaSuccess)
                return fail(sfail(h, e, "cudaStreamCreate"));
        if ((e = cudaMalloc(&d.acc_base, (1 + kAccSteps) * sizeof(paper::StatsAccum))) != cudaSuccess)
            return fail(sfail(h, e, "cudaMalloc(stats)"));
        d.acc_steps = kAccSteps;
        d.slots.resize((size_t)std::min<int64_t>(buffers, s->dynamic ? s->nchunks : (int64_t)d.chunks.size()));
        for (auto& sl : d.slots)
            for (cudaEvent_t* pe : {&sl.comp_done, &sl.d2h_done})
                if ((e = cudaEventCreateWithFlags(pe, cudaEventDisableTiming)) != cudaSuccess)
                    return fail(sfail(h, e, "cudaEventCreate"));
    }
    st = ensure_flat(h);
    if (st != SPREAD_OK) return fail(st);
    h->ev.resize((size_t)s->nchunks);  // events created on first use (record_at)
    *out = h;
    return SPREAD_OK;
}

spread_status somier_stream_generate(somier_stream_t h, double* x, double* y, double* z, double* vx, double* vy,
                                     double* vz) {
    PAPER_NVTX("somier_stream_generate");
    if (!h || !x || !y || !z || !vx || !vy || !vz) PAPER_FAIL(SPREAD_EINVAL, "somier_stream_generate: NULL argument");
    if (!h->sticky.empty()) PAPER_FAIL(SPREAD_ECUDA, "%s", h->sticky.c_str());
    {
        const spread_status st = ensure_flat(h);
        if (st != SPREAD_OK) return st;
    }
    double* X[3] = {x, y, z};
    const int64_t n0 = h->p.n[0];
    const size_t grid = (size_t)(h->p.n[0] * h->p.n[1] * h->p.n[2]);
    std::memset(vx, 0, grid * sizeof(double));
    std::memset(vy, 0, grid * sizeof(double));
    std::memset(vz, 0, grid * sizeof(double));
    size_t maxm = 0;
    for (auto& d : h->devs) maxm = std::max(maxm, d.chunks.size());
    for (size_t m = 0; m < maxm; m++) {
        for (auto& d : h->devs) {
            if (m >= d.chunks.size()) continue;
            Slot& sl = d.slots[m % d.slots.size()];
            const paper::ChunkInfo c = h->spread.chunk_info(d.chunks[m]);
            const paper::SlabGeom g = geom_of(h, c);
            S_TRY(h, cudaSetDevice(d.device));
            if (sl.used) S_TRY(h, cudaStreamWaitEvent(d.s_comp, sl.d2h_done, 0));
            paper::InitArgs ia;
            ia.x0 = sl.x_in;
            ia.x1 = sl.x_out;  // scratch second buffer
            ia.g = g;
            ia.spacing = h->p.spacing;
            ia.amplitude = h->p.amplitude;
            ia.seed = h->p.seed;
            S_TRY(h, paper::launch_init(ia, d.s_comp));
            S_TRY(h, cudaEventRecord(sl.comp_done, d.s_comp));
            S_TRY(h, cudaStreamWaitEvent(d.s_d2h, sl.comp_done, 0));
            for (int q = 0; q < 3; q++) {
                S_TRY(h, paper::copy_slab_planes(g, sl.x_in, q, 1, X[q], c.start, c.size, cudaMemcpyDeviceToHost,
                                                 d.s_d2h));
                if (c.start == 1)
                    S_TRY(h, paper::copy_slab_planes(g, sl.x_in, q, 0, X[q], 0, 1, cudaMemcpyDeviceToHost, d.s_d2h));
                if (c.start + c.size == n0 - 1)
                    S_TRY(h, paper::copy_slab_planes(g, sl.x_in, q, c.size + 1, X[q], n0 - 1, 1,
                                                     cudaMemcpyDeviceToHost, d.s_d2h));
            }
            S_TRY(h, cudaEventRecord(sl.d2h_done, d.s_d2h));
            sl.used = true;
        }
    }
    return sync_devs(h);
}

spread_status somier_stream_step(somier_stream_t h, const double* x, const double* y, const double* z, double* vx,
                                 double* vy, double* vz, double* xn, double* yn, double* zn, somier_stats_t* stats) {
    if (!h || !x || !y || !z || !vx || !vy || !vz || !xn || !yn || !zn)
        PAPER_FAIL(SPREAD_EINVAL, "somier_stream_step: NULL argument");
    if (x == xn || y == yn || z == zn) PAPER_FAIL(SPREAD_EINVAL, "somier_stream_step: X_t and X_{t+1} alias (Jacobi)");
    double* X[3] = {const_cast<double*>(x), const_cast<double*>(y), const_cast<double*>(z)};
    double* XN[3] = {xn, yn, zn};
    double* V[3] = {vx, vy, vz};
    return stream_run(h, X, V, XN, 1, stats);
}

spread_status somier_stream_run(somier_stream_t h, double* x, double* y, double* z, double* vx, double* vy,
                                double* vz, double* xn, double* yn, double* zn, int64_t nsteps,
                                somier_stats_t* stats) {
    if (!h || !x || !y || !z || !vx || !vy || !vz || !xn || !yn || !zn)
        PAPER_FAIL(SPREAD_EINVAL, "somier_stream_run: NULL argument");
    if (nsteps < 0) PAPER_FAIL(SPREAD_EINVAL, "somier_stream_run: nsteps %lld < 0", (long long)nsteps);
    if (x == xn || y == yn || z == zn) PAPER_FAIL(SPREAD_EINVAL, "somier_stream_run: the two X buffers alias");
    if (nsteps == 0) return SPREAD_OK;
    double* X[3] = {x, y, z};
    double* XN[3] = {xn, yn, zn};
    double* V[3] = {vx, vy, vz};
    return stream_run(h, X, V, XN, nsteps, stats);
}

spread_status somier_stream_run2(somier_stream_t h, double* x, double* y, double* z, double* vx, double* vy,
                                 double* vz, double* xn, double* yn, double* zn, double* vxn, double* vyn,
                                 double* vzn, int64_t nsteps, somier_stats_t* stats) {
    if (!h || !x || !y || !z || !vx || !vy || !vz || !xn || !yn || !zn || !vxn || !vyn || !vzn)
        PAPER_FAIL(SPREAD_EINVAL, "somier_stream_run2: NULL argument");
    if (nsteps < 0) PAPER_FAIL(SPREAD_EINVAL, "somier_stream_run2: nsteps %lld < 0", (long long)nsteps);
    if (x == xn || y == yn || z == zn || vx == vxn || vy == vyn || vz == vzn)
        PAPER_FAIL(SPREAD_EINVAL, "somier_stream_run2: the two X or the two V buffers alias");
    if (nsteps == 0) return SPREAD_OK;
    double* X[3] = {x, y, z};
    double* XN[3] = {xn, yn, zn};
    double* V[3] = {vx, vy, vz};
    double* VN[3] = {vxn, vyn, vzn};
    return stream_run_blocked(h, X, V, XN, VN, nsteps, 2, stats);  // trips of two steps
}

spread_status somier_stream_run_blocked(somier_stream_t h, double* x, double* y, double* z, double* vx, double* vy,
                                        double* vz, double* xn, double* yn, double* zn, double* vxn, double* vyn,
                                        double* vzn, int64_t nsteps, int64_t steps_per_trip, somier_stats_t* stats) {
    if (!h || !x || !y || !z || !vx || !vy || !vz || !xn || !yn || !zn || !vxn || !vyn || !vzn)
        PAPER_FAIL(SPREAD_EINVAL, "somier_stream_run_blocked: NULL argument");
    if (nsteps < 0) PAPER_FAIL(SPREAD_EINVAL, "somier_stream_run_blocked: nsteps %lld < 0", (long long)nsteps);
    if (steps_per_trip < 1 || steps_per_trip > 256)
        PAPER_FAIL(SPREAD_EINVAL, "somier_stream_run_blocked: steps_per_trip %lld outside [1, 256]",
                   (long long)steps_per_trip);
    if (x == xn || y == yn || z == zn || vx == vxn || vy == vyn || vz == vzn)
        PAPER_FAIL(SPREAD_EINVAL, "somier_stream_run_blocked: the two X or the two V buffers alias");
    if (nsteps == 0) return SPREAD_OK;
    double* X[3] = {x, y, z};
    double* XN[3] = {xn, yn, zn};
    double* V[3] = {vx, vy, vz};
    double* VN[3] = {vxn, vyn, vzn};
    return stream_run_blocked(h, X, V, XN, VN, nsteps, steps_per_trip, stats);
}

spread_status somier_stream_traffic_blocked(somier_stream_t h, int64_t steps_per_trip, int64_t* h2d_bytes,
                                            int64_t* d2h_bytes) {
    if (!h || steps_per_trip < 1) PAPER_FAIL(SPREAD_EINVAL, "somier_stream_traffic_blocked: bad argument");
    const int64_t n0 = h->p.n[0], s = steps_per_trip;
    const int64_t plane = 3 * h->p.n[1] * h->p.n[2] * (int64_t)sizeof(double);
    int64_t in = 0, outb = 0;
    for (int64_t c = 0; c < h->spread.nchunks; c++) {
        const paper::ChunkInfo ci = h->spread.chunk_info(c);
        const int64_t xp = std::min<int64_t>(n0, ci.start + ci.size + s) - std::max<int64_t>(0, ci.start - s);
        const int64_t vd = std::max<int64_t>(1, s - 1);
        const int64_t vp = std::min<int64_t>(n0, ci.start + ci.size + vd) - std::max<int64_t>(0, ci.start - vd);
        in += plane * (xp + vp);
        outb += 2 * plane * ci.size;
    }
    outb += 4 * plane;  // fixed end planes of X and V
    if (h2d_bytes) *h2d_bytes = in;
    if (d2h_bytes) *d2h_bytes = outb;
    return SPREAD_OK;
}

spread_status somier_stream_traffic2(somier_stream_t h, int64_t* h2d_bytes, int64_t* d2h_bytes) {
    if (!h) PAPER_FAIL(SPREAD_EINVAL, "somier_stream_traffic2: NULL handle");
    return somier_stream_traffic_blocked(h, 2, h2d_bytes, d2h_bytes);
}

spread_status somier_stream_traffic(somier_stream_t h, int64_t* h2d_bytes, int64_t* d2h_bytes, int64_t* launches) {
    if (!h) PAPER_FAIL(SPREAD_EINVAL, "somier_stream_traffic: NULL handle");
    const int64_t plane = 3 * h->p.n[1] * h->p.n[2] * (int64_t)sizeof(double);
    int64_t in = 0, outb = 0;
    for (int64_t c = 0; c < h->spread.nchunks; c++) {
        const paper::ChunkInfo ci = h->spread.chunk_info(c);
        in += plane * (ci.size + 2) + plane * ci.size;
        outb += 2 * plane * ci.size;
    }
    outb += 2 * plane;  // fixed end planes
    if (h2d_bytes) *h2d_bytes = in;
    if (d2h_bytes) *d2h_bytes = outb;
    if (launches) *launches = h->launches;
    return SPREAD_OK;
}

spread_status somier_stream_set_delay(somier_stream_t h, int device_pos, int64_t ns) {
    if (!h || device_pos < 0 || device_pos >= (int)h->devs.size() || ns < 0)
        PAPER_FAIL(SPREAD_EINVAL, "somier_stream_set_delay: bad arguments");
    h->devs[(size_t)device_pos].delay_ns = ns;
    return SPREAD_OK;
}

spread_status somier_stream_chunk_counts(somier_stream_t h, int64_t* counts) {
    if (!h || !counts) PAPER_FAIL(SPREAD_EINVAL, "somier_stream_chunk_counts: NULL argument");
    for (size_t q = 0; q < h->devs.size(); q++) counts[q] = h->devs[q].chunks_run;
    return SPREAD_OK;
}

spread_status somier_stream_destroy(somier_stream_t h) {
    if (!h) return SPREAD_OK;
    destroy_all(h);
    delete h;
    return SPREAD_OK;
}

}  // extern "C"
