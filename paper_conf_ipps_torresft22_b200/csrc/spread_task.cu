// spread_task.cu -- chunk-level `depend` between spread constructs: the
// paper's future work (Listing 13; 727: "synchronizing data
// transfers with kernel computations at the chunk level, making the enclosing
// taskgroup directive no longer necessary").
//
//   spread_enter_data   target enter data spread map(to|alloc: A[start-lo : size+lo+hi])
//                       depend(out: A[start : size]) nowait
//   spread_task_stencil3 target spread map(A[start-1 : size+2], B[start : size])
//                       depend(in: A[start-1 : size+2]) depend(out: B[start : size]) nowait
//                       for (i ...) B[i] = A[i-1] + A[i] + A[i+1]        (Listing 3)
//   spread_task_reduce  target spread map(A[start : size]) depend(in: A[start : size])
//                       reduction(op: r) nowait
//   spread_exit_data    target exit data spread map(from: A[start : size]) depend(in: A[start : size]) nowait
//   spread_taskwait     taskwait: the only host barrier
//
// Every chunk has its own stream on its device; a task on chunk c waits only
// for the events of the chunk-level tasks its array sections overlap: the last
// write of each chunk whose owned elements it reads (RAW), the reads of the
// chunk it writes since that chunk's last write (WAR). An `in` section reaching
// into neighbour chunks (the stencil's halo) first refreshes the chunk's halo
// copy from the neighbours' device memory (peer copies) once they have written
// it. So chunk m+1's map(to) runs while chunk m's loop runs, across constructs,
// and a device never idles at a construct boundary.
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <new>
#include <string>
#include <vector>

#include "kernels/stats.cuh"
#include "spread.h"
#include "spread_impl.hpp"
#include "status.hpp"
#include "trace.hpp"

namespace {

__global__ void task_stencil3_kernel(const double* __restrict__ a, double* __restrict__ b, int64_t size) {
    // a: A[start-1 .. start+size], b: B[start .. start+size-1]; left to right as
    // the C expression A[i-1] + A[i] + A[i+1]
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < size; i += (int64_t)gridDim.x * blockDim.x)
        b[i] = __dadd_rn(__dadd_rn(a[i], a[i + 1]), a[i + 2]);
}

struct SumAcc {
    unsigned long long lo, hi, flags;  // exact 128-bit sum; flags 1: outside the exact domain
};

// SPREAD_REDUCE_SUM of one chunk into the task's accumulator (the exact split
// of spread_reduce / stats.cuh: q = round_half_even(x 2^scale_exp) = h 2^32 + l)
__global__ void __launch_bounds__(256) task_sum_kernel(const double* __restrict__ a, int64_t size, double scale,
                                                        SumAcc* acc) {
    __int128 s = 0;
    unsigned flags = 0;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < size; i += (int64_t)gridDim.x * blockDim.x) {
        const double v = __dmul_rn(a[i], scale);
        if (!(fabs(v) < 0x1p62)) {
            flags |= 1u;
        } else {
            const long long h = __double2ll_rn(v);
            const double r = __dsub_rn(v, (double)h);
            const long long l = __double2ll_rn(__dmul_rn(r, 0x1p32));
            s += (__int128)h * ((__int128)1 << 32) + (__int128)l;
        }
    }
#pragma unroll
    for (int m = 16; m > 0; m >>= 1) {
        s += paper::shfl_xor_i128(s, m);
        flags |= __shfl_xor_sync(0xffffffffu, flags, m);
    }
    if ((threadIdx.x & 31) == 0) {
        paper::atomic_add_i128(&acc->lo, &acc->hi, s);
        if (flags) atomicOr(&acc->flags, (unsigned long long)flags);
    }
}

int grid_for(int64_t n) { return (int)std::max<int64_t>(1, std::min<int64_t>((n + 255) / 256, 148 * 8)); }

using PFN_wait32 = CUresult (*)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
PFN_wait32 load_wait32() {
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult qr;
    if (cudaGetDriverEntryPoint("cuStreamWaitValue32", &fn, cudaEnableDefault, &qr) != cudaSuccess ||
        qr != cudaDriverEntryPointSuccess)
        return nullptr;
    return (PFN_wait32)fn;
}

}  // namespace

struct spread_data_s;

struct spread_tasks_s {
    spread_s spread;
    std::vector<int> cuda_dev;             // per list position
    std::vector<cudaStream_t> streams;     // per chunk
    std::vector<cudaEvent_t> live_events;  // destroyed at taskwait
    std::vector<spread_data_s*> data;
    struct ReduceTask {
        spread_reduce_result* out;
        int scale_exp;
        int64_t count;
        std::vector<SumAcc*> accs;  // per chunk, on the chunk's device
    };
    std::vector<ReduceTask> reductions;
    bool trace = false;
    struct TraceRec {
        int64_t chunk;
        int kind;
        cudaEvent_t a, b;
    };
    std::vector<TraceRec> trace_recs;
    cudaEvent_t trace_origin = nullptr;
    uint32_t* hold_word = nullptr;  // spread_tasks_hold: mapped pinned word the held streams wait on
    std::string sticky;
};

struct spread_data_s {
    spread_tasks_s* q = nullptr;
    int64_t n = 0, lo = 0, hi = 0;
    struct Chunk {
        double* ptr = nullptr;  // A[start-lo : size+lo+hi] (clipped to [0, n)), element first
        int64_t first = 0, len = 0;
        cudaEvent_t last_write = nullptr;    // of the owned elements [start, start+size)
        uint64_t version = 0;                // owned elements written so far (0: by enter data)
        std::vector<cudaEvent_t> reads;      // tasks that read the owned elements since the last write
        uint64_t halo_lo_ver = 0, halo_hi_ver = 0;  // owners' versions the halo copies hold
        int64_t halo_lo_owner = -1, halo_hi_owner = -1;
    };
    std::vector<Chunk> ch;
};

namespace {

struct Err {
    std::string msg;
    bool ok(cudaError_t r, const char* what) {
        if (r != cudaSuccess && msg.empty()) msg = std::string(what) + ": " + cudaGetErrorString(r);
        return r == cudaSuccess;
    }
};

spread_status fail_cuda(spread_tasks_s* q, const std::string& m) {
    if (q->sticky.empty()) q->sticky = m;
    PAPER_FAIL(SPREAD_ECUDA, "%s", m.c_str());
}

// an event recorded on chunk c's stream now (kept until the taskwait)
cudaEvent_t mark(spread_tasks_s* q, int64_t c, Err& e) {
    cudaEvent_t ev = nullptr;
    if (!e.ok(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming), "cudaEventCreate")) return nullptr;
    q->live_events.push_back(ev);
    e.ok(cudaEventRecord(ev, q->streams[(size_t)c]), "cudaEventRecord");
    return ev;
}

// trace: timing events around one task of chunk c
struct TraceScope {
    spread_tasks_s* q;
    int64_t c;
    int kind;
    cudaEvent_t a = nullptr;
    TraceScope(spread_tasks_s* q_, int64_t c_, int kind_, Err& e) : q(q_), c(c_), kind(kind_) {
        if (!q->trace) return;
        if (e.ok(cudaEventCreate(&a), "cudaEventCreate")) e.ok(cudaEventRecord(a, q->streams[(size_t)c]), "trace");
    }
    void end(Err& e) {
        if (!q->trace || !a) return;
        cudaEvent_t b = nullptr;
        if (e.ok(cudaEventCreate(&b), "cudaEventCreate")) e.ok(cudaEventRecord(b, q->streams[(size_t)c]), "trace");
        q->trace_recs.push_back({c, kind, a, b});
    }
};

spread_status check_open(spread_tasks_s* q, const char* who) {
    if (!q) PAPER_FAIL(SPREAD_EINVAL, "%s: NULL task queue", who);
    if (!q->sticky.empty()) PAPER_FAIL(SPREAD_ECUDA, "%s: %s", who, q->sticky.c_str());
    return SPREAD_OK;
}

// RAW: chunk c's stream waits for the last writes of the chunks owning any of
// the elements [x0, x1) it is about to read; the reads are recorded for WAR.
// Elements outside the spread's range are constant after enter data.
void depend_in(spread_data_s* d, int64_t c, int64_t x0, int64_t x1, Err& e, std::vector<int64_t>* owners) {
    spread_tasks_s* q = d->q;
    const spread_s& s = q->spread;
    const int64_t r0 = std::max(x0, s.range_start), r1 = std::min(x1, s.range_start + s.range_len);
    if (r0 >= r1) return;
    for (int64_t o = s.chunk_of(r0); o <= s.chunk_of(r1 - 1); o++) {
        auto& oc = d->ch[(size_t)o];
        if (oc.last_write) e.ok(cudaStreamWaitEvent(q->streams[(size_t)c], oc.last_write, 0), "depend(in)");
        if (owners) owners->push_back(o);
    }
}

// WAR / WAW: before chunk c's owned elements are rewritten
void depend_out(spread_data_s* d, int64_t c, Err& e) {
    spread_tasks_s* q = d->q;
    auto& cc = d->ch[(size_t)c];
    for (cudaEvent_t r : cc.reads) e.ok(cudaStreamWaitEvent(q->streams[(size_t)c], r, 0), "depend(out)");
    if (cc.last_write) e.ok(cudaStreamWaitEvent(q->streams[(size_t)c], cc.last_write, 0), "depend(out)");
}

void wrote(spread_data_s* d, int64_t c, Err& e) {
    auto& cc = d->ch[(size_t)c];
    cc.last_write = mark(d->q, c, e);
    cc.version++;
    cc.reads.clear();
}

// Bring chunk c's copies of elements [x0, x1) that other chunks own up to date
// (peer copies on chunk c's stream after the owners' writes), then note the
// reads in the owners' WAR lists. Used for the halo of an `in` section.
void refresh_halo(spread_data_s* d, int64_t c, int64_t x0, int64_t x1, bool lo_side, Err& e) {
    spread_tasks_s* q = d->q;
    const spread_s& s = q->spread;
    auto& cc = d->ch[(size_t)c];
    const int64_t r0 = std::max(x0, s.range_start), r1 = std::min(x1, s.range_start + s.range_len);
    if (r0 >= r1) return;
    for (int64_t o = s.chunk_of(r0); o <= s.chunk_of(r1 - 1); o++) {
        if (o == c) continue;
        auto& oc = d->ch[(size_t)o];
        uint64_t& have = lo_side ? cc.halo_lo_ver : cc.halo_hi_ver;
        int64_t& owner = lo_side ? cc.halo_lo_owner : cc.halo_hi_owner;
        const paper::ChunkInfo oi = s.chunk_info(o);
        const int64_t e0 = std::max(r0, oi.start), e1 = std::min(r1, oi.start + oi.size);
        if (owner == o && have == oc.version) continue;  // the copy is current (e.g. from enter data)
        if (oc.last_write) e.ok(cudaStreamWaitEvent(q->streams[(size_t)c], oc.last_write, 0), "depend(in: halo)");
        const int dst_dev = q->cuda_dev[(size_t)s.chunk_info(c).pos], src_dev = q->cuda_dev[(size_t)oi.pos];
        e.ok(cudaMemcpyPeerAsync(cc.ptr + (e0 - cc.first), dst_dev, oc.ptr + (e0 - oc.first), src_dev,
                                 (size_t)(e1 - e0) * sizeof(double), q->streams[(size_t)c]),
             "halo copy");
        oc.reads.push_back(mark(q, c, e));
        have = oc.version;
        owner = o;
    }
}

}  // namespace

extern "C" {

spread_status spread_tasks_create(spread_t s, const int* cuda_devices, spread_tasks_t* out) {
    if (!s || !out) PAPER_FAIL(SPREAD_EINVAL, "spread_tasks_create: NULL argument");
    *out = nullptr;
    if (s->dynamic)
        PAPER_FAIL(SPREAD_ENOTSUP, "spread_tasks_create: device-resident data is bound to its chunk's device "
                   "(dynamic schedules apply to the host-array loops and the host-streamed Somier)");
    int ndev = 0;
    cudaError_t r = cudaGetDeviceCount(&ndev);
    if (r != cudaSuccess) PAPER_FAIL(SPREAD_ENODEV, "spread_tasks_create: no CUDA device (%s)", cudaGetErrorString(r));
    spread_tasks_s* q = new (std::nothrow) spread_tasks_s;
    if (!q) PAPER_FAIL(SPREAD_ENOMEM, "spread_tasks_create: out of host memory");
    q->spread = *s;
    for (size_t p = 0; p < s->devices.size(); p++) {
        const int dev = cuda_devices ? cuda_devices[p] : s->devices[p];
        if (dev < 0 || dev >= ndev) {
            delete q;
            PAPER_FAIL(SPREAD_ENODEV, "spread_tasks_create: device %d not present (%d visible)", dev, ndev);
        }
        q->cuda_dev.push_back(dev);
    }
    Err e;
    for (int64_t c = 0; c < s->nchunks && e.msg.empty(); c++) {
        cudaStream_t st = nullptr;
        if (e.ok(cudaSetDevice(q->cuda_dev[(size_t)s->chunk_info(c).pos]), "cudaSetDevice") &&
            e.ok(cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking), "cudaStreamCreate"))
            q->streams.push_back(st);
    }
    // peer access between the devices of neighbouring chunks (halo copies)
    for (int64_t c = 0; c + 1 < s->nchunks && e.msg.empty(); c++) {
        const int a = q->cuda_dev[(size_t)s->chunk_info(c).pos], b = q->cuda_dev[(size_t)s->chunk_info(c + 1).pos];
        if (a == b) continue;
        for (int dir = 0; dir < 2; dir++) {
            int can = 0;
            cudaDeviceCanAccessPeer(&can, dir ? b : a, dir ? a : b);
            if (!can) continue;  // cudaMemcpyPeerAsync stages through the host
            cudaSetDevice(dir ? b : a);
            cudaError_t pe = cudaDeviceEnablePeerAccess(dir ? a : b, 0);
            if (pe == cudaErrorPeerAccessAlreadyEnabled) cudaGetLastError();
            else e.ok(pe, "cudaDeviceEnablePeerAccess");
        }
    }
    if (!e.msg.empty()) {
        spread_tasks_destroy(q);
        PAPER_FAIL(SPREAD_ECUDA, "spread_tasks_create: %s", e.msg.c_str());
    }
    *out = q;
    return SPREAD_OK;
}

spread_status spread_enter_data(spread_tasks_t q, const double* host, int64_t n, spread_map m, spread_data_t* out) {
    PAPER_NVTX("spread_enter_data");
    spread_status st = check_open(q, "spread_enter_data");
    if (st != SPREAD_OK) return st;
    if (!out || n < 0 || m.lo_halo < 0 || m.hi_halo < 0) PAPER_FAIL(SPREAD_EINVAL, "spread_enter_data: bad arguments");
    if (m.type != SPREAD_MAP_ALLOC && m.type != SPREAD_MAP_TO)
        PAPER_FAIL(SPREAD_EINVAL, "spread_enter_data: map type must be alloc or to");
    if (m.type == SPREAD_MAP_TO && !host) PAPER_FAIL(SPREAD_EINVAL, "spread_enter_data: map(to) needs a host array");
    const spread_s& s = q->spread;
    if (s.nchunks > 0 && (s.range_start < 0 || s.range_start + s.range_len > n))
        PAPER_FAIL(SPREAD_EINVAL, "spread_enter_data: range outside the array [0, %lld)", (long long)n);
    *out = nullptr;
    spread_data_s* d = new (std::nothrow) spread_data_s;
    if (!d) PAPER_FAIL(SPREAD_ENOMEM, "spread_enter_data: out of host memory");
    d->q = q;
    d->n = n;
    d->lo = m.lo_halo;
    d->hi = m.hi_halo;
    d->ch.resize((size_t)s.nchunks);
    q->data.push_back(d);
    Err e;
    for (int64_t c = 0; c < s.nchunks && e.msg.empty(); c++) {
        const paper::ChunkInfo ci = s.chunk_info(c);
        auto& cc = d->ch[(size_t)c];
        cc.first = std::max<int64_t>(0, ci.start - m.lo_halo);
        cc.len = std::min<int64_t>(n, ci.start + ci.size + m.hi_halo) - cc.first;
        if (!e.ok(cudaSetDevice(q->cuda_dev[(size_t)ci.pos]), "cudaSetDevice")) break;
        if (!e.ok(cudaMallocAsync((void**)&cc.ptr, std::max<int64_t>(1, cc.len) * sizeof(double),
                                  q->streams[(size_t)c]), "cudaMallocAsync"))
            break;
        TraceScope tr(q, c, 0, e);
        if (m.type == SPREAD_MAP_TO)
            e.ok(cudaMemcpyAsync(cc.ptr, host + cc.first, cc.len * sizeof(double), cudaMemcpyHostToDevice,
                                 q->streams[(size_t)c]), "map(to)");
        tr.end(e);
        // the halo copies hold the values the host had: current w.r.t. the owners' enter
        cc.halo_lo_owner = ci.start > s.range_start ? c - 1 : -1;
        cc.halo_hi_owner = ci.start + ci.size < s.range_start + s.range_len ? c + 1 : -1;
        wrote(d, c, e);
        cc.version = 0;
    }
    *out = d;  // owned by the queue (released at spread_tasks_destroy)
    if (!e.msg.empty()) return fail_cuda(q, "spread_enter_data: " + e.msg);
    return SPREAD_OK;
}

spread_status spread_task_stencil3(spread_tasks_t q, spread_data_t a, spread_data_t b) {
    PAPER_NVTX("spread_task_stencil3");
    spread_status st = check_open(q, "spread_task_stencil3");
    if (st != SPREAD_OK) return st;
    if (!a || !b || a->q != q || b->q != q || a == b)
        PAPER_FAIL(SPREAD_EINVAL, "spread_task_stencil3: A and B must be two data of this queue");
    const spread_s& s = q->spread;
    if (a->lo < 1 || a->hi < 1) PAPER_FAIL(SPREAD_EINVAL, "spread_task_stencil3: A needs a one-element halo (map A[start-1:size+2])");
    if (s.nchunks > 0 && (s.range_start < 1 || s.range_start + s.range_len > a->n - 1 || b->n != a->n))
        PAPER_FAIL(SPREAD_EINVAL, "spread_task_stencil3: range outside the loop [1, n-1)");
    Err e;
    for (int64_t c = 0; c < s.nchunks && e.msg.empty(); c++) {
        const paper::ChunkInfo ci = s.chunk_info(c);
        auto& ac = a->ch[(size_t)c];
        auto& bc = b->ch[(size_t)c];
        if (!e.ok(cudaSetDevice(q->cuda_dev[(size_t)ci.pos]), "cudaSetDevice")) break;
        // depend(in: A[start-1 : size+2]): own chunk + the neighbours' edge elements
        depend_in(a, c, ci.start, ci.start + ci.size, e, nullptr);
        refresh_halo(a, c, ci.start - 1, ci.start, true, e);
        refresh_halo(a, c, ci.start + ci.size, ci.start + ci.size + 1, false, e);
        // depend(out: B[start : size])
        depend_out(b, c, e);
        TraceScope tr(q, c, 1, e);
        task_stencil3_kernel<<<grid_for(ci.size), 256, 0, q->streams[(size_t)c]>>>(
            ac.ptr + (ci.start - 1 - ac.first), bc.ptr + (ci.start - bc.first), ci.size);
        e.ok(cudaGetLastError(), "stencil3 kernel");
        tr.end(e);
        ac.reads.push_back(mark(q, c, e));
        wrote(b, c, e);
    }
    if (!e.msg.empty()) return fail_cuda(q, "spread_task_stencil3: " + e.msg);
    return SPREAD_OK;
}

spread_status spread_task_reduce(spread_tasks_t q, spread_data_t a, int scale_exp, spread_reduce_result* out) {
    PAPER_NVTX("spread_task_reduce");
    spread_status st = check_open(q, "spread_task_reduce");
    if (st != SPREAD_OK) return st;
    if (!a || a->q != q || !out) PAPER_FAIL(SPREAD_EINVAL, "spread_task_reduce: bad arguments");
    if (scale_exp < -990 || scale_exp > 1023)
        PAPER_FAIL(SPREAD_EINVAL, "spread_task_reduce: scale_exp %d outside [-990, 1023]", scale_exp);
    const spread_s& s = q->spread;
    if (s.range_len >= ((int64_t)1 << 33)) PAPER_FAIL(SPREAD_EINVAL, "spread_task_reduce: more than 2^33 iterations");
    spread_tasks_s::ReduceTask rt;
    rt.out = out;
    rt.scale_exp = scale_exp;
    rt.count = s.range_len;
    const double kscale = std::ldexp(1.0, scale_exp - 32);
    Err e;
    for (int64_t c = 0; c < s.nchunks && e.msg.empty(); c++) {
        const paper::ChunkInfo ci = s.chunk_info(c);
        auto& ac = a->ch[(size_t)c];
        SumAcc* acc = nullptr;
        if (!e.ok(cudaSetDevice(q->cuda_dev[(size_t)ci.pos]), "cudaSetDevice")) break;
        cudaStream_t sc = q->streams[(size_t)c];
        if (!e.ok(cudaMallocAsync((void**)&acc, sizeof(SumAcc), sc), "cudaMallocAsync")) break;
        rt.accs.push_back(acc);
        e.ok(cudaMemsetAsync(acc, 0, sizeof(SumAcc), sc), "cudaMemsetAsync");
        depend_in(a, c, ci.start, ci.start + ci.size, e, nullptr);  // depend(in: A[start : size])
        TraceScope tr(q, c, 2, e);
        task_sum_kernel<<<grid_for(ci.size), 256, 0, sc>>>(ac.ptr + (ci.start - ac.first), ci.size, kscale, acc);
        e.ok(cudaGetLastError(), "reduce kernel");
        tr.end(e);
        ac.reads.push_back(mark(q, c, e));
    }
    q->reductions.push_back(rt);
    if (!e.msg.empty()) return fail_cuda(q, "spread_task_reduce: " + e.msg);
    return SPREAD_OK;
}

spread_status spread_exit_data(spread_tasks_t q, spread_data_t a, double* host) {
    PAPER_NVTX("spread_exit_data");
    spread_status st = check_open(q, "spread_exit_data");
    if (st != SPREAD_OK) return st;
    if (!a || a->q != q || !host) PAPER_FAIL(SPREAD_EINVAL, "spread_exit_data: bad arguments");
    const spread_s& s = q->spread;
    Err e;
    for (int64_t c = 0; c < s.nchunks && e.msg.empty(); c++) {
        const paper::ChunkInfo ci = s.chunk_info(c);
        auto& ac = a->ch[(size_t)c];
        if (!e.ok(cudaSetDevice(q->cuda_dev[(size_t)ci.pos]), "cudaSetDevice")) break;
        depend_in(a, c, ci.start, ci.start + ci.size, e, nullptr);  // depend(in: A[start : size])
        TraceScope tr(q, c, 3, e);
        e.ok(cudaMemcpyAsync(host + ci.start, ac.ptr + (ci.start - ac.first), ci.size * sizeof(double),
                             cudaMemcpyDeviceToHost, q->streams[(size_t)c]), "map(from)");
        tr.end(e);
        ac.reads.push_back(mark(q, c, e));
    }
    if (!e.msg.empty()) return fail_cuda(q, "spread_exit_data: " + e.msg);
    return SPREAD_OK;
}

spread_status spread_taskwait(spread_tasks_t q) {
    PAPER_NVTX("spread_taskwait");
    if (!q) PAPER_FAIL(SPREAD_EINVAL, "spread_taskwait: NULL task queue");
    Err e;
    for (int64_t c = 0; c < (int64_t)q->streams.size(); c++) {
        e.ok(cudaSetDevice(q->cuda_dev[(size_t)q->spread.chunk_info(c).pos]), "cudaSetDevice");
        e.ok(cudaStreamSynchronize(q->streams[(size_t)c]), "taskwait");
    }
    bool domain = false;
    for (auto& rt : q->reductions) {
        __int128 sum = 0;
        for (size_t c = 0; c < rt.accs.size(); c++) {
            SumAcc r{};
            e.ok(cudaSetDevice(q->cuda_dev[(size_t)q->spread.chunk_info((int64_t)c).pos]), "cudaSetDevice");
            e.ok(cudaMemcpy(&r, rt.accs[c], sizeof r, cudaMemcpyDeviceToHost), "reduction result");
            sum += (__int128)(((unsigned __int128)r.hi << 64) | r.lo);
            domain = domain || (r.flags & 1u);
            cudaFreeAsync(rt.accs[c], q->streams[c]);
        }
        rt.out->count = rt.count;
        rt.out->sum_lo = (uint64_t)(unsigned __int128)sum;
        rt.out->sum_hi = (int64_t)(sum >> 64);
        rt.out->value = std::ldexp((double)sum, -rt.scale_exp);
    }
    q->reductions.clear();
    // every dependency is satisfied now: the chunk states start over
    for (cudaEvent_t ev : q->live_events) cudaEventDestroy(ev);
    q->live_events.clear();
    for (auto* d : q->data)
        for (auto& cc : d->ch) {
            cc.last_write = nullptr;
            cc.reads.clear();
        }
    if (!e.msg.empty()) return fail_cuda(q, "spread_taskwait: " + e.msg);
    if (domain) PAPER_FAIL(SPREAD_EINVAL, "spread_taskwait: a reduced element is outside the exact domain");
    return SPREAD_OK;
}

spread_status spread_tasks_hold(spread_tasks_t q, int64_t chunk) {
    if (!q || chunk < 0 || chunk >= (int64_t)q->streams.size())
        PAPER_FAIL(SPREAD_EINVAL, "spread_tasks_hold: bad arguments");
    static PFN_wait32 wait32 = load_wait32();
    if (!wait32) PAPER_FAIL(SPREAD_ECUDA, "spread_tasks_hold: cuStreamWaitValue32 unavailable");
    if (!q->hold_word) {
        cudaSetDevice(q->cuda_dev[(size_t)q->spread.chunk_info(0).pos]);
        if (cudaHostAlloc((void**)&q->hold_word, sizeof(uint32_t), cudaHostAllocMapped | cudaHostAllocPortable) !=
            cudaSuccess)
            PAPER_FAIL(SPREAD_ENOMEM, "spread_tasks_hold: cudaHostAlloc");
        *q->hold_word = 0u;
    }
    void* dptr = nullptr;
    cudaSetDevice(q->cuda_dev[(size_t)q->spread.chunk_info(chunk).pos]);
    if (cudaHostGetDevicePointer(&dptr, (void*)q->hold_word, 0) != cudaSuccess)
        PAPER_FAIL(SPREAD_ECUDA, "spread_tasks_hold: cudaHostGetDevicePointer");
    *q->hold_word = 0u;
    if (wait32((CUstream)q->streams[(size_t)chunk], (CUdeviceptr)dptr, 1u, CU_STREAM_WAIT_VALUE_GEQ) != CUDA_SUCCESS)
        PAPER_FAIL(SPREAD_ECUDA, "spread_tasks_hold: cuStreamWaitValue32");
    return SPREAD_OK;
}

spread_status spread_tasks_release(spread_tasks_t q) {
    if (!q) PAPER_FAIL(SPREAD_EINVAL, "spread_tasks_release: NULL task queue");
    if (q->hold_word) *(volatile uint32_t*)q->hold_word = 1u;
    return SPREAD_OK;
}

spread_status spread_tasks_set_trace(spread_tasks_t q, int on) {
    if (!q) PAPER_FAIL(SPREAD_EINVAL, "spread_tasks_set_trace: NULL task queue");
    q->trace = on != 0;
    if (q->trace && !q->trace_origin && !q->streams.empty()) {
        cudaSetDevice(q->cuda_dev[(size_t)q->spread.chunk_info(0).pos]);
        if (cudaEventCreate(&q->trace_origin) != cudaSuccess ||
            cudaEventRecord(q->trace_origin, q->streams[0]) != cudaSuccess)
            PAPER_FAIL(SPREAD_ECUDA, "spread_tasks_set_trace: event");
    }
    return SPREAD_OK;
}

spread_status spread_tasks_trace(spread_tasks_t q, spread_task_record* recs, int64_t cap, int64_t* count) {
    if (!q || !count || (cap > 0 && !recs)) PAPER_FAIL(SPREAD_EINVAL, "spread_tasks_trace: bad arguments");
    spread_status st = spread_taskwait(q);
    if (st != SPREAD_OK) return st;
    *count = (int64_t)q->trace_recs.size();
    for (int64_t i = 0; i < std::min<int64_t>(cap, *count); i++) {
        const auto& r = q->trace_recs[(size_t)i];
        float a = 0.f, b = 0.f;
        cudaEventElapsedTime(&a, q->trace_origin, r.a);
        cudaEventElapsedTime(&b, q->trace_origin, r.b);
        recs[i].chunk = r.chunk;
        recs[i].kind = r.kind;
        recs[i].start_ms = a;
        recs[i].end_ms = b;
    }
    return SPREAD_OK;
}

spread_status spread_tasks_destroy(spread_tasks_t q) {
    if (!q) return SPREAD_OK;
    if (q->hold_word) *(volatile uint32_t*)q->hold_word = 1u;  // never leave a held stream behind
    for (int64_t c = 0; c < (int64_t)q->streams.size(); c++) {
        cudaSetDevice(q->cuda_dev[(size_t)q->spread.chunk_info(c).pos]);
        cudaStreamSynchronize(q->streams[(size_t)c]);
    }
    for (auto& rt : q->reductions)
        for (size_t c = 0; c < rt.accs.size(); c++) {
            cudaSetDevice(q->cuda_dev[(size_t)q->spread.chunk_info((int64_t)c).pos]);
            cudaFreeAsync(rt.accs[c], q->streams[c]);
        }
    for (auto* d : q->data) {
        for (size_t c = 0; c < d->ch.size(); c++)
            if (d->ch[c].ptr) {
                cudaSetDevice(q->cuda_dev[(size_t)q->spread.chunk_info((int64_t)c).pos]);
                cudaFreeAsync(d->ch[c].ptr, q->streams[c]);
            }
        delete d;
    }
    for (int64_t c = 0; c < (int64_t)q->streams.size(); c++) {
        cudaSetDevice(q->cuda_dev[(size_t)q->spread.chunk_info(c).pos]);
        cudaStreamSynchronize(q->streams[(size_t)c]);
    }
    for (cudaEvent_t ev : q->live_events) cudaEventDestroy(ev);
    for (auto& r : q->trace_recs) {
        cudaEventDestroy(r.a);
        cudaEventDestroy(r.b);
    }
    if (q->trace_origin) cudaEventDestroy(q->trace_origin);
    if (q->hold_word) cudaFreeHost(q->hold_word);
    for (int64_t c = 0; c < (int64_t)q->streams.size(); c++) {
        cudaSetDevice(q->cuda_dev[(size_t)q->spread.chunk_info(c).pos]);
        cudaStreamDestroy(q->streams[(size_t)c]);
    }
    delete q;
    return SPREAD_OK;
}

}  // extern "C"
