// spread.cpp -- the "target spread" descriptor: device list + iteration range +
// static round-robin schedule, and halo map extents (include/spread.h).
// Host-only logic; PAPER.md:95-116 (§III-B.1), 144-173 (Listing 5).
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <new>
#include <set>
#include <string>
#include <vector>

#include "spread_impl.hpp"
#include "status.hpp"

namespace paper {

static thread_local std::string g_last_error;

void set_last_error(const char* fmt, ...) {
    char buf[1024];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    g_last_error = buf;
}

void clear_last_error() { g_last_error.clear(); }

const char* last_error() { return g_last_error.c_str(); }

}  // namespace paper

using paper::set_last_error;

extern "C" {

spread_status spread_create(const int* devices, int ndevices, int64_t range_start, int64_t range_len,
                            spread_sched sched, int64_t chunk, spread_t* out) {
    if (!out) PAPER_FAIL(SPREAD_EINVAL, "spread_create: out is NULL");
    *out = nullptr;
    if (sched != SPREAD_SCHED_STATIC && sched != SPREAD_SCHED_DYNAMIC)
        PAPER_FAIL(SPREAD_ENOTSUP, "spread_create: unknown schedule %d (static: PAPER.md:101; dynamic: 771)",
                   (int)sched);
    if (!devices || ndevices < 1) PAPER_FAIL(SPREAD_EINVAL, "spread_create: empty devices() list");
    if (range_len < 0) PAPER_FAIL(SPREAD_EINVAL, "spread_create: range length %lld < 0", (long long)range_len);
    if (chunk < 0) PAPER_FAIL(SPREAD_EINVAL, "spread_create: chunk %lld < 0", (long long)chunk);
    std::set<int> seen;
    for (int i = 0; i < ndevices; i++) {
        if (devices[i] < 0) PAPER_FAIL(SPREAD_EINVAL, "spread_create: device id %d < 0", devices[i]);
        if (!seen.insert(devices[i]).second)
            PAPER_FAIL(SPREAD_EINVAL, "spread_create: device id %d listed twice", devices[i]);
    }
    spread_s* s = new (std::nothrow) spread_s;
    if (!s) PAPER_FAIL(SPREAD_ENOMEM, "spread_create: out of host memory");
    s->devices.assign(devices, devices + ndevices);
    s->range_start = range_start;
    s->range_len = range_len;
    s->dynamic = sched == SPREAD_SCHED_DYNAMIC;
    if (chunk == 0) chunk = range_len == 0 ? 1 : (range_len + ndevices - 1) / ndevices;
    s->chunk = chunk;
    s->nchunks = range_len == 0 ? 0 : (range_len + chunk - 1) / chunk;
    *out = s;
    return SPREAD_OK;
}

spread_status spread_create_sizes(const int* devices, int ndevices, int64_t range_start, int64_t range_len,
                                  const int64_t* sizes, int64_t nsizes, spread_t* out) {
    if (!out) PAPER_FAIL(SPREAD_EINVAL, "spread_create_sizes: out is NULL");
    *out = nullptr;
    if (nsizes < 0 || (nsizes > 0 && !sizes)) PAPER_FAIL(SPREAD_EINVAL, "spread_create_sizes: bad sizes array");
    int64_t total = 0, largest = 1;
    for (int64_t c = 0; c < nsizes; c++) {
        if (sizes[c] < 1)
            PAPER_FAIL(SPREAD_EINVAL, "spread_create_sizes: chunk %lld has size %lld < 1", (long long)c,
                       (long long)sizes[c]);
        if (sizes[c] > range_len - total)
            PAPER_FAIL(SPREAD_EINVAL, "spread_create_sizes: chunk sizes exceed the range length %lld",
                       (long long)range_len);
        total += sizes[c];
        largest = std::max<int64_t>(largest, sizes[c]);
    }
    if (total != range_len)
        PAPER_FAIL(SPREAD_EINVAL, "spread_create_sizes: chunk sizes sum to %lld, range length is %lld",
                   (long long)total, (long long)range_len);
    spread_t s = nullptr;
    spread_status st = spread_create(devices, ndevices, range_start, range_len, SPREAD_SCHED_STATIC, 0, &s);
    if (st != SPREAD_OK) return st;
    try {
        s->offsets.resize((size_t)nsizes + 1);
    } catch (...) {
        delete s;
        PAPER_FAIL(SPREAD_ENOMEM, "spread_create_sizes: out of host memory");
    }
    s->offsets[0] = 0;
    for (int64_t c = 0; c < nsizes; c++) s->offsets[c + 1] = s->offsets[c] + sizes[c];
    s->nchunks = nsizes;
    s->chunk = largest;
    *out = s;
    return SPREAD_OK;
}

spread_status spread_create_weighted(const int* devices, int ndevices, int64_t range_start, int64_t range_len,
                                     const double* weights, spread_t* out) {
    if (!out) PAPER_FAIL(SPREAD_EINVAL, "spread_create_weighted: out is NULL");
    *out = nullptr;
    if (!devices || ndevices < 1) PAPER_FAIL(SPREAD_EINVAL, "spread_create_weighted: empty devices() list");
    if (!weights) PAPER_FAIL(SPREAD_EINVAL, "spread_create_weighted: weights is NULL");
    if (range_len < ndevices)
        PAPER_FAIL(SPREAD_EINVAL, "spread_create_weighted: range length %lld < %d devices", (long long)range_len,
                   ndevices);
    double wsum = 0.0;
    for (int d = 0; d < ndevices; d++) {
        if (!(weights[d] > 0.0) || !std::isfinite(weights[d]))
            PAPER_FAIL(SPREAD_EINVAL, "spread_create_weighted: weight %d is not a positive finite number", d);
        wsum += weights[d];
    }
    if (!std::isfinite(wsum)) PAPER_FAIL(SPREAD_EINVAL, "spread_create_weighted: weights overflow");
    // One chunk per list position: 1 iteration each, the remaining len - p
    // shared by largest remainder of w_d / sum(w) (ties to the earlier position).
    std::vector<int64_t> sizes((size_t)ndevices, 1);
    std::vector<double> rem((size_t)ndevices);
    const int64_t spare = range_len - ndevices;
    int64_t given = 0;
    for (int d = 0; d < ndevices; d++) {
        const double share = (double)spare * (weights[d] / wsum);
        int64_t f = (int64_t)std::floor(share);
        f = std::min<int64_t>(f, spare - given);
        sizes[d] += f;
        given += f;
        rem[d] = share - (double)f;
    }
    while (given < spare) {
        int best = 0;
        for (int d = 1; d < ndevices; d++)
            if (rem[d] > rem[best]) best = d;
        sizes[best] += 1;
        rem[best] = -1.0;
        given += 1;
    }
    return spread_create_sizes(devices, ndevices, range_start, range_len, sizes.data(), ndevices, out);
}

spread_status spread_destroy(spread_t s) {
    delete s;
    return SPREAD_OK;
}

spread_status spread_num_chunks(spread_t s, int64_t* nchunks) {
    if (!s) PAPER_FAIL(SPREAD_EINVAL, "spread_num_chunks: NULL handle");
    if (nchunks) *nchunks = s->nchunks;
    return SPREAD_OK;
}

spread_status spread_num_devices(spread_t s, int* ndevices) {
    if (!s) PAPER_FAIL(SPREAD_EINVAL, "spread_num_devices: NULL handle");
    if (ndevices) *ndevices = (int)s->devices.size();
    return SPREAD_OK;
}

spread_status spread_device(spread_t s, int pos, int* device_id) {
    if (!s) PAPER_FAIL(SPREAD_EINVAL, "spread_device: NULL handle");
    if (pos < 0 || pos >= (int)s->devices.size())
        PAPER_FAIL(SPREAD_EINVAL, "spread_device: position %d outside the %zu-device list", pos, s->devices.size());
    if (device_id) *device_id = s->devices[pos];
    return SPREAD_OK;
}

spread_status spread_schedule_kind(spread_t s, spread_sched* sched) {
    if (!s || !sched) PAPER_FAIL(SPREAD_EINVAL, "spread_schedule_kind: NULL argument");
    *sched = s->dynamic ? SPREAD_SCHED_DYNAMIC : SPREAD_SCHED_STATIC;
    return SPREAD_OK;
}

spread_status spread_chunk_size(spread_t s, int64_t* chunk) {
    if (!s) PAPER_FAIL(SPREAD_EINVAL, "spread_chunk_size: NULL handle");
    if (chunk) *chunk = s->chunk;
    return SPREAD_OK;
}

spread_status spread_range(spread_t s, int64_t* range_start, int64_t* range_len) {
    if (!s) PAPER_FAIL(SPREAD_EINVAL, "spread_range: NULL handle");
    if (range_start) *range_start = s->range_start;
    if (range_len) *range_len = s->range_len;
    return SPREAD_OK;
}

spread_status spread_get_chunk(spread_t s, int64_t c, int* device_pos, int* device_id, int64_t* start,
                               int64_t* size) {
    if (!s) PAPER_FAIL(SPREAD_EINVAL, "spread_get_chunk: NULL handle");
    if (c < 0 || c >= s->nchunks)
        PAPER_FAIL(SPREAD_EINVAL, "spread_get_chunk: chunk %lld outside [0, %lld)", (long long)c,
                   (long long)s->nchunks);
    paper::ChunkInfo ci = s->chunk_info(c);
    if (device_pos) *device_pos = ci.pos;
    if (device_id) *device_id = ci.device;
    if (start) *start = ci.start;
    if (size) *size = ci.size;
    return SPREAD_OK;
}

spread_status spread_chunk_of(spread_t s, int64_t iter, int64_t* chunk_index) {
    if (!s) PAPER_FAIL(SPREAD_EINVAL, "spread_chunk_of: NULL handle");
    if (iter < s->range_start || iter >= s->range_start + s->range_len)
        PAPER_FAIL(SPREAD_EINVAL, "spread_chunk_of: iteration %lld outside the range", (long long)iter);
    if (chunk_index) *chunk_index = s->chunk_of(iter);
    return SPREAD_OK;
}

spread_status spread_map_extent(spread_t s, int64_t c, spread_map m, int64_t array_len, int64_t* first,
                                int64_t* len) {
    if (!s) PAPER_FAIL(SPREAD_EINVAL, "spread_map_extent: NULL handle");
    if (c < 0 || c >= s->nchunks)
        PAPER_FAIL(SPREAD_EINVAL, "spread_map_extent: chunk %lld outside [0, %lld)", (long long)c,
                   (long long)s->nchunks);
    if (m.type < SPREAD_MAP_ALLOC || m.type > SPREAD_MAP_TOFROM)
        PAPER_FAIL(SPREAD_EINVAL, "spread_map_extent: unknown map type %d", (int)m.type);
    if (m.lo_halo < 0 || m.hi_halo < 0) PAPER_FAIL(SPREAD_EINVAL, "spread_map_extent: negative halo");
    paper::ChunkInfo ci = s->chunk_info(c);
    int64_t f = ci.start - m.lo_halo;
    int64_t l = ci.size + m.lo_halo + m.hi_halo;
    if (f < 0 || f + l > array_len)
        PAPER_FAIL(SPREAD_EINVAL,
                   "spread_map_extent: section [%lld, %lld) of chunk %lld leaves the array [0, %lld)",
                   (long long)f, (long long)(f + l), (long long)c, (long long)array_len);
    if (first) *first = f;
    if (len) *len = l;
    return SPREAD_OK;
}

const char* spread_last_error(void) { return paper::last_error(); }

const char* spread_status_string(spread_status st) {
    switch (st) {
        case SPREAD_OK: return "SPREAD_OK";
        case SPREAD_EINVAL: return "SPREAD_EINVAL";
        case SPREAD_ENODEV: return "SPREAD_ENODEV";
        case SPREAD_ENOMEM: return "SPREAD_ENOMEM";
        case SPREAD_ECUDA: return "SPREAD_ECUDA";
        case SPREAD_ENCCL: return "SPREAD_ENCCL";
        case SPREAD_ENOTSUP: return "SPREAD_ENOTSUP";
        case SPREAD_ESTATE: return "SPREAD_ESTATE";
    }
    return "SPREAD_<unknown>";
}

}  // extern "C"
