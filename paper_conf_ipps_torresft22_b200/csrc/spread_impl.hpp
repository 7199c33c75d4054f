// spread_impl.hpp -- the descriptor behind the opaque spread_t.
#pragma once
#include <algorithm>
#include <cstdint>
#include <vector>

#include "spread.h"

namespace paper {

struct ChunkInfo {
    int64_t index;   // chunk number c
    int pos;         // list position (c mod ndevices): distribution order
    int device;      // device id at that position
    int64_t start;   // omp_spread_start
    int64_t size;    // omp_spread_size
};

const char* last_error();

}  // namespace paper

struct spread_s {
    std::vector<int> devices;
    int64_t range_start = 0;
    int64_t range_len = 0;
    int64_t chunk = 1;      // regular: the chunk size; irregular: the largest chunk
    int64_t nchunks = 0;
    bool dynamic = false;   // spread_schedule(dynamic, chunk): positions chosen at run time
    // Irregular static schedule (future work): chunk c covers
    // [range_start + offsets[c], range_start + offsets[c+1]). Empty = regular.
    std::vector<int64_t> offsets;

    // Static round-robin: chunk c covers iterations
    // [start + c*chunk, min(start + (c+1)*chunk, start + len)) on list position c mod p.
    paper::ChunkInfo chunk_info(int64_t c) const {
        paper::ChunkInfo ci;
        ci.index = c;
        ci.pos = (int)(c % (int64_t)devices.size());
        ci.device = devices[ci.pos];
        if (!offsets.empty()) {
            ci.start = range_start + offsets[c];
            ci.size = offsets[c + 1] - offsets[c];
            return ci;
        }
        ci.start = range_start + c * chunk;
        int64_t end = range_start + range_len;
        ci.size = (ci.start + chunk <= end) ? chunk : end - ci.start;
        return ci;
    }

    // The chunk that executes iteration `iter` (inside the range).
    int64_t chunk_of(int64_t iter) const {
        const int64_t r = iter - range_start;
        if (offsets.empty()) return r / chunk;
        return (int64_t)(std::upper_bound(offsets.begin(), offsets.end(), r) - offsets.begin()) - 1;
    }

    // Largest chunk (buffer sizing).
    int64_t max_chunk() const { return std::min<int64_t>(chunk, range_len); }
};
