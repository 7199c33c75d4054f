// guard.hpp -- SOMIER_GUARD: a device-memory bounds check for debug runs.
//
// With SOMIER_GUARD=1 in the environment (off by default: the layouts are then
// exactly the unguarded ones), every device block the Somier handles allocate
// for their state -- the resident chunks (X_0, X_1, V, V', stats) and the
// host-streamed slots (X in/out, V) -- gets guard zones before, between and
// after its regions, at least two planes or 64 KiB each, filled with
// kGuardByte. The handles' synchronising calls copy the zones back and fail
// with SPREAD_ECUDA (sticky) naming the zone if any byte changed: an
// out-of-bounds write by a kernel, a fused halo store or a copy. It is the
// device-memory check of the GPU suite where compute-sanitizer is unavailable
// (tests/test_gpu_guard.py runs the parity and stream suites under it).
// SOMIER_GUARD_SELFTEST=1 clobbers one guard byte at allocation: the test of
// the check itself.
#pragma once
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

namespace paper {

constexpr unsigned char kGuardByte = 0xA5;

inline bool env_flag(const char* name) {
    const char* e = std::getenv(name);
    return e && *e && std::strcmp(e, "0") != 0;
}

// guard zone size for blocks of planes of `plane` bytes (0: guard mode off)
inline size_t guard_bytes(size_t plane) {
    static const bool on = env_flag("SOMIER_GUARD");
    if (!on) return 0;
    const size_t g = std::max<size_t>(65536, 2 * plane);
    return (g + 4095) / 4096 * 4096;
}

inline bool guard_selftest() {
    static const bool on = env_flag("SOMIER_GUARD_SELFTEST");
    return on;
}

// Offsets of a block of regions laid out as [guard] r0 [guard] r1 ... [guard]
// (no guards when G == 0). Regions start 4096-aligned when their sizes are.
struct GuardLayout {
    size_t G = 0, bytes = 0;
    std::vector<size_t> off;              // region offsets
    std::vector<size_t> guard_off;        // guard zone offsets
    std::vector<const char*> guard_name;  // the region each zone precedes ("end" for the last)

    void plan(size_t guard, const std::vector<std::pair<size_t, const char*>>& regions) {
        G = guard;
        off.clear();
        guard_off.clear();
        guard_name.clear();
        size_t at = 0;
        for (const auto& r : regions) {
            if (G) {
                guard_off.push_back(at);
                guard_name.push_back(r.second);
            }
            off.push_back(at + G);
            at += G + r.first;
        }
        bytes = (at + 4095) / 4096 * 4096;
        if (G) {
            guard_off.push_back(bytes);
            guard_name.push_back("end");
            bytes += G;
        }
    }
};

// fill the zones (and, in self-test mode, clobber one byte of the second zone)
inline cudaError_t guard_fill(const GuardLayout& L, void* base, cudaStream_t s) {
    for (size_t o : L.guard_off) {
        cudaError_t e = cudaMemsetAsync((char*)base + o, kGuardByte, L.G, s);
        if (e != cudaSuccess) return e;
    }
    if (L.G && guard_selftest() && L.guard_off.size() > 1)
        return cudaMemsetAsync((char*)base + L.guard_off[1] + L.G / 2, 0, 1, s);
    return cudaSuccess;
}

// compare the zones with kGuardByte (the caller has synchronised); false and a
// message naming the first damaged zone if any byte changed
inline bool guard_check(const GuardLayout& L, const void* base, const char* what, std::string& msg, cudaError_t& err) {
    err = cudaSuccess;
    if (!L.G || !base) return true;
    std::vector<unsigned char> buf(L.G);
    for (size_t z = 0; z < L.guard_off.size(); z++) {
        err = cudaMemcpy(buf.data(), (const char*)base + L.guard_off[z], L.G, cudaMemcpyDeviceToHost);
        if (err != cudaSuccess) return false;
        size_t bad = 0, first = 0;
        for (size_t b = 0; b < L.G; b++)
            if (buf[b] != kGuardByte && bad++ == 0) first = b;
        if (bad) {
            char m[256];
            std::snprintf(m, sizeof m, "SOMIER_GUARD: %zu byte(s) written out of bounds in the guard zone before %s of %s, "
                          "first at +%zu", bad, L.guard_name[z], what, first);
            msg = m;
            return false;
        }
    }
    return true;
}

}  // namespace paper
