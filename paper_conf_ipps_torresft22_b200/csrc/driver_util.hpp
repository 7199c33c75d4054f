// driver_util.hpp -- helpers shared by the resident driver (somier.cpp) and the
// host-streamed driver (somier_stream.cpp).
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>

#include "kernels.hpp"
#include "somier.h"

namespace paper {

// Parameter validation of somier_params (EINVAL with a message).
spread_status check_somier_params(const somier_params* p);

// centre = S * 2^-60 / (n0 n1 n2), vmax = sqrt(max v.v); fills every field.
void finish_somier_stats(const somier_params* p, const __int128 sums[3], unsigned long long vmax2, int64_t nodes,
                         int64_t step, somier_stats_t* out, bool in_domain = true);

// cudaMemcpy3DAsync between `nplanes` planes of one component of a slab
// (planes of 3 component blocks, row pitch g.ld) and a dense host grid of that
// component (n0 x n1 x n2).
cudaError_t copy_slab_planes(const SlabGeom& g, double* slab, int comp, int64_t slab_plane, double* host,
                             int64_t host_plane, int64_t nplanes, cudaMemcpyKind kind, cudaStream_t s);

// 4-D fp64 TMA descriptor over a slab: dims (n2, n1, 3, planes), box (box_k, box_j, 3, 1).
spread_status encode_slab_tmap(CUtensorMap* map, const SlabGeom& g, double* base, int64_t planes, uint32_t box_k,
                               uint32_t box_j);

// Box shapes K1_MARCH expects for the X and V maps.
constexpr uint32_t kXBoxK = 36, kXBoxJ = 10, kVBoxK = 32, kVBoxJ = 8;
// ... and K1_MARCH2 (two rows per warp, 32 x 16 tiles)
constexpr uint32_t kX2BoxJ = 18, kV2BoxJ = 16;
// ... and K1_TB2 (owned 30 x 22 tiles, ring-extended 32 x 24, boxes with a one-node ring)
constexpr uint32_t kTB2XBoxK = 36, kTB2XBoxJ = 2 * kTB2Warps + 2, kTB2VBoxK = 34, kTB2VBoxJ = 2 * kTB2Warps;

// somier_params.kernel -> K1 implementation (AUTO = the fastest measured)
inline K1Variant k1_variant(int32_t kernel) {
    switch (kernel) {
        case SOMIER_K1_DIRECT: return K1Variant::Direct;
        case SOMIER_K1_MARCH: return K1Variant::March;
        case SOMIER_K1_MARCH2: return K1Variant::March2;
        case SOMIER_K1_TB2: return K1Variant::March2;  // TB2 impossible (a chunk of one plane among several)
        default: return K1Variant::March2;  // measured fastest at 512^3
    }
}

// Row pitch (doubles) of a slab for rows of n2 nodes: 256-byte aligned rows.
inline int64_t slab_ld(int64_t n2) { return (n2 + 31) / 32 * 32; }

}  // namespace paper
