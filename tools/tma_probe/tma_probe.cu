// TMA probe: which fp64 tensor-map configurations does UTMALDG accept on this B200?
// Usage: tma_probe <variant>; prints OK or the CUDA error. One variant per process.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdlib>
#include <cstring>

using PFN_encodeTiled = CUresult (*)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                     const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                     CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int R>
__global__ void probe(const __grid_constant__ CUtensorMap map, int c0, int c1, int c2, int c3, unsigned bytes, double* out) {
  extern __shared__ __align__(128) unsigned char smem[];
  __shared__ __align__(8) unsigned long long bar;
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(smem_u32(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;");
    asm volatile("fence.proxy.async.shared::cta;");
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(smem_u32(&bar)), "r"(bytes));
    if (R == 4)
      asm volatile("cp.async.bulk.tensor.4d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5}], [%6];"
        :: "r"(smem_u32(smem)), "l"((uint64_t)&map), "r"(c0), "r"(c1), "r"(c2), "r"(c3), "r"(smem_u32(&bar)) : "memory");
    else
      asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
        :: "r"(smem_u32(smem)), "l"((uint64_t)&map), "r"(c0), "r"(c1), "r"(smem_u32(&bar)) : "memory");
    asm volatile("{\n.reg .pred p;\nW%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n@!p bra W%=;\n}" :: "r"(smem_u32(&bar)));
    out[0] = ((double*)smem)[0];
    out[1] = ((double*)smem)[1];
  }
}

int main(int argc, char** argv) {
  int v = argc > 1 ? atoi(argv[1]) : 0;
  void* fn; cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q);
  PFN_encodeTiled enc = (PFN_encodeTiled)fn;
  int n2 = 16, n1 = 16, ld = 32, planes = 16;
  double* g; cudaMalloc(&g, (size_t)ld * n1 * 3 * planes * 8 + 4096);
  cudaMemset(g, 0, (size_t)ld * n1 * 3 * planes * 8);
  double* out; cudaMalloc(&out, 64);
  CUtensorMap map; memset(&map, 0, sizeof map);
  cuuint64_t dims4[4] = {(cuuint64_t)n2, (cuuint64_t)n1, 3, (cuuint64_t)planes};
  cuuint64_t str4[3] = {(cuuint64_t)ld * 8, (cuuint64_t)ld * n1 * 8, (cuuint64_t)ld * n1 * 3 * 8};
  cuuint32_t es[4] = {1, 1, 1, 1};
  CUtensorMapDataType dt = (v == 5) ? CU_TENSOR_MAP_DATA_TYPE_UINT64 : CU_TENSOR_MAP_DATA_TYPE_FLOAT64;
  CUresult r; unsigned bytes; int rank = 4; int c[4] = {0, 0, 0, 1};
  cuuint32_t box[4] = {34, 10, 3, 1};
  if (v == 0 || v == 5) { c[0] = -1; c[1] = -1; }
  if (v == 2 || v == 6) { box[0] = 32; box[1] = 8; }
  if (v == 6) { box[0] = 16; box[1] = 8; }
  if (v == 7) { box[0] = 34; box[1] = 10; box[2] = 1; }
  if (v == 8) { dims4[0] = 64; box[0] = 34; c[0] = -1; }
  if (v == 9) { dims4[0] = 64; c[0] = 1; }
  if (v == 10) { dims4[0] = 64; c[0] = 2; }
  if (v == 11) { dims4[0] = 64; c[1] = -1; }
  if (v == 12) { dims4[0] = 64; c[0] = -2; }
  if (v == 13) { dims4[0] = 64; c[0] = 31; }
  bytes = box[0] * box[1] * box[2] * box[3] * 8;
  if (v == 3) {
    rank = 2; cuuint64_t d2[2] = {(cuuint64_t)n2, (cuuint64_t)n1 * 3 * planes}; cuuint64_t s2[1] = {(cuuint64_t)ld * 8};
    cuuint32_t b2[2] = {16, 8};
    r = enc(&map, dt, 2, g, d2, s2, b2, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    bytes = 16 * 8 * 8;
  } else {
    r = enc(&map, dt, 4, g, dims4, str4, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
            v == 4 ? CU_TENSOR_MAP_L2_PROMOTION_NONE : CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  }
  printf("variant %d encode=%d box=(%u,%u,%u,%u) bytes=%u ", v, (int)r, box[0], box[1], box[2], box[3], bytes);
  if (rank == 4) probe<4><<<1, 32, 16384>>>(map, c[0], c[1], c[2], c[3], bytes, out);
  else probe<2><<<1, 32, 16384>>>(map, 0, 0, 0, 0, bytes, out);
  cudaError_t e = cudaDeviceSynchronize();
  printf("-> %s\n", cudaGetErrorString(e));
  return 0;
}
