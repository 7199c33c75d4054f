// Microbenchmark: fp64 pipe throughput on B200 (DFMA, DADD, DMUL, sqrt_rn, div_rn),
// plus a streaming copy of doubles. Informs DESIGN.md's ALU roofline for K1.
#include <cstdio>
#include <cuda_runtime.h>
#define CK(x) do{cudaError_t e=(x); if(e!=cudaSuccess){printf("err %s line %d\n",cudaGetErrorString(e),__LINE__);return 1;}}while(0)

__global__ void dfma_k(double* out, int iters, double a, double b) {
  double x0 = threadIdx.x * 1e-3, x1 = x0 + 1, x2 = x0 + 2, x3 = x0 + 3, x4=x0+4,x5=x0+5,x6=x0+6,x7=x0+7;
  for (int i = 0; i < iters; i++) {
#pragma unroll
    for (int u = 0; u < 16; u++) {
      x0 = __fma_rn(x0, a, b); x1 = __fma_rn(x1, a, b); x2 = __fma_rn(x2, a, b); x3 = __fma_rn(x3, a, b);
      x4 = __fma_rn(x4, a, b); x5 = __fma_rn(x5, a, b); x6 = __fma_rn(x6, a, b); x7 = __fma_rn(x7, a, b);
    }
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = x0+x1+x2+x3+x4+x5+x6+x7;
}
// DADD / DMUL chains (same issue pattern as dfma_k): is every fp64 opcode one pipe slot?
template <int kOp>
__global__ void dop_k(double* out, int iters, double a) {
  double x0 = threadIdx.x * 1e-3, x1 = x0 + 1, x2 = x0 + 2, x3 = x0 + 3, x4=x0+4,x5=x0+5,x6=x0+6,x7=x0+7;
  for (int i = 0; i < iters; i++) {
#pragma unroll
    for (int u = 0; u < 16; u++) {
      if (kOp == 0) {
        x0 = __dadd_rn(x0, a); x1 = __dadd_rn(x1, a); x2 = __dadd_rn(x2, a); x3 = __dadd_rn(x3, a);
        x4 = __dadd_rn(x4, a); x5 = __dadd_rn(x5, a); x6 = __dadd_rn(x6, a); x7 = __dadd_rn(x7, a);
      } else {
        x0 = __dmul_rn(x0, a); x1 = __dmul_rn(x1, a); x2 = __dmul_rn(x2, a); x3 = __dmul_rn(x3, a);
        x4 = __dmul_rn(x4, a); x5 = __dmul_rn(x5, a); x6 = __dmul_rn(x6, a); x7 = __dmul_rn(x7, a);
      }
    }
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = x0+x1+x2+x3+x4+x5+x6+x7;
}
__global__ void dsqrtdiv_k(double* out, int iters, double a) {
  double x0 = 1.0 + threadIdx.x * 1e-3, x1 = x0 + 1, x2 = x0 + 2, x3 = x0 + 3;
  for (int i = 0; i < iters; i++) {
#pragma unroll
    for (int u = 0; u < 4; u++) {
      x0 = __ddiv_rn(a, __dsqrt_rn(x0)) + 1.0; x1 = __ddiv_rn(a, __dsqrt_rn(x1)) + 1.0;
      x2 = __ddiv_rn(a, __dsqrt_rn(x2)) + 1.0; x3 = __ddiv_rn(a, __dsqrt_rn(x3)) + 1.0;
    }
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = x0+x1+x2+x3;
}
__global__ void copy_k(const double2* __restrict__ a, double2* __restrict__ b, size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) b[i] = a[i];
}
int main() {
  cudaDeviceProp p; CK(cudaGetDeviceProperties(&p, 0));
  printf("device %s SMs %d cc %d.%d clock(kHz) %d l2 %d MB smemPerBlockOptin %zu\n", p.name, p.multiProcessorCount, p.major, p.minor, p.clockRate, p.l2CacheSize>>20, p.sharedMemPerBlockOptin);
  double* out; CK(cudaMalloc(&out, 148*64*1024*sizeof(double)));
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  int blocks = p.multiProcessorCount * 8, threads = 256, iters = 2000;
  double best[3] = {0, 0, 0};  // DFMA, DADD, DMUL lane-instructions/s
  for (int rep = 0; rep < 3; rep++) {
    cudaEventRecord(e0); dfma_k<<<blocks, threads>>>(out, iters, 0.999999, 1e-7); cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    double ops = (double)blocks * threads * iters * 16 * 8;
    printf("DFMA: %.3f ms, %.3f Tinstr/s (%.2f per SM per clk @1965)\n", ms, ops / ms / 1e9, ops / (ms*1e-3) / 148 / 1.965e9);
    if (ops / ms / 1e9 > best[0]) best[0] = ops / ms / 1e9;
  }
  for (int op = 0; op < 2; op++)
  for (int rep = 0; rep < 3; rep++) {
    cudaEventRecord(e0);
    if (op == 0) dop_k<0><<<blocks, threads>>>(out, iters, 1e-9); else dop_k<1><<<blocks, threads>>>(out, iters, 0.9999999);
    cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    double ops = (double)blocks * threads * iters * 16 * 8;
    printf("%s: %.3f ms, %.3f Tinstr/s (%.2f per SM per clk @1965)\n", op ? "DMUL" : "DADD", ms, ops / ms / 1e9, ops / (ms*1e-3) / 148 / 1.965e9);
    if (ops / ms / 1e9 > best[1 + op]) best[1 + op] = ops / ms / 1e9;
  }
  iters = 500;
  for (int rep = 0; rep < 3; rep++) {
    cudaEventRecord(e0); dsqrtdiv_k<<<blocks, threads>>>(out, iters, 3.0); cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    double ops = (double)blocks * threads * iters * 4 * 4;
    printf("sqrt+div+add: %.3f ms, %.3f G(sqrt+div)/s, %.1f ns-per-pair/SM-ish\n", ms, ops / ms / 1e6, 0.0);
  }
  size_t n = (size_t)1 << 28; double2 *a, *b; CK(cudaMalloc(&a, n * 16)); CK(cudaMalloc(&b, n * 16));
  cudaMemset(a, 0, n*16);
  for (int rep = 0; rep < 5; rep++) {
    cudaEventRecord(e0); copy_k<<<p.multiProcessorCount * 16, 256>>>(a, b, n); cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    printf("copy: %.3f ms %.1f GB/s\n", ms, 2.0 * n * 16 / ms / 1e6);
  }
  const double peak = best[0] > best[1] ? (best[0] > best[2] ? best[0] : best[2]) : (best[1] > best[2] ? best[1] : best[2]);
  printf("{\"fp64_tinstr_s\": %.4f, \"dfma_tinstr_s\": %.4f, \"dadd_tinstr_s\": %.4f, \"dmul_tinstr_s\": %.4f, "
         "\"how\": \"tools/microbench/fp64_rate: 8 independent chains per thread, 1184 x 256 threads, best of 3 per opcode; "
         "peak = the fastest opcode\"}\n", peak, best[0], best[1], best[2]);
  return 0;
}
