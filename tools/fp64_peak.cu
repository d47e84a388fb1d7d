// Microbenchmark: sustained fp64 DFMA lane-op throughput on the device (the "alu" roofline
// denominator for the fp64 hydro cycle).  8 independent FMA chains per
// thread so the FP64 pipe, not latency, is the limit.
#include <cstdio>
#include <cuda_runtime.h>
__global__ void dfma_loop(double* out, int iters, double a, double b) {
  double r0 = threadIdx.x * 1e-9, r1 = r0 + 1, r2 = r0 + 2, r3 = r0 + 3, r4 = r0 + 4, r5 = r0 + 5,
         r6 = r0 + 6, r7 = r0 + 7;
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      r0 = fma(r0, a, b); r1 = fma(r1, a, b); r2 = fma(r2, a, b); r3 = fma(r3, a, b);
      r4 = fma(r4, a, b); r5 = fma(r5, a, b); r6 = fma(r6, a, b); r7 = fma(r7, a, b);
    }
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = r0 + r1 + r2 + r3 + r4 + r5 + r6 + r7;
}
int main() {
  int dev = 0; cudaDeviceProp p; cudaGetDeviceProperties(&p, dev);
  int sms = p.multiProcessorCount;
  double* out; cudaMalloc(&out, sizeof(double) * sms * 8 * 1024);
  int iters = 4096;
  for (int bpsm : {2, 4, 8}) {
    int blocks = sms * bpsm, threads = 256;
    dfma_loop<<<blocks, threads>>>(out, 16, 0.999999, 1e-7);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    float best = 1e30f;
    for (int rep = 0; rep < 5; ++rep) {
      cudaEventRecord(e0);
      dfma_loop<<<blocks, threads>>>(out, iters, 0.999999, 1e-7);
      cudaEventRecord(e1); cudaEventSynchronize(e1);
      float ms; cudaEventElapsedTime(&ms, e0, e1); if (ms < best) best = ms;
    }
    double lane_ops = (double)blocks * threads * iters * 64.0;
    printf("{\"blocks_per_sm\": %d, \"ms\": %.4f, \"dfma_lane_ops_per_s\": %.4e, \"fp64_tflops\": %.3f, \"sms\": %d}\n",
           bpsm, best, lane_ops / (best * 1e-3), 2 * lane_ops / (best * 1e-3) / 1e12, sms);
  }
  return 0;
}
