// shfl_vs_lds.cu -- does a warp shuffle consume the shared-memory (LSU) wavefront bandwidth on
// B200?  The node/energy stage is bound by shared-memory wavefronts; if SHFL runs on
// a separate path, x-neighbour values could move lane to lane instead of through shared memory.
//
// One 512-thread CTA per SM, each thread runs ITERS trips of
//   mode 0: 8 independent LDS.64 (consecutive words across the warp: 2 wavefronts each)
//   mode 1: 8 independent 64-bit shuffles (2 SHFL.32 each)
//   mode 2: both (8 LDS.64 + 8 shuffles per trip)
// and the kernel time gives warp-instructions per SM per clock.  If mode 2 takes about
// max(mode 0, mode 1), the shuffles do not compete with the loads for the same pipe; if it takes
// the sum, they do.
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/shfl_vs_lds tools/shfl_vs_lds.cu
#include <cstdio>
#include <cuda_runtime.h>

constexpr int NT = 512, ITERS = 4096, SMW = 4096;

template <int MODE>
__global__ void __launch_bounds__(NT, 1) k(double *out, int salt) {
  __shared__ double s[SMW];
  for (int i = threadIdx.x; i < SMW; i += NT) s[i] = i * 0.5 + salt;
  __syncthreads();
  double a[8];
#pragma unroll
  for (int r = 0; r < 8; ++r) a[r] = threadIdx.x + r;
  int idx = threadIdx.x;
  for (int it = 0; it < ITERS; ++it) {
    if (MODE != 1) {
#pragma unroll
      for (int r = 0; r < 8; ++r) a[r] += s[(idx + r * 256) & (SMW - 1)];
    }
    if (MODE != 0) {
#pragma unroll
      for (int r = 0; r < 8; ++r) a[r] += __shfl_xor_sync(0xffffffffu, a[r], 1 + (r & 3));
    }
    idx = (idx + 32) & (SMW - 1);
  }
  double t = 0;
#pragma unroll
  for (int r = 0; r < 8; ++r) t += a[r];
  if (t == 12345.678) out[0] = t;  // keep the work
}

template <int MODE>
float run(int nsm, double *out) {
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  k<MODE><<<nsm, NT>>>(out, 1);
  cudaEventRecord(e0);
  for (int r = 0; r < 5; ++r) k<MODE><<<nsm, NT>>>(out, r);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms;
  cudaEventElapsedTime(&ms, e0, e1);
  return ms / 5;
}

int main() {
  int dev = 0, nsm, clk;
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, dev);  // kHz
  double *out;
  cudaMalloc(&out, 8);
  const float t0 = run<0>(nsm, out), t1 = run<1>(nsm, out), t2 = run<2>(nsm, out);
  const double warps = NT / 32.0 * ITERS;  // per SM
  const double cyc = clk * 1e3;
  auto rate = [&](float ms, double inst) { return inst * warps / (ms * 1e-3 * cyc); };
  printf("SMs %d, clock %.0f MHz (nominal)\n", nsm, clk / 1e3);
  printf("mode 0 (8 LDS.64/trip):          %.3f ms  %.3f LDS.64 warp-inst/SM/clk\n", t0,
         rate(t0, 8));
  printf("mode 1 (8 shfl64/trip):          %.3f ms  %.3f shfl64 warp-inst/SM/clk\n", t1,
         rate(t1, 8));
  printf("mode 2 (8 LDS.64 + 8 shfl64):    %.3f ms  (sum of 0+1 = %.3f ms, max = %.3f ms)\n", t2,
         t0 + t1, t0 > t1 ? t0 : t1);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) { printf("CUDA error %s\n", cudaGetErrorString(e)); return 1; }
  return 0;
}
