// Accuracy of the SFU seeds behind frcp / frsqrt (csrc/fastmath.cuh) and of 1..3 Newton steps,
// against correctly rounded 1/x and 1/sqrt(x) (IEEE div / sqrt), over log-uniform x.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/fastmath_acc tools/fastmath_acc.cu
#include <cstdio>
#include <cmath>
#include <cstdint>
#include <cstring>

__device__ unsigned long long g_max[8];  // rel-error bits (non-negative doubles order as uint64)

__device__ __forceinline__ uint64_t mix(uint64_t z) {
  z += 0x9e3779b97f4a7c15ull;
  z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ull;
  z = (z ^ (z >> 27)) * 0x94d049bb133111ebull;
  return z ^ (z >> 31);
}

__device__ void upd(int k, double e) {
  atomicMax(&g_max[k], (unsigned long long)__double_as_longlong(fabs(e)));
}

__global__ void k_acc(long n) {
  for (long i = blockIdx.x * (long)blockDim.x + threadIdx.x; i < n; i += (long)gridDim.x * blockDim.x) {
    const uint64_t r = mix((uint64_t)i);
    const double u = (double)(r >> 11) * 0x1p-53;
    const double x = exp2(-1000.0 + 2000.0 * u);  // 2^-1000 .. 2^1000
    const double ref = 1.0 / x;
    double s;
    asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(s) : "d"(x));
    upd(0, (s - ref) / ref);
    double rr = s;
    for (int k = 1; k <= 3; ++k) {
      const double e = fma(-x, rr, 1.0);
      rr = fma(rr, e, rr);
      upd(k, (rr - ref) / ref);
    }
    const double rs = 1.0 / sqrt(x);
    double y;
    asm("rsqrt.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(x));
    upd(4, (y - rs) / rs);
    const double h = 0.5 * x;
    for (int k = 1; k <= 3; ++k) {
      y = y * fma(-h * y, y, 1.5);
      upd(4 + k, (y - rs) / rs);
    }
  }
}

int main() {
  unsigned long long z[8] = {};
  cudaMemcpyToSymbol(g_max, z, sizeof(z));
  k_acc<<<148 * 8, 256>>>(1L << 28);
  cudaMemcpyFromSymbol(z, g_max, sizeof(z));
  const char *name[8] = {"rcp seed", "rcp 1 step", "rcp 2 steps", "rcp 3 steps",
                         "rsqrt seed", "rsqrt 1 step", "rsqrt 2 steps", "rsqrt 3 steps"};
  for (int k = 0; k < 8; ++k) {
    double e;
    memcpy(&e, &z[k], 8);
    printf("%-14s max rel err %.3e  (2^%.1f)\n", name[k], e, e > 0 ? log2(e) : -1e9);
  }
  return 0;
}
