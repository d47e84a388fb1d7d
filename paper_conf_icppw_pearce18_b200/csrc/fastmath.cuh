// fastmath.cuh -- branch-free fp64 reciprocal / sqrt for the fused kernel.
//
// CUDA's IEEE fp64 division and sqrt carry a slow path (a call plus a reconvergence branch per
// use); the fused kernel needs six of them per zone.  Here: the SFU seed (MUFU.RCP64H /
// MUFU.RSQ64H) refined by Newton steps in DFMA.  Measured on B200 (tools/fastmath_acc.cu,
// profiles/r01_fastmath_acc.txt, 2^28 log-uniform inputs over 2^-1000..2^1000): the seeds are
// good to 2^-20, so two steps suffice -- rcp then matches IEEE 1/x exactly on every sample,
// rsqrt is within 4e-16 relative -- which the north_star tolerance (1e-12) absorbs (reading R12).
#pragma once

namespace hydro {

__device__ __forceinline__ double frcp(double x) {  // 1/x for finite non-zero x
  double r;
  asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(x));
  double e = fma(-x, r, 1.0);
  r = fma(r, e, r);
  e = fma(-x, r, 1.0);
  return fma(r, e, r);
}

__device__ __forceinline__ double frsqrt(double x) {  // 1/sqrt(x) for finite x > 0
  double y;
  asm("rsqrt.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(x));
  const double h = 0.5 * x;
  y = y * fma(-h * y, y, 1.5);
  return y * fma(-h * y, y, 1.5);
}

__device__ __forceinline__ double fsqrt(double x) {  // sqrt(x) for finite x >= 0
  // subnormal inputs (e.g. a nearly cold zone's e) are scaled by 2^108 so the flush-to-zero SFU
  // seed stays valid; the result is scaled back by 2^-54
  const bool tiny = x < 2.2250738585072014e-308;
  const double xs = tiny ? x * 0x1p108 : x;
  const double y = frsqrt(xs);
  const double s = xs * y;
  const double r = fma(-s, s, xs);
  const double out = fma(r, 0.5 * y, s) * (tiny ? 0x1p-54 : 1.0);
  return x > 0.0 ? out : 0.0;
}

}  // namespace hydro
