// zone_physics.cuh -- per-zone physics of the cycle as device functions (SURVEY §8c.2-8c.3,
// DESIGN.md §3): S2 geometry, S3 EOS with the energy predictor, S4 artificial viscosity,
// S6 zone dt.  Written independently of oracle/ (which it must match within the north_star
// tolerance, not bitwise): face vectors are kept unscaled (2A) and the factor 1/2 is folded into
// the corner-vector weight 1/8, and FMA contraction is allowed.
#pragma once
#include <cmath>

#include "device.cuh"

namespace hydro {

// Unscaled face vector 2A = d1 x d2.
__device__ __forceinline__ void cross3(double ax, double ay, double az, double bx, double by,
                                       double bz, double &cx, double &cy, double &cz) {
  cx = ay * bz - az * by;
  cy = az * bx - ax * bz;
  cz = ax * by - ay * bx;
}

// Face vector (unscaled) of the quad p0,p1,p2,p3 given as d1 = p_diag1 - p_a, d2 = p_diag2 - p_b.
#define HYDRO_FACE(X, Y, Z, i1, i0, j1, j0, ox, oy, oz)                                     \
  cross3(X[i1] - X[i0], Y[i1] - Y[i0], Z[i1] - Z[i0], X[j1] - X[j0], Y[j1] - Y[j0],           \
         Z[j1] - Z[j0], ox, oy, oz)

// S2: corner vectors B_l (8 x 3), volume V and max squared (unscaled) face area of one hex.
__device__ __forceinline__ void hex_geometry(const double X[8], const double Y[8],
                                             const double Z[8], double Bx[8], double By[8],
                                             double Bz[8], double &V, double &A2max) {
  double fx[6], fy[6], fz[6];  // faces: AX0, AX1, AY0, AY1, AZ0, AZ1 (unscaled)
#pragma unroll
  for (int a = 0; a < 2; ++a) HYDRO_FACE(X, Y, Z, a + 6, a, a + 4, a + 2, fx[a], fy[a], fz[a]);
#pragma unroll
  for (int b = 0; b < 2; ++b)
    HYDRO_FACE(X, Y, Z, 5 + 2 * b, 2 * b, 1 + 2 * b, 2 * b + 4, fx[2 + b], fy[2 + b], fz[2 + b]);
#pragma unroll
  for (int c = 0; c < 2; ++c)
    HYDRO_FACE(X, Y, Z, 3 + 4 * c, 4 * c, 2 + 4 * c, 1 + 4 * c, fx[4 + c], fy[4 + c], fz[4 + c]);
#pragma unroll
  for (int l = 0; l < 8; ++l) {
    const int a = l & 1, b = (l >> 1) & 1, c = (l >> 2) & 1;
    const double sx = (a ? fx[1] : -fx[0]) + (b ? fx[3] : -fx[2]) + (c ? fx[5] : -fx[4]);
    const double sy = (a ? fy[1] : -fy[0]) + (b ? fy[3] : -fy[2]) + (c ? fy[5] : -fy[4]);
    const double sz = (a ? fz[1] : -fz[0]) + (b ? fz[3] : -fz[2]) + (c ? fz[5] : -fz[4]);
    Bx[l] = 0.125 * sx;
    By[l] = 0.125 * sy;
    Bz[l] = 0.125 * sz;
  }
  double s = 0.0;
#pragma unroll
  for (int l = 1; l < 8; ++l)
    s += (X[l] - X[0]) * Bx[l] + (Y[l] - Y[0]) * By[l] + (Z[l] - Z[0]) * Bz[l];
  V = s * (1.0 / 3.0);
  double a2 = 0.0;
#pragma unroll
  for (int f = 0; f < 6; ++f) a2 = fmax(a2, fx[f] * fx[f] + fy[f] * fy[f] + fz[f] * fz[f]);
  A2max = a2;
}

struct ZoneEos {
  double rho, p, c, q, P, dtz;
};

// S2 (rho, D) + S3 + S4 + S6 given V, L = 2V/sqrt(A2max_unscaled), DV = sum u.B.
__device__ __forceinline__ ZoneEos zone_eos(double V, double A2max, double DV, double m,
                                            double e, double hh, const Phys &ph) {
  ZoneEos r;
  const double L = 2.0 * V / sqrt(A2max);
  const double inv = 1.0 / V;
  const double rho = m * inv;
  const double D = DV * inv;
  const double epos = fmax(e, 0.0);
  const double ep = e - (hh * (ph.gm1 * rho) * epos) * DV / m;
  const double eppos = fmax(ep, 0.0);
  const double p = ph.gm1 * rho * eppos;
  const double c = sqrt(ph.ggm1 * eppos);
  double qr = 0.0;
  if (D < 0.0) {
    const double s = -L * D;
    qr = s * (ph.q_quad * s + ph.q_lin * c);
  }
  r.rho = rho;
  r.p = p;
  r.c = c;
  r.q = rho * qr;
  r.P = p + r.q;
  const double sig = sqrt(c * c + 2.0 * qr);
  const double dtc = (sig > 0.0) ? ph.cfl * L / sig : INFINITY;
  const double dtv = (D != 0.0) ? ph.c_vol / fabs(D) : INFINITY;
  r.dtz = fmin(dtc, dtv);
  return r;
}

// Warp + block min of a non-negative double, one atomicMin on its bit pattern per block;
// red: 32 doubles of shared scratch.
__device__ __forceinline__ void block_min_dt_smem(double v, unsigned long long *acc, double *red) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fmin(v, __shfl_xor_sync(0xffffffffu, v, o));
  const int tid = threadIdx.x + blockDim.x * (threadIdx.y + blockDim.y * threadIdx.z);
  const int nthr = blockDim.x * blockDim.y * blockDim.z;
  const int lane = tid & 31, warp = tid >> 5;
  if (lane == 0) red[warp] = v;
  __syncthreads();
  if (warp == 0) {
    v = (lane < (nthr + 31) / 32) ? red[lane] : INFINITY;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v = fmin(v, __shfl_xor_sync(0xffffffffu, v, o));
    if (lane == 0 && v < INFINITY) atomicMin(acc, (unsigned long long)__double_as_longlong(v));
  }
}

__device__ __forceinline__ void block_min_dt(double v, unsigned long long *acc) {
  __shared__ double red[32];
  block_min_dt_smem(v, acc, red);
}

}  // namespace hydro
