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

// f1 (reading R17): viscous hourglass corner forces, Flanagan-Belytschko form,
// added to P B_l.  Hourglass base vectors h_a,l in {-1, +1} (a = 0..3: eta zeta, zeta xi, xi eta,
// xi eta zeta with xi = +-1 by corner bit a, ...).  The projection uses C = H M^-1 with
// M_dk = sum_l B_l,d X_l,k and H_ak = sum_l h_a,l X_l,k, so gamma_a = h_a - C_a . B is orthogonal
// to every linear field on any hex; g_a = sum_l gamma_a,l u_l (u^n); the corner force is
// f_l = -kappa rho c V^(2/3) sum_a gamma_a,l g_a.  Adds into F (x, y, z per corner).
__device__ __forceinline__ double hg_sign(int a, int l) {
  const double xi = (l & 1) ? 1.0 : -1.0, eta = (l & 2) ? 1.0 : -1.0, zeta = (l & 4) ? 1.0 : -1.0;
  return a == 0 ? eta * zeta : a == 1 ? zeta * xi : a == 2 ? xi * eta : xi * eta * zeta;
}
__device__ __forceinline__ void hourglass_add(const double X[8], const double Y[8],
                                              const double Z[8], const double U[8],
                                              const double Vv[8], const double W[8],
                                              const double Bx[8], const double By[8],
                                              const double Bz[8], double V, double rho, double c,
                                              double kappa, double Fx[8], double Fy[8],
                                              double Fz[8]) {
  const double *P3[3] = {X, Y, Z};
  const double *B3[3] = {Bx, By, Bz};
  double M[3][3], H[4][3];
#pragma unroll
  for (int d = 0; d < 3; ++d)
#pragma unroll
    for (int k = 0; k < 3; ++k) {
      double s = 0.0;
#pragma unroll
      for (int l = 0; l < 8; ++l) s = fma(B3[d][l], P3[k][l], s);
      M[d][k] = s;
    }
#pragma unroll
  for (int a = 0; a < 4; ++a)
#pragma unroll
    for (int k = 0; k < 3; ++k) {
      double s = 0.0;
#pragma unroll
      for (int l = 0; l < 8; ++l) s += hg_sign(a, l) * P3[k][l];
      H[a][k] = s;
    }
  // adjugate inverse: (M^-1)_kd = adj(M)_kd / det = cof(M)_dk / det
  double cf[3][3];
#pragma unroll
  for (int r = 0; r < 3; ++r)
#pragma unroll
    for (int q = 0; q < 3; ++q)
      cf[r][q] = M[(r + 1) % 3][(q + 1) % 3] * M[(r + 2) % 3][(q + 2) % 3] -
                 M[(r + 1) % 3][(q + 2) % 3] * M[(r + 2) % 3][(q + 1) % 3];
  const double idet = 1.0 / (M[0][0] * cf[0][0] + M[0][1] * cf[0][1] + M[0][2] * cf[0][2]);
  double C[4][3];
#pragma unroll
  for (int a = 0; a < 4; ++a)
#pragma unroll
    for (int d = 0; d < 3; ++d)
      C[a][d] = (H[a][0] * cf[d][0] + H[a][1] * cf[d][1] + H[a][2] * cf[d][2]) * idet;
  double gam[4][8], g[4][3];
#pragma unroll
  for (int a = 0; a < 4; ++a) {
    double gx = 0.0, gy = 0.0, gz = 0.0;
#pragma unroll
    for (int l = 0; l < 8; ++l) {
      gam[a][l] = hg_sign(a, l) - (C[a][0] * Bx[l] + C[a][1] * By[l] + C[a][2] * Bz[l]);
      gx = fma(gam[a][l], U[l], gx);
      gy = fma(gam[a][l], Vv[l], gy);
      gz = fma(gam[a][l], W[l], gz);
    }
    g[a][0] = gx; g[a][1] = gy; g[a][2] = gz;
  }
  const double v13 = cbrt(V);
  const double coef = -kappa * rho * c * v13 * v13;
#pragma unroll
  for (int l = 0; l < 8; ++l) {
    double sx = 0.0, sy = 0.0, sz = 0.0;
#pragma unroll
    for (int a = 0; a < 4; ++a) {
      sx = fma(gam[a][l], g[a][0], sx);
      sy = fma(gam[a][l], g[a][1], sy);
      sz = fma(gam[a][l], g[a][2], sz);
    }
    Fx[l] = fma(coef, sx, Fx[l]);
    Fy[l] = fma(coef, sy, Fy[l]);
    Fz[l] = fma(coef, sz, Fz[l]);
  }
}

struct ZoneEos {
  double rho, p, c, q, P, dtz;
};

// f1 / reading R24 (monotone q): strain rate eps_d = (du_d . dx_d)/|dx_d|^2 and length
// L_d = |dx_d| of a zone along each logical direction d, from the face-centre differences dx_d,
// du_d (corners with bit d set minus those without, / 4).
__device__ __forceinline__ void zone_strain(const double X[8], const double Y[8],
                                            const double Z[8], const double U[8],
                                            const double Vv[8], const double W[8],
                                            double eps[3], double L[3]) {
#pragma unroll
  for (int dd = 0; dd < 3; ++dd) {
    double dx = 0.0, dy = 0.0, dz = 0.0, du = 0.0, dv = 0.0, dw = 0.0;
#pragma unroll
    for (int l = 0; l < 8; ++l) {
      const double sg = ((l >> dd) & 1) ? 0.25 : -0.25;
      dx = fma(sg, X[l], dx); dy = fma(sg, Y[l], dy); dz = fma(sg, Z[l], dz);
      du = fma(sg, U[l], du); dv = fma(sg, Vv[l], dv); dw = fma(sg, W[l], dw);
    }
    const double L2 = dx * dx + dy * dy + dz * dz;
    eps[dd] = (du * dx + dv * dy + dw * dz) / L2;
    L[dd] = sqrt(L2);
  }
}

// Reading R24: phi = max(0, min((r- + r+)/2, 2 r-, 2 r+, 1)), r = neighbour / own strain rate.
__device__ __forceinline__ double mono_limiter(double em, double e0, double ep) {
  if (e0 == 0.0) return 1.0;
  const double rm = em / e0, rp = ep / e0;
  double phi = 0.5 * (rm + rp);
  phi = (2.0 * rm < phi) ? 2.0 * rm : phi;
  phi = (2.0 * rp < phi) ? 2.0 * rp : phi;
  phi = (1.0 < phi) ? 1.0 : phi;
  return (phi < 0.0) ? 0.0 : phi;
}

// Strain rate eps_d of global zone (g0, g1, g2), read from its owner domain on this GPU: the
// calling domain `self` itself when it owns the zone (one load), else through the owner tables.
__device__ __forceinline__ double mono_eps(const MonoMap &M, const DomView &self, int64_t g0,
                                           int64_t g1, int64_t g2, int dd) {
  const int64_t l0 = g0 - self.lo[0], l1 = g1 - self.lo[1], l2 = g2 - self.lo[2];
  if (l0 >= 0 && l0 < self.n[0] && l1 >= 0 && l1 < self.n[1] && l2 >= 0 && l2 < self.n[2])
    return self.eps[(int64_t)dd * self.nzone + self.zid((int)l0, (int)l1, (int)l2)];
  const int dom = (M.zown[2][g2] * M.ndy + M.zown[1][g1]) * M.ndx + M.zown[0][g0];
  const DomView &v = M.views[M.slot[dom]];
  const int64_t id = v.zid((int)(g0 - v.lo[0]), (int)(g1 - v.lo[1]), (int)(g2 - v.lo[2]));
  return v.eps[(int64_t)dd * v.nzone + id];
}

// Reading R24: the three limiter values of global zone g (a neighbour outside the mesh mirrors
// the zone at a reflecting wall and is unstrained at a free boundary).
__device__ __forceinline__ void mono_phi(const MonoMap &M, const DomView &self,
                                         const int64_t g[3], uint32_t reflect_mask,
                                         double phi[3]) {
#pragma unroll
  for (int dd = 0; dd < 3; ++dd) {
    const double e0 = mono_eps(M, self, g[0], g[1], g[2], dd);
    int64_t gm[3] = {g[0], g[1], g[2]}, gp[3] = {g[0], g[1], g[2]};
    gm[dd] -= 1;
    gp[dd] += 1;
    const double em = gm[dd] >= 0 ? mono_eps(M, self, gm[0], gm[1], gm[2], dd)
                      : ((reflect_mask >> (2 * dd)) & 1u) ? e0 : 0.0;
    const double ep = gp[dd] < self.N[dd] ? mono_eps(M, self, gp[0], gp[1], gp[2], dd)
                      : ((reflect_mask >> (2 * dd + 1)) & 1u) ? e0 : 0.0;
    phi[dd] = mono_limiter(em, e0, ep);
  }
}

// S2 (rho, D) + S3 + S4 + S6 given V, L = 2V/sqrt(A2max_unscaled), DV = sum u.B.  phi / epsL
// (monotone q, R24): the zone's limiter values and its own strain rates eps[3] and lengths
// epsL[3..5]; nullptr = the scalar q of R7.
__device__ __forceinline__ ZoneEos zone_eos(double V, double A2max, double DV, double m,
                                            double e, double hh, const Phys &ph,
                                            const double *phi = nullptr,
                                            const double *epsL = nullptr) {
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
  if (D < 0.0 && !phi) {
    const double s = -L * D;
    qr = s * (ph.q_quad * s + ph.q_lin * c);
  } else if (D < 0.0) {
#pragma unroll
    for (int dd = 0; dd < 3; ++dd) {
      const double dv = epsL[3 + dd] * fmax(-epsL[dd], 0.0);
      qr += (ph.q_quad * dv) * dv * (1.0 - phi[dd] * phi[dd]) + (ph.q_lin * c) * dv * (1.0 - phi[dd]);
    }
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
