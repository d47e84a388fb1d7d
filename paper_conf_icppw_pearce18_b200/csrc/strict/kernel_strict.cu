// kernel_strict.cu -- HYDRO_FLAG_STRICT: the cycle S1-S8 in the canonical operation order of
// SURVEY.md §8c.2-8c.3 (reading R13), one thread per element, compiled on its own with
// -fmad=false (reading R12: no contraction; fp64 '/' and sqrt are IEEE correctly rounded), so
// that every zone and node value is the unique IEEE result of the written order.  The oracle
// (oracle/, -O2 -ffp-contract=off) evaluates the same written order, so this path is BITWISE
// equal to it (tests/test_gpu_strict.py), which turns the tolerance
// argument of the fast paths into a proof for one path.  Nothing here is shared with oracle/:
// both sides restate the definitions of §8c.
//
// Canonical orders used (each sum's first term initialises it, no 0 + x):
//   faces   AX_a = 0.5 (X[a+6]-X[a]) x (X[a+4]-X[a+2]); AY_b = 0.5 (X[5+2b]-X[2b]) x
//           (X[1+2b]-X[2b+4]); AZ_c = 0.5 (X[3+4c]-X[4c]) x (X[2+4c]-X[1+4c]),
//           cross (a1 b2 - a2 b1, a2 b0 - a0 b2, a0 b1 - a1 b0);
//   corner  B_l = 0.25 ((s(a) AX_a + s(b) AY_b) + s(c) AZ_c);
//   volume  V = (1/3) * sum_{l=1..7} (X_l - X_0).B_l;  dot = (x x' + y y') + z z';
//   length  L = V / sqrt(max_f |A_f|^2), faces in the order AX0 AX1 AY0 AY1 AZ0 AZ1;
//   S2-S6   DV = sum_l u_l.B_l; inv = 1/V; rho = m inv; D = DV inv; p~ = (gm1 rho) e+;
//           e_p = e - ((hh p~) DV)/m; p = (gm1 rho) ep+; c = sqrt(ggm1 ep+);
//           q: s = L (-D), qr = s ((q_quad s) + (q_lin c)); q = rho qr; P = p + q;
//           sigma = sqrt(c c + 2 qr); dt_z = min((cfl L)/sigma, c_vol/|D|);
//   S7      F = sum over existing zones l' = 0..7 of f_{7-l'}; m_p = 0.125 sum m; a = F (1/m_p);
//           u' = u + dt a; u_half = (u + u') 0.5; x' = x + dt u_half;
//   S8      W = sum_l f_l.u_half_l; e' = e - (dt W)/m.
#include <cmath>

#include "../kernels.h"
#include "../zone_physics.cuh"

namespace hydro {

namespace {

constexpr int SBX = 32, SBY = 4;

__device__ __forceinline__ double smin(double a, double b) { return (b < a) ? b : a; }
__device__ __forceinline__ double smax(double a, double b) { return (a < b) ? b : a; }
__device__ __forceinline__ double sdot(const double a[3], const double b[3]) {
  return (a[0] * b[0] + a[1] * b[1]) + a[2] * b[2];
}

__device__ __forceinline__ void sface(const double *P, int i1, int i0, int j1, int j0,
                                      double o[3]) {
  double a[3], b[3];
#pragma unroll
  for (int d = 0; d < 3; ++d) {
    a[d] = P[3 * i1 + d] - P[3 * i0 + d];
    b[d] = P[3 * j1 + d] - P[3 * j0 + d];
  }
  o[0] = 0.5 * (a[1] * b[2] - a[2] * b[1]);
  o[1] = 0.5 * (a[2] * b[0] - a[0] * b[2]);
  o[2] = 0.5 * (a[0] * b[1] - a[1] * b[0]);
}

// S2 geometry.  X: 8 corners x 3 (corner-major).
__device__ void s_geometry(const double X[24], double B[24], double &V, double &L) {
  double F[6][3];  // AX0 AX1 AY0 AY1 AZ0 AZ1
#pragma unroll
  for (int a = 0; a < 2; ++a) sface(X, a + 6, a, a + 4, a + 2, F[a]);
#pragma unroll
  for (int b = 0; b < 2; ++b) sface(X, 5 + 2 * b, 2 * b, 1 + 2 * b, 2 * b + 4, F[2 + b]);
#pragma unroll
  for (int c = 0; c < 2; ++c) sface(X, 3 + 4 * c, 4 * c, 2 + 4 * c, 1 + 4 * c, F[4 + c]);
#pragma unroll
  for (int l = 0; l < 8; ++l) {
    const int a = l & 1, b = (l >> 1) & 1, c = (l >> 2) & 1;
#pragma unroll
    for (int d = 0; d < 3; ++d) {
      const double sa = a ? F[1][d] : -F[0][d];
      const double sb = b ? F[3][d] : -F[2][d];
      const double sc = c ? F[5][d] : -F[4][d];
      B[3 * l + d] = 0.25 * ((sa + sb) + sc);
    }
  }
  double s = 0.0;
#pragma unroll
  for (int l = 1; l < 8; ++l) {
    double r[3];
#pragma unroll
    for (int d = 0; d < 3; ++d) r[d] = X[3 * l + d] - X[d];
    const double t = sdot(r, &B[3 * l]);
    s = (l == 1) ? t : s + t;
  }
  V = (1.0 / 3.0) * s;
  double a2max = 0.0;
#pragma unroll
  for (int f = 0; f < 6; ++f) {
    const double a2 = sdot(F[f], F[f]);
    a2max = (f == 0) ? a2 : smax(a2max, a2);
  }
  L = V / sqrt(a2max);
}

struct SOut {
  double rho, p, c, q, P, dtz, V;
};

// Reading R24 strain rates in the written order (face sums over corners in ascending l, each
// sum initialised by its first term; dx = 0.25 (sum+ - sum-); L^2 = dx.dx; eps = du.dx / L^2).
__device__ void s_strain(const double X[24], const double U[24], double eps[3], double L[3]) {
#pragma unroll
  for (int dd = 0; dd < 3; ++dd) {
    double xs[2][3], us[2][3];
    bool first[2] = {true, true};
#pragma unroll
    for (int l = 0; l < 8; ++l) {
      const int side = (l >> dd) & 1;
#pragma unroll
      for (int k = 0; k < 3; ++k) {
        xs[side][k] = first[side] ? X[3 * l + k] : xs[side][k] + X[3 * l + k];
        us[side][k] = first[side] ? U[3 * l + k] : us[side][k] + U[3 * l + k];
      }
      first[side] = false;
    }
    double dx[3], du[3];
#pragma unroll
    for (int k = 0; k < 3; ++k) {
      dx[k] = 0.25 * (xs[1][k] - xs[0][k]);
      du[k] = 0.25 * (us[1][k] - us[0][k]);
    }
    const double L2 = sdot(dx, dx);
    eps[dd] = sdot(du, dx) / L2;
    L[dd] = sqrt(L2);
  }
}

// S2 (DV, rho, D) + S3 + S4 + S6 of one zone; B is returned for S5.
__device__ void s_zone_state(const double X[24], const double U[24], double m, double e,
                             double hh, const Phys &ph, double B[24], SOut &o,
                             const double *phi = nullptr) {
  double V, L;
  s_geometry(X, B, V, L);
  double DV = 0.0;
#pragma unroll
  for (int l = 0; l < 8; ++l) {
    const double t = sdot(&U[3 * l], &B[3 * l]);
    DV = (l == 0) ? t : DV + t;
  }
  const double inv = 1.0 / V;
  const double rho = m * inv;
  const double D = DV * inv;
  const double epos = smax(e, 0.0);
  const double pt = (ph.gm1 * rho) * epos;
  const double ep = e - ((hh * pt) * DV) / m;
  const double eppos = smax(ep, 0.0);
  const double p = (ph.gm1 * rho) * eppos;
  const double c = sqrt(ph.ggm1 * eppos);
  double qr = 0.0;
  if (D < 0.0 && !phi) {
    const double s = L * (-D);
    qr = s * ((ph.q_quad * s) + (ph.q_lin * c));
  } else if (D < 0.0) {  // reading R24
    double eps[3], Ld[3];
    s_strain(X, U, eps, Ld);
#pragma unroll
    for (int dd = 0; dd < 3; ++dd) {
      const double dv = Ld[dd] * smax(-eps[dd], 0.0);
      const double t = ((ph.q_quad * dv) * dv) * (1.0 - phi[dd] * phi[dd]) +
                       ((ph.q_lin * c) * dv) * (1.0 - phi[dd]);
      qr = (dd == 0) ? t : qr + t;
    }
  }
  const double q = rho * qr;
  const double sig = sqrt(c * c + 2.0 * qr);
  const double dtc = (sig > 0.0) ? (ph.cfl * L) / sig : INFINITY;
  const double dtv = (D != 0.0) ? ph.c_vol / fabs(D) : INFINITY;
  o.rho = rho;
  o.p = p;
  o.c = c;
  o.q = q;
  o.P = p + q;
  o.dtz = smin(dtc, dtv);
  o.V = V;
}

// f1 / reading R17 in the written order (M, H, adjugate inverse, C, gamma, g, force).  cbrt is
// not correctly rounded on either side, so kappa > 0 is STRICT to within an ulp of V^(1/3), not
// bitwise.
__device__ void s_hourglass(const double X[24], const double U[24], const double B[24],
                            double V, double rho, double c, double kappa, double Fh[24]) {
  double h[4][8];
#pragma unroll
  for (int l = 0; l < 8; ++l) {
    const double xi = 2.0 * (l & 1) - 1.0, eta = 2.0 * ((l >> 1) & 1) - 1.0,
                 zeta = 2.0 * ((l >> 2) & 1) - 1.0;
    h[0][l] = eta * zeta;
    h[1][l] = zeta * xi;
    h[2][l] = xi * eta;
    h[3][l] = (xi * eta) * zeta;
  }
  double M[3][3], H[4][3];
  for (int d = 0; d < 3; ++d)
    for (int k = 0; k < 3; ++k) {
      double s = 0.0;
      for (int l = 0; l < 8; ++l) {
        const double t = B[3 * l + d] * X[3 * l + k];
        s = (l == 0) ? t : s + t;
      }
      M[d][k] = s;
    }
  for (int a = 0; a < 4; ++a)
    for (int k = 0; k < 3; ++k) {
      double s = 0.0;
      for (int l = 0; l < 8; ++l) {
        const double t = h[a][l] * X[3 * l + k];
        s = (l == 0) ? t : s + t;
      }
      H[a][k] = s;
    }
  double cof[3][3];
  for (int r = 0; r < 3; ++r)
    for (int q = 0; q < 3; ++q) {
      const int r1 = (r + 1) % 3, r2 = (r + 2) % 3, q1 = (q + 1) % 3, q2 = (q + 2) % 3;
      cof[r][q] = M[r1][q1] * M[r2][q2] - M[r1][q2] * M[r2][q1];
    }
  const double det = (M[0][0] * cof[0][0] + M[0][1] * cof[0][1]) + M[0][2] * cof[0][2];
  double Mi[3][3];
  for (int k = 0; k < 3; ++k)
    for (int d = 0; d < 3; ++d) Mi[k][d] = cof[d][k] / det;
  double C[4][3];
  for (int a = 0; a < 4; ++a)
    for (int d = 0; d < 3; ++d)
      C[a][d] = (H[a][0] * Mi[0][d] + H[a][1] * Mi[1][d]) + H[a][2] * Mi[2][d];
  double gam[4][8];
  for (int a = 0; a < 4; ++a)
    for (int l = 0; l < 8; ++l)
      gam[a][l] = h[a][l] - ((C[a][0] * B[3 * l] + C[a][1] * B[3 * l + 1]) +
                             C[a][2] * B[3 * l + 2]);
  double g[4][3];
  for (int a = 0; a < 4; ++a)
    for (int d = 0; d < 3; ++d) {
      double s = 0.0;
      for (int l = 0; l < 8; ++l) {
        const double t = gam[a][l] * U[3 * l + d];
        s = (l == 0) ? t : s + t;
      }
      g[a][d] = s;
    }
  const double v13 = cbrt(V);
  const double coef = -(((kappa * rho) * c) * (v13 * v13));
  for (int l = 0; l < 8; ++l)
    for (int d = 0; d < 3; ++d) {
      double s = 0.0;
      for (int a = 0; a < 4; ++a) {
        const double t = gam[a][l] * g[a][d];
        s = (a == 0) ? t : s + t;
      }
      Fh[3 * l + d] = coef * s;
    }
}

__device__ __forceinline__ bool s_exists(const DomView &d, int i, int j, int k) {
  const int64_t gx = d.lo[0] + i, gy = d.lo[1] + j, gz = d.lo[2] + k;
  return gx >= 0 && gx < d.N[0] && gy >= 0 && gy < d.N[1] && gz >= 0 && gz < d.N[2];
}
__device__ __forceinline__ int64_t s_gzone(const DomView &d, int i, int j, int k) {
  return ((d.lo[2] + k) * (int64_t)d.N[1] + (d.lo[1] + j)) * (int64_t)d.N[0] + (d.lo[0] + i);
}

// Corners of local zone (i,j,k): positions x + hh u (S1; hh = 0: x itself) and velocities.
__device__ __forceinline__ void s_gather(const DomView &d, int i, int j, int k, double hh,
                                         bool next, double X[24], double U[24]) {
  const double *x = next ? d.xn : d.x, *y = next ? d.yn : d.y, *z = next ? d.zn : d.z;
  const double *u = next ? d.un : d.u, *v = next ? d.vn : d.v, *w = next ? d.wn : d.w;
#pragma unroll
  for (int l = 0; l < 8; ++l) {
    const int64_t id = d.nid(i + (l & 1), j + ((l >> 1) & 1), k + ((l >> 2) & 1));
    U[3 * l] = u[id];
    U[3 * l + 1] = v[id];
    U[3 * l + 2] = w[id];
    X[3 * l] = (hh == 0.0) ? x[id] : x[id] + hh * U[3 * l];
    X[3 * l + 1] = (hh == 0.0) ? y[id] : y[id] + hh * U[3 * l + 1];
    X[3 * l + 2] = (hh == 0.0) ? z[id] : z[id] + hh * U[3 * l + 2];
  }
}

// R24 limiter inputs of local zone (i,j,k) (mono_phi: owner lookups + the written limiter)
__device__ __forceinline__ const double *s_phi(const DomView &d, const Phys &ph,
                                               const MonoMap &M, int i, int j, int k,
                                               double phi[3]) {
  if (ph.q_kind != 1) return nullptr;
  const int64_t g[3] = {d.lo[0] + i, d.lo[1] + j, d.lo[2] + k};
  mono_phi(M, d, g, ph.reflect_mask, phi);
  return phi;
}

__device__ __forceinline__ void s_flag(DevState *st, unsigned bits, int64_t gz) {
  atomicOr(&st->err, bits);
  atomicMin(&st->bad_zone, (unsigned long long)gz);
}

__device__ __forceinline__ void s_min_dt(double v, DevState *st) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const double w = __shfl_xor_sync(0xffffffffu, v, o);
    v = smin(v, w);
  }
  if ((threadIdx.x & 31) == 0 && v < INFINITY)
    atomicMin(&st->dtz_acc, (unsigned long long)__double_as_longlong(v));
}

// Zone masses (S start-up: m = rho0 V(X^0), or rho V for USER) and the Sedov corner energy.
__global__ void k_s_init_zones(DomView d, int kind, double rho0, double e0, double E) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x - 1;
  const int j = blockIdx.y * blockDim.y + threadIdx.y - 1;
  const int k = blockIdx.z - 1;
  if (i > d.n[0] || j > d.n[1] || !s_exists(d, i, j, k)) return;
  double X[24], U[24], B[24], V, L;
  s_gather(d, i, j, k, 0.0, false, X, U);
  s_geometry(X, B, V, L);
  const int64_t id = d.zid(i, j, k);
  double *m = const_cast<double *>(d.m);
  double *e = const_cast<double *>(d.e);
  if (kind == 0) {
    m[id] = rho0 * V;
    const bool corner = d.lo[0] + i == 0 && d.lo[1] + j == 0 && d.lo[2] + k == 0;
    e[id] = corner ? E / m[id] : e0;
  } else if (kind == 1) {
    m[id] = d.P[id] * V;
  }
}

// R24: strain rates of the owned zones at x + hh u (at_x: hh = 0).
__global__ void k_s_strain(DomView d, const DevState *st, int at_x) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  const int j = blockIdx.y * blockDim.y + threadIdx.y;
  const int k = blockIdx.z;
  if (i >= d.n[0] || j >= d.n[1]) return;
  double X[24], U[24], eps[3], L[3];
  s_gather(d, i, j, k, at_x ? 0.0 : 0.5 * st->dt, false, X, U);
  s_strain(X, U, eps, L);
  const int64_t id = d.zid(i, j, k);
  for (int dd = 0; dd < 3; ++dd) d.eps[(int64_t)dd * d.nzone + id] = eps[dd];
}

// dt^0: S2-S6 at x^0, no predictor, owned zones; also x^{n+1} := x (the other parity).
__global__ void k_s_dt0(DomView d, Phys ph, DevState *st, MonoMap M) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  const int j = blockIdx.y * blockDim.y + threadIdx.y;
  const int k = blockIdx.z;
  double dtz = INFINITY;
  if (i < d.n[0] && j < d.n[1]) {
    double X[24], U[24], B[24];
    SOut o;
    s_gather(d, i, j, k, 0.0, false, X, U);
    const int64_t id = d.zid(i, j, k);
    double phi[3];
    s_zone_state(X, U, d.m[id], d.e[id], 0.0, ph, B, o, s_phi(d, ph, M, i, j, k, phi));
    if (!(o.V > 0.0)) s_flag(st, ERR_TANGLED, s_gzone(d, i, j, k));
    dtz = (o.dtz == o.dtz) ? o.dtz : INFINITY;
  }
  s_min_dt(dtz, st);
}

// K1 (S1-S6): every existing zone of the domain and its ghost ring: corner forces
// f_l = P B_l (+ f_hg_l) into the 24 planes of d.B; dt_z over owned zones.
__global__ void k_s_zone(DomView d, Phys ph, DevState *st, MonoMap M) {
  if ((st->halted | st->done) != 0u) return;
  const int i = blockIdx.x * blockDim.x + threadIdx.x - 1;
  const int j = blockIdx.y * blockDim.y + threadIdx.y - 1;
  const int k = blockIdx.z - 1;
  const double hh = 0.5 * st->dt;
  double dtz = INFINITY;
  if (i <= d.n[0] && j <= d.n[1] && s_exists(d, i, j, k)) {
    double X[24], U[24], B[24];
    SOut o;
    s_gather(d, i, j, k, hh, false, X, U);
    const int64_t id = d.zid(i, j, k);
    double phi[3];
    s_zone_state(X, U, d.m[id], d.e[id], hh, ph, B, o, s_phi(d, ph, M, i, j, k, phi));
    double f[24];
#pragma unroll
    for (int c = 0; c < 24; ++c) f[c] = o.P * B[c];
    if (ph.hg > 0.0) {
      double Fh[24];
      s_hourglass(X, U, B, o.V, o.rho, o.c, ph.hg, Fh);
#pragma unroll
      for (int c = 0; c < 24; ++c) f[c] = f[c] + Fh[c];
    }
#pragma unroll
    for (int c = 0; c < 24; ++c) d.B[(int64_t)c * d.nzone + id] = f[c];
    d.P[id] = o.P;
    const bool owned = i >= 0 && j >= 0 && k >= 0 && i < d.n[0] && j < d.n[1] && k < d.n[2];
    if (owned) {
      if (!(o.V > 0.0)) s_flag(st, ERR_TANGLED, s_gzone(d, i, j, k));
      else if (!isfinite(o.P)) s_flag(st, ERR_NONFINITE, s_gzone(d, i, j, k));
      dtz = (o.dtz == o.dtz) ? o.dtz : INFINITY;
    }
  }
  s_min_dt(dtz, st);
}

// K2 (S7) for owned nodes (halted: carry the state to the next parity).
__global__ void k_s_node(DomView d, Phys ph, DevState *st) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  const int j = blockIdx.y * blockDim.y + threadIdx.y;
  const int k = blockIdx.z;
  if (i > d.n[0] || j > d.n[1]) return;
  const int64_t id = d.nid(i, j, k);
  if ((st->halted | st->done) != 0u) {
    d.xn[id] = d.x[id]; d.yn[id] = d.y[id]; d.zn[id] = d.z[id];
    d.un[id] = d.u[id]; d.vn[id] = d.v[id]; d.wn[id] = d.w[id];
    return;
  }
  const double dt = st->dt;
  double F[3] = {0.0, 0.0, 0.0}, ms = 0.0;
  bool first = true;
  for (int lp = 0; lp < 8; ++lp) {
    const int zi = i - 1 + (lp & 1), zj = j - 1 + ((lp >> 1) & 1), zk = k - 1 + ((lp >> 2) & 1);
    if (!s_exists(d, zi, zj, zk)) continue;
    const int64_t z = d.zid(zi, zj, zk);
    const int l = 7 - lp;
#pragma unroll
    for (int c = 0; c < 3; ++c) {
      const double f = d.B[(int64_t)(3 * l + c) * d.nzone + z];
      F[c] = first ? f : F[c] + f;
    }
    ms = first ? d.m[z] : ms + d.m[z];
    first = false;
  }
  const double mp = 0.125 * ms;
  const double rinv = 1.0 / mp;
  double a[3] = {F[0] * rinv, F[1] * rinv, F[2] * rinv};
  const int64_t g[3] = {d.lo[0] + i, d.lo[1] + j, d.lo[2] + k};
  const uint32_t rm = ph.reflect_mask;
#pragma unroll
  for (int c = 0; c < 3; ++c) {
    if (g[c] == 0 && ((rm >> (2 * c)) & 1u)) a[c] = 0.0;
    if (g[c] == d.N[c] && ((rm >> (2 * c + 1)) & 1u)) a[c] = 0.0;
  }
  const double *x[3] = {d.x, d.y, d.z}, *u[3] = {d.u, d.v, d.w};
  double *xn[3] = {d.xn, d.yn, d.zn}, *un[3] = {d.un, d.vn, d.wn};
#pragma unroll
  for (int c = 0; c < 3; ++c) {
    const double unc = u[c][id] + dt * a[c];
    const double uh = (u[c][id] + unc) * 0.5;
    un[c][id] = unc;
    xn[c][id] = x[c][id] + dt * uh;
  }
}

// K3 (S8) for owned zones.
__global__ void k_s_energy(DomView d, Phys ph, DevState *st) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  const int j = blockIdx.y * blockDim.y + threadIdx.y;
  const int k = blockIdx.z;
  if (i >= d.n[0] || j >= d.n[1]) return;
  const int64_t id = d.zid(i, j, k);
  if ((st->halted | st->done) != 0u) {
    d.en[id] = d.e[id];
    return;
  }
  const double dt = st->dt;
  double W = 0.0;
#pragma unroll
  for (int l = 0; l < 8; ++l) {
    const int64_t n = d.nid(i + (l & 1), j + ((l >> 1) & 1), k + ((l >> 2) & 1));
    const double uh[3] = {(d.u[n] + d.un[n]) * 0.5, (d.v[n] + d.vn[n]) * 0.5,
                          (d.w[n] + d.wn[n]) * 0.5};
    double f[3];
#pragma unroll
    for (int c = 0; c < 3; ++c) f[c] = d.B[(int64_t)(3 * l + c) * d.nzone + id];
    const double t = sdot(f, uh);
    W = (l == 0) ? t : W + t;
  }
  d.en[id] = d.e[id] - (dt * W) / d.m[id];
}

// Outputs: rho, p, q, c, V by S2-S4 at (x, u) with e_p = e.
__global__ void k_s_derive(DomView d, Phys ph, MonoMap M) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  const int j = blockIdx.y * blockDim.y + threadIdx.y;
  const int k = blockIdx.z;
  if (i >= d.n[0] || j >= d.n[1]) return;
  double X[24], U[24], B[24];
  SOut o;
  s_gather(d, i, j, k, 0.0, false, X, U);
  const int64_t id = d.zid(i, j, k);
  double phi[3];
  s_zone_state(X, U, d.m[id], d.e[id], 0.0, ph, B, o, s_phi(d, ph, M, i, j, k, phi));
  d.aux[0 * d.nzone + id] = o.rho;
  d.aux[1 * d.nzone + id] = o.p;
  d.aux[2 * d.nzone + id] = o.q;
  d.aux[3 * d.nzone + id] = o.c;
  d.aux[4 * d.nzone + id] = o.V;
}

dim3 sgrid(int nx, int ny, int nz) { return dim3((nx + SBX - 1) / SBX, (ny + SBY - 1) / SBY, nz); }

}  // namespace

void launch_strict_init_zones(const DomView &d, int kind, double rho0, double e0, double E,
                              cudaStream_t s) {
  k_s_init_zones<<<sgrid(d.n[0] + 2, d.n[1] + 2, d.n[2] + 2), dim3(SBX, SBY), 0, s>>>(
      d, kind, rho0, e0, E);
}
void launch_strict_dt0(const DomView &d, const Phys &ph, DevState *st, const MonoMap &M,
                       cudaStream_t s) {
  k_s_dt0<<<sgrid(d.n[0], d.n[1], d.n[2]), dim3(SBX, SBY), 0, s>>>(d, ph, st, M);
}
void launch_strict_strain(const DomView &d, const DevState *st, int at_x, cudaStream_t s) {
  k_s_strain<<<sgrid(d.n[0], d.n[1], d.n[2]), dim3(SBX, SBY), 0, s>>>(d, st, at_x);
}
void launch_strict_zone(const DomView &d, const Phys &ph, DevState *st, const MonoMap &M,
                        cudaStream_t s) {
  k_s_zone<<<sgrid(d.n[0] + 2, d.n[1] + 2, d.n[2] + 2), dim3(SBX, SBY), 0, s>>>(d, ph, st, M);
}
void launch_strict_node(const DomView &d, const Phys &ph, DevState *st, cudaStream_t s) {
  k_s_node<<<sgrid(d.n[0] + 1, d.n[1] + 1, d.n[2] + 1), dim3(SBX, SBY), 0, s>>>(d, ph, st);
}
void launch_strict_energy(const DomView &d, const Phys &ph, DevState *st, cudaStream_t s) {
  k_s_energy<<<sgrid(d.n[0], d.n[1], d.n[2]), dim3(SBX, SBY), 0, s>>>(d, ph, st);
}
void launch_strict_derive(const DomView &d, const Phys &ph, const MonoMap &M, cudaStream_t s) {
  k_s_derive<<<sgrid(d.n[0], d.n[1], d.n[2]), dim3(SBX, SBY), 0, s>>>(d, ph, M);
}

}  // namespace hydro
