// kernels_common.cu -- initialisation, dt bookkeeping (S9), halo copy and output derivation
// kernels, plus the split 3-kernel pipeline (zone / node / energy) that serves as the plain,
// one-thread-per-element GPU path (HYDRO_FLAG_SPLIT).  The fused default path is in
// kernel_fused.cu.
#include <algorithm>
#include <cmath>

#include "kernels.h"
#include "zone_physics.cuh"

namespace hydro {

namespace {

constexpr int BX = 32, BY = 4;

__device__ __forceinline__ bool stopped(const DevState *st) {
  return (st->halted | st->done) != 0u;
}

__device__ __forceinline__ bool exists_zone(const DomView &d, int i, int j, int k) {
  const int64_t gx = d.lo[0] + i, gy = d.lo[1] + j, gz = d.lo[2] + k;
  return gx >= 0 && gx < d.N[0] && gy >= 0 && gy < d.N[1] && gz >= 0 && gz < d.N[2];
}

__device__ __forceinline__ int64_t global_zone(const DomView &d, int i, int j, int k) {
  return ((d.lo[2] + k) * (int64_t)d.N[1] + (d.lo[1] + j)) * (int64_t)d.N[0] + (d.lo[0] + i);
}

// Gather the 8 corners of local zone (i,j,k): positions advanced by hh*u, and velocities.
__device__ __forceinline__ void gather(const DomView &d, int i, int j, int k, double hh,
                                       double X[8], double Y[8], double Z[8], double U[8],
                                       double V[8], double W[8]) {
#pragma unroll
  for (int l = 0; l < 8; ++l) {
    const int64_t id = d.nid(i + (l & 1), j + ((l >> 1) & 1), k + ((l >> 2) & 1));
    U[l] = d.u[id];
    V[l] = d.v[id];
    W[l] = d.w[id];
    X[l] = d.x[id] + hh * U[l];
    Y[l] = d.y[id] + hh * V[l];
    Z[l] = d.z[id] + hh * W[l];
  }
}

__device__ __forceinline__ void flag_error(DevState *st, unsigned bits, int64_t gzone) {
  atomicOr(&st->err, bits);
  atomicMin(&st->bad_zone, (unsigned long long)gzone);
}

// ------------------------------------------------------------------------------- init
__global__ void k_init_nodes(DomView d, double ox, double oy, double oz, double lx, double ly,
                             double lz) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x - 1;
  const int j = blockIdx.y * blockDim.y + threadIdx.y - 1;
  const int k = blockIdx.z - 1;
  if (i > d.n[0] + 1 || j > d.n[1] + 1) return;
  const int64_t id = d.nid(i, j, k);
  // reading R1: origin + (extent*g)/N (also for ghost nodes beyond the physical boundary)
  const double X = ox + (lx * (double)(d.lo[0] + i)) / (double)d.N[0];
  const double Y = oy + (ly * (double)(d.lo[1] + j)) / (double)d.N[1];
  const double Z = oz + (lz * (double)(d.lo[2] + k)) / (double)d.N[2];
  const_cast<double *>(d.x)[id] = X;
  const_cast<double *>(d.y)[id] = Y;
  const_cast<double *>(d.z)[id] = Z;
  d.xn[id] = X;
  d.yn[id] = Y;
  d.zn[id] = Z;
}

__global__ void k_init_zones(DomView d, int kind, double rho0, double e0, double E) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x - 1;
  const int j = blockIdx.y * blockDim.y + threadIdx.y - 1;
  const int k = blockIdx.z - 1;
  if (i > d.n[0] || j > d.n[1] || !exists_zone(d, i, j, k)) return;
  double X[8], Y[8], Z[8], U[8], Vv[8], W[8], Bx[8], By[8], Bz[8], V, A2;
  gather(d, i, j, k, 0.0, X, Y, Z, U, Vv, W);
  hex_geometry(X, Y, Z, Bx, By, Bz, V, A2);
  const int64_t id = d.zid(i, j, k);
  double *m = const_cast<double *>(d.m);
  double *e = const_cast<double *>(d.e);
  if (kind == 0) {
    m[id] = rho0 * V;
    const bool corner = d.lo[0] + i == 0 && d.lo[1] + j == 0 && d.lo[2] + k == 0;
    e[id] = corner ? E / m[id] : e0;
  } else if (kind == 1) {
    m[id] = d.P[id] * V;  // USER: rho staged in the P scratch
  }
}

// Nodal inverse mass for the cycle kernels (S7: m_p = sum_z m_z / 8; zones outside the mesh have
// m = 0).  Summed in the order the node stage used to sum it on the fly (x pairs, y pairs, then
// the plane below + the plane above).
__global__ void k_nodal_mass(DomView d) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  const int j = blockIdx.y * blockDim.y + threadIdx.y;
  const int k = blockIdx.z;
  if (i > d.n[0] || j > d.n[1]) return;
  double ms[2];
#pragma unroll
  for (int c = 0; c < 2; ++c) {
    const int kk = k - 1 + c;
    ms[c] = (d.m[d.zid(i - 1, j - 1, kk)] + d.m[d.zid(i, j - 1, kk)]) +
            (d.m[d.zid(i - 1, j, kk)] + d.m[d.zid(i, j, kk)]);
  }
  const double M = ms[0] + ms[1];
  d.mn8[d.nid(i, j, k)] = M > 0.0 ? 8.0 / M : 0.0;
}

__global__ void k_inv_mass(DomView d, int64_t nz) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nz;
       i += (int64_t)gridDim.x * blockDim.x) {
    const double m = d.m[i];
    d.mi[i] = m > 0.0 ? 1.0 / m : 0.0;
  }
}

// dt^0: S2-S6 at x^0 with no predictor over owned zones.
// Reading R24 (monotone q): the limiter values and the zone's own strain data (phi[3],
// epsL[6]) of local zone (i,j,k) from its corners; false = scalar q.
__device__ __forceinline__ bool mono_inputs(const DomView &d, const Phys &ph, const MonoMap &M,
                                            int i, int j, int k, const double X[8],
                                            const double Y[8], const double Z[8],
                                            const double U[8], const double Vv[8],
                                            const double W[8], double phi[3], double epsL[6]) {
  if (ph.q_kind != 1) return false;
  const int64_t g[3] = {d.lo[0] + i, d.lo[1] + j, d.lo[2] + k};
  mono_phi(M, d, g, ph.reflect_mask, phi);
  zone_strain(X, Y, Z, U, Vv, W, epsL, epsL + 3);
  return true;
}

// Reading R24: strain rates of the owned zones at x + hh u (hh = dt/2, or 0 with at_x).
__global__ void k_strain(DomView d, const DevState *st, int at_x) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  const int j = blockIdx.y * blockDim.y + threadIdx.y;
  const int k = blockIdx.z;
  if (i >= d.n[0] || j >= d.n[1]) return;
  const double hh = at_x ? 0.0 : 0.5 * st->dt;
  double X[8], Y[8], Z[8], U[8], Vv[8], W[8], eps[3], L[3];
  gather(d, i, j, k, hh, X, Y, Z, U, Vv, W);
  zone_strain(X, Y, Z, U, Vv, W, eps, L);
  const int64_t id = d.zid(i, j, k);
#pragma unroll
  for (int dd = 0; dd < 3; ++dd) d.eps[(int64_t)dd * d.nzone + id] = eps[dd];
}

__global__ void k_dt0(DomView d, Phys ph, DevState *st, MonoMap M) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  const int j = blockIdx.y * blockDim.y + threadIdx.y;
  const int k = blockIdx.z;
  double dtz = INFINITY;
  if (i < d.n[0] && j < d.n[1]) {
    double X[8], Y[8], Z[8], U[8], Vv[8], W[8], Bx[8], By[8], Bz[8], V, A2;
    gather(d, i, j, k, 0.0, X, Y, Z, U, Vv, W);
    hex_geometry(X, Y, Z, Bx, By, Bz, V, A2);
    double DV = 0.0;
#pragma unroll
    for (int l = 0; l < 8; ++l) DV += U[l] * Bx[l] + Vv[l] * By[l] + W[l] * Bz[l];
    const int64_t id = d.zid(i, j, k);
    double phi[3], epsL[6];
    const bool mono = mono_inputs(d, ph, M, i, j, k, X, Y, Z, U, Vv, W, phi, epsL);
    const ZoneEos r = zone_eos(V, A2, DV, d.m[id], d.e[id], 0.0, ph, mono ? phi : nullptr,
                               mono ? epsL : nullptr);
    if (!(V > 0.0)) flag_error(st, ERR_TANGLED, global_zone(d, i, j, k));
    dtz = (r.dtz == r.dtz) ? r.dtz : INFINITY;
  }
  block_min_dt(dtz, &st->dtz_acc);
}

__global__ void k_finalize_init(DevState *st, double dt_first, double dt_init, double dt_max,
                                double t_stop, double t0, double dt_floor) {
  const double dtmin = __longlong_as_double((long long)st->dtz_acc);
  double dt = dt_first > 0.0 ? dt_first : fmin(fmin(dt_init, dt_max), dtmin);
  // reading R23: the dt-collapse floor, relative to dt^0 (before the t_stop clamp) unless given
  st->dt_floor = dt_floor > 0.0 ? dt_floor : (dt_floor == 0.0 && isfinite(dt)) ? 1e-6 * dt : 0.0;
  if (t_stop > 0.0) dt = fmin(dt, t_stop - t0);
  st->t = t0;
  st->dt = dt;
  st->dtz_last = dtmin;
  st->dtz_acc = (unsigned long long)__double_as_longlong(INFINITY);
  st->cycle = 0;
  st->halted = st->err;
  st->done = (t_stop > 0.0 && t0 >= t_stop) ? 1u : 0u;
}

// S9 as its own kernel (multi-domain / multi-rank cycles; see finalize_cycle).
__global__ void k_finalize(DevState *st, Phys ph) {
  pdl_wait_and_trigger();
  finalize_cycle(st, ph);
}

// ------------------------------------------------------------------ split pipeline
// K1: S1-S6 for every existing local zone (owned and ghost): P and the 24 corner-vector
// components to scratch, dt_z min over owned zones.
__global__ void k_zone_split(DomView d, Phys ph, DevState *st, MonoMap M) {
  if (stopped(st)) return;
  const int i = blockIdx.x * blockDim.x + threadIdx.x - 1;
  const int j = blockIdx.y * blockDim.y + threadIdx.y - 1;
  const int k = blockIdx.z - 1;
  const double hh = 0.5 * st->dt;
  double dtz = INFINITY;
  if (i <= d.n[0] && j <= d.n[1] && exists_zone(d, i, j, k)) {
    double X[8], Y[8], Z[8], U[8], Vv[8], W[8], Bx[8], By[8], Bz[8], V, A2;
    gather(d, i, j, k, hh, X, Y, Z, U, Vv, W);
    hex_geometry(X, Y, Z, Bx, By, Bz, V, A2);
    double DV = 0.0;
#pragma unroll
    for (int l = 0; l < 8; ++l) DV += U[l] * Bx[l] + Vv[l] * By[l] + W[l] * Bz[l];
    const int64_t id = d.zid(i, j, k);
    double phi[3], epsL[6];
    const bool mono = mono_inputs(d, ph, M, i, j, k, X, Y, Z, U, Vv, W, phi, epsL);
    const ZoneEos r = zone_eos(V, A2, DV, d.m[id], d.e[id], hh, ph, mono ? phi : nullptr,
                               mono ? epsL : nullptr);
    d.P[id] = r.P;
    // S5 corner forces f_l = P B_l (+ the f1 hourglass force), 24 planes for K2 and K3
    double Fx[8], Fy[8], Fz[8];
#pragma unroll
    for (int l = 0; l < 8; ++l) {
      Fx[l] = r.P * Bx[l];
      Fy[l] = r.P * By[l];
      Fz[l] = r.P * Bz[l];
    }
    if (ph.hg > 0.0)
      hourglass_add(X, Y, Z, U, Vv, W, Bx, By, Bz, V, r.rho, r.c, ph.hg, Fx, Fy, Fz);
#pragma unroll
    for (int l = 0; l < 8; ++l) {
      d.B[(3 * l + 0) * d.nzone + id] = Fx[l];
      d.B[(3 * l + 1) * d.nzone + id] = Fy[l];
      d.B[(3 * l + 2) * d.nzone + id] = Fz[l];
    }
    const bool owned = i >= 0 && j >= 0 && k >= 0 && i < d.n[0] && j < d.n[1] && k < d.n[2];
    if (owned) {
      if (!(V > 0.0)) flag_error(st, ERR_TANGLED, global_zone(d, i, j, k));
      else if (!isfinite(r.P)) flag_error(st, ERR_NONFINITE, global_zone(d, i, j, k));
      dtz = (r.dtz == r.dtz) ? r.dtz : INFINITY;
    }
  }
  block_min_dt(dtz, &st->dtz_acc);
}

// K2: S5 + S7 for owned nodes: gather the corner forces f from the existing zones around the node,
// acceleration, reflecting walls, velocity and position update.
__global__ void k_node_split(DomView d, Phys ph, DevState *st) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  const int j = blockIdx.y * blockDim.y + threadIdx.y;
  const int k = blockIdx.z;
  if (i > d.n[0] || j > d.n[1]) return;
  const int64_t id = d.nid(i, j, k);
  if (stopped(st)) {
    d.xn[id] = d.x[id]; d.yn[id] = d.y[id]; d.zn[id] = d.z[id];
    d.un[id] = d.u[id]; d.vn[id] = d.v[id]; d.wn[id] = d.w[id];
    return;
  }
  const double dt = st->dt;
  double Fx = 0.0, Fy = 0.0, Fz = 0.0, ms = 0.0;
#pragma unroll
  for (int lp = 0; lp < 8; ++lp) {
    const int zi = i - 1 + (lp & 1), zj = j - 1 + ((lp >> 1) & 1), zk = k - 1 + ((lp >> 2) & 1);
    if (!exists_zone(d, zi, zj, zk)) continue;
    const int64_t z = d.zid(zi, zj, zk);
    const int l = 7 - lp;
    Fx += d.B[(3 * l + 0) * d.nzone + z];
    Fy += d.B[(3 * l + 1) * d.nzone + z];
    Fz += d.B[(3 * l + 2) * d.nzone + z];
    ms += d.m[z];
  }
  const double rinv = 1.0 / (0.125 * ms);
  double ax = Fx * rinv, ay = Fy * rinv, az = Fz * rinv;
  const int64_t g[3] = {d.lo[0] + i, d.lo[1] + j, d.lo[2] + k};
  const uint32_t rm = ph.reflect_mask;
  if ((g[0] == 0 && (rm & 1u)) || (g[0] == d.N[0] && (rm & 2u))) ax = 0.0;
  if ((g[1] == 0 && (rm & 4u)) || (g[1] == d.N[1] && (rm & 8u))) ay = 0.0;
  if ((g[2] == 0 && (rm & 16u)) || (g[2] == d.N[2] && (rm & 32u))) az = 0.0;
  const double u = d.u[id], v = d.v[id], w = d.w[id];
  const double un = u + dt * ax, vn = v + dt * ay, wn = w + dt * az;
  const double uh = (u + un) * 0.5, vh = (v + vn) * 0.5, wh = (w + wn) * 0.5;
  d.un[id] = un;
  d.vn[id] = vn;
  d.wn[id] = wn;
  d.xn[id] = d.x[id] + dt * uh;
  d.yn[id] = d.y[id] + dt * vh;
  d.zn[id] = d.z[id] + dt * wh;
}

// K3: S8 for owned zones: W = sum_l f_l.u_half_l, e' = e - dt W / m.
__global__ void k_energy_split(DomView d, Phys ph, DevState *st) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  const int j = blockIdx.y * blockDim.y + threadIdx.y;
  const int k = blockIdx.z;
  if (i >= d.n[0] || j >= d.n[1]) return;
  const int64_t id = d.zid(i, j, k);
  if (stopped(st)) {
    d.en[id] = d.e[id];
    return;
  }
  const double dt = st->dt;
  double Wk = 0.0;
#pragma unroll
  for (int l = 0; l < 8; ++l) {
    const int64_t n = d.nid(i + (l & 1), j + ((l >> 1) & 1), k + ((l >> 2) & 1));
    const double uh = (d.u[n] + d.un[n]) * 0.5;
    const double vh = (d.v[n] + d.vn[n]) * 0.5;
    const double wh = (d.w[n] + d.wn[n]) * 0.5;
    Wk += d.B[(3 * l + 0) * d.nzone + id] * uh + d.B[(3 * l + 1) * d.nzone + id] * vh +
          d.B[(3 * l + 2) * d.nzone + id] * wh;
  }
  d.en[id] = d.e[id] - dt * Wk / d.m[id];
}

// ---------------------------------------------------------------------- halo copy
__global__ void k_halo_copy(const DomView *views, const HaloCopy *chunks) {
  // one CTA per chunk of HALO_CHUNK slab elements (host-built list): no idle CTAs
  // for the many small edge and corner slabs.  32-bit index arithmetic (slabs and domain storage
  // are below 2^31 elements).
  const HaloCopy p = chunks[blockIdx.x];
  const DomView &D = views[p.dst];
  const DomView &S = views[p.src];
  if (p.kind == 0) {
    const int nx = (int)(p.nhi[0] - p.nlo[0]), ny = (int)(p.nhi[1] - p.nlo[1]);
    const int dsx = (int)D.nsx, dsxy = (int)D.nsxy, ssx = (int)S.nsx, ssxy = (int)S.nsxy;
    const int d0 = (int)D.nid((int)(p.nlo[0] - D.lo[0]), (int)(p.nlo[1] - D.lo[1]),
                              (int)(p.nlo[2] - D.lo[2]));
    const int s0 = (int)S.nid((int)(p.nlo[0] - S.lo[0]), (int)(p.nlo[1] - S.lo[1]),
                              (int)(p.nlo[2] - S.lo[2]));
    // Sources are read through the read-only path and every load of an element pair is issued
    // before its stores (a source element is never a ghost written by this kernel, so the loads
    // need not wait for earlier stores): two elements, twelve loads in flight per thread.
    const int end = p.start + p.count;
    for (int t = p.start + threadIdx.x; t < end; t += 2 * blockDim.x) {
      const int t2 = t + blockDim.x < end ? t + blockDim.x : t;
      const int a = t % nx, r = t / nx, b = r % ny, c = r / ny;
      const int a2 = t2 % nx, r2 = t2 / nx, b2 = r2 % ny, c2 = r2 / ny;
      const int di = d0 + c * dsxy + b * dsx + a, si = s0 + c * ssxy + b * ssx + a;
      const int di2 = d0 + c2 * dsxy + b2 * dsx + a2, si2 = s0 + c2 * ssxy + b2 * ssx + a2;
      const double v0 = __ldg(S.xn + si), v1 = __ldg(S.yn + si), v2 = __ldg(S.zn + si);
      const double v3 = __ldg(S.un + si), v4 = __ldg(S.vn + si), v5 = __ldg(S.wn + si);
      const double w0 = __ldg(S.xn + si2), w1 = __ldg(S.yn + si2), w2 = __ldg(S.zn + si2);
      const double w3 = __ldg(S.un + si2), w4 = __ldg(S.vn + si2), w5 = __ldg(S.wn + si2);
      D.xn[di] = v0; D.yn[di] = v1; D.zn[di] = v2;
      D.un[di] = v3; D.vn[di] = v4; D.wn[di] = v5;
      D.xn[di2] = w0; D.yn[di2] = w1; D.zn[di2] = w2;
      D.un[di2] = w3; D.vn[di2] = w4; D.wn[di2] = w5;
    }
  } else {
    const int zx = (int)(p.zhi[0] - p.zlo[0]), zy = (int)(p.zhi[1] - p.zlo[1]);
    const int zdsx = (int)D.zsx, zdsxy = (int)D.zsxy, zssx = (int)S.zsx, zssxy = (int)S.zsxy;
    const int zd0 = (int)D.zid((int)(p.zlo[0] - D.lo[0]), (int)(p.zlo[1] - D.lo[1]),
                               (int)(p.zlo[2] - D.lo[2]));
    const int zs0 = (int)S.zid((int)(p.zlo[0] - S.lo[0]), (int)(p.zlo[1] - S.lo[1]),
                               (int)(p.zlo[2] - S.lo[2]));
    // kind 1: next-parity e; kind 2: this cycle's P (zone-stage ring zones, before the node
    // stage)
    const double *src = p.kind == 2 ? S.P : S.en;
    double *dst = p.kind == 2 ? D.P : D.en;
    for (int t = p.start + threadIdx.x; t < p.start + p.count; t += blockDim.x) {
      const int a = t % zx, r = t / zx, b = r % zy, c = r / zy;
      dst[zd0 + c * zdsxy + b * zdsx + a] = __ldg(src + zs0 + c * zssxy + b * zssx + a);
    }
  }
}

// ------------------------------------------------------------------------ outputs
__global__ void k_derive(DomView d, Phys ph, MonoMap M) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  const int j = blockIdx.y * blockDim.y + threadIdx.y;
  const int k = blockIdx.z;
  if (i >= d.n[0] || j >= d.n[1]) return;
  double X[8], Y[8], Z[8], U[8], Vv[8], W[8], Bx[8], By[8], Bz[8], V, A2;
  gather(d, i, j, k, 0.0, X, Y, Z, U, Vv, W);
  hex_geometry(X, Y, Z, Bx, By, Bz, V, A2);
  double DV = 0.0;
#pragma unroll
  for (int l = 0; l < 8; ++l) DV += U[l] * Bx[l] + Vv[l] * By[l] + W[l] * Bz[l];
  const int64_t id = d.zid(i, j, k);
  double phi[3], epsL[6];
  const bool mono = mono_inputs(d, ph, M, i, j, k, X, Y, Z, U, Vv, W, phi, epsL);
  const ZoneEos r = zone_eos(V, A2, DV, d.m[id], d.e[id], 0.0, ph, mono ? phi : nullptr,
                             mono ? epsL : nullptr);
  d.aux[0 * d.nzone + id] = r.rho;
  d.aux[1 * d.nzone + id] = r.p;
  d.aux[2 * d.nzone + id] = r.q;
  d.aux[3 * d.nzone + id] = r.c;
  d.aux[4 * d.nzone + id] = V;
}

// Strided 3-D box copy between device arrays (host transfers go through a contiguous staging
// buffer: one full-bandwidth DMA plus this kernel, instead of a row-by-row 3-D memcpy).
__global__ void k_copy3d(const double *__restrict__ src, int64_t ssx, int64_t ssxy,
                         double *__restrict__ dst, int64_t dsx, int64_t dsxy, int ex) {
  const int j = blockIdx.y, k = blockIdx.z;
  const double *s = src + k * ssxy + j * ssx;
  double *d = dst + k * dsxy + j * dsx;
  for (int i = threadIdx.x; i < ex; i += blockDim.x) d[i] = s[i];
}

dim3 grid_for(int nx, int ny, int nz) {
  return dim3((nx + BX - 1) / BX, (ny + BY - 1) / BY, nz);
}

}  // namespace

void launch_init_nodes(const DomView &d, const double o[3], const double L[3], cudaStream_t s) {
  k_init_nodes<<<grid_for(d.n[0] + 3, d.n[1] + 3, d.n[2] + 3), dim3(BX, BY), 0, s>>>(
      d, o[0], o[1], o[2], L[0], L[1], L[2]);
}
void launch_init_zones(const DomView &d, int kind, double rho0, double e0, double E,
                       cudaStream_t s) {
  k_init_zones<<<grid_for(d.n[0] + 2, d.n[1] + 2, d.n[2] + 2), dim3(BX, BY), 0, s>>>(
      d, kind, rho0, e0, E);
}
void launch_nodal_mass(const DomView &d, cudaStream_t s) {
  const int64_t nz = d.zsxy * (d.n[2] + 2);
  k_inv_mass<<<(int)std::min<int64_t>((nz + 255) / 256, 4096), 256, 0, s>>>(d, nz);
  k_nodal_mass<<<grid_for(d.n[0] + 1, d.n[1] + 1, d.n[2] + 1), dim3(BX, BY), 0, s>>>(d);
}
void launch_strain(const DomView &d, const DevState *st, int at_x, cudaStream_t s) {
  k_strain<<<grid_for(d.n[0], d.n[1], d.n[2]), dim3(BX, BY), 0, s>>>(d, st, at_x);
}
void launch_dt0(const DomView &d, const Phys &ph, DevState *st, const MonoMap &M,
                cudaStream_t s) {
  k_dt0<<<grid_for(d.n[0], d.n[1], d.n[2]), dim3(BX, BY), 0, s>>>(d, ph, st, M);
}
void launch_finalize_init(DevState *st, double dt_first, double dt_init, double dt_max,
                          double t_stop, double t0, double dt_floor, cudaStream_t s) {
  k_finalize_init<<<1, 1, 0, s>>>(st, dt_first, dt_init, dt_max, t_stop, t0, dt_floor);
}
// hydro_run_batch: a fresh clock for the next batch (t, dt given; cycle 0; errors cleared).
__global__ void k_reset_clock(DevState *st, double t, double dt, unsigned done) {
  st->t = t;
  st->dt = dt;
  st->cycle = 0;
  st->err = 0;
  st->halted = 0;
  st->done = done;
  st->bad_zone = ~0ull;
  st->dtz_acc = (unsigned long long)__double_as_longlong(INFINITY);
}
void launch_reset_clock(DevState *st, double t, double dt, unsigned done, cudaStream_t s) {
  k_reset_clock<<<1, 1, 0, s>>>(st, t, dt, done);
}
void launch_zone_split(const DomView &d, const Phys &ph, DevState *st, const MonoMap &M,
                       cudaStream_t s) {
  k_zone_split<<<grid_for(d.n[0] + 2, d.n[1] + 2, d.n[2] + 2), dim3(BX, BY), 0, s>>>(d, ph, st,
                                                                                     M);
}
void launch_node_split(const DomView &d, const Phys &ph, DevState *st, cudaStream_t s) {
  k_node_split<<<grid_for(d.n[0] + 1, d.n[1] + 1, d.n[2] + 1), dim3(BX, BY), 0, s>>>(d, ph, st);
}
void launch_energy_split(const DomView &d, const Phys &ph, DevState *st, cudaStream_t s) {
  k_energy_split<<<grid_for(d.n[0], d.n[1], d.n[2]), dim3(BX, BY), 0, s>>>(d, ph, st);
}
bool pdl_enabled() {
  static const int on = getenv("HYDRO_NO_PDL") && atoi(getenv("HYDRO_NO_PDL")) ? 0 : 1;
  return on != 0;
}

void launch_finalize(DevState *st, const Phys &ph, cudaStream_t s) {
  launch_pdl(k_finalize, dim3(1), dim3(1), 0, s, st, ph);
}
void launch_halo_copy(const DomView *views_dev, const HaloCopy *chunks_dev, int nchunks,
                      cudaStream_t s) {
  if (nchunks <= 0) return;
  k_halo_copy<<<nchunks, 256, 0, s>>>(views_dev, chunks_dev);
}
void launch_copy3d(const double *src, int64_t ssx, int64_t ssxy, double *dst, int64_t dsx,
                   int64_t dsxy, int ex, int ey, int ez, cudaStream_t s) {
  if (ex <= 0 || ey <= 0 || ez <= 0) return;
  k_copy3d<<<dim3(1, ey, ez), 128, 0, s>>>(src, ssx, ssxy, dst, dsx, dsxy, ex);
}

void launch_derive(const DomView &d, const Phys &ph, const MonoMap &M, cudaStream_t s) {
  k_derive<<<grid_for(d.n[0], d.n[1], d.n[2]), dim3(BX, BY), 0, s>>>(d, ph, M);
}

}  // namespace hydro
