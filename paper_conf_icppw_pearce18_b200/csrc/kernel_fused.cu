// kernel_fused.cu -- the whole cycle S1-S8 (+ the block part of S9's dt min) in ONE kernel.
//
// Blocking.  A block owns a TX x TY column of zones of one domain and marches it
// through a z-chunk [k0, k1) ("2.5-D" blocking).  Node planes stream in through TMA
// (cp.async.bulk.tensor, one 36x15 box per field, mbarrier completion) into a 3-slot ring two
// planes ahead of use, so HBM latency is off the critical path.  Per zone plane p, separated by
// __syncthreads:
//   X  half-step positions x_p = x + dt/2 u of node plane p+1 (S1) into a 2-plane ring;
//   Z  zone stage on the (TX+2) x (TY+2) zones of plane p, i.e. the tile plus a one-zone ring
//      that is recomputed redundantly instead of exchanged: faces, corner vectors, V, DV,
//      predictor, EOS, q, P, dt_z^2 (S2-S4, S6);
//   G  per-face force vectors g_f = (P_below - P_above) A_f / 4 of each zone's three low faces
//      (the face form of S5: the node force sum_z P_z B_z,l regrouped by faces);
//   N  node stage on node plane p: F = sum of the 12 incident g_f, m_p, a, reflecting walls,
//      u', u_half, x' (S7), written to HBM;
//   E  energy stage on zone plane p-1: W = P sum_l B_l.u_half_l in face form
//      (psi_f = A_f . sum of u_half over the face), e' = e - dt W / m (S8), written to HBM.
// HBM traffic per zone-cycle is the algorithmic minimum (read x,u,m,e; write x,u,e) plus the
// re-read of the tile's halo columns; every intermediate lives in registers or shared memory.
// No tensor cores: nothing here is a dense contraction (BASELINE.json north_star).
#include <algorithm>
#include <cmath>

#include "fastmath.cuh"
#include "kernels.h"
#include "zone_physics.cuh"

namespace hydro {

namespace {

template <int TX, int TY>
struct Tile {
  static constexpr int TXT = TX + 2, TYT = TY + 2;  // zone-stage tile (owned + 1 ring)
  static constexpr int NZT = TXT * TYT;
  static constexpr int NTHR = (NZT + 31) / 32 * 32;
  static constexpr int ZS = NTHR;                   // stride of per-zone smem arrays
  static constexpr int BXN = FUSED_BOX_X, BYN = TY + 3;  // TMA node box (x padded to 16 B)
  static constexpr int NN = BXN * BYN;
  static constexpr int RS = (NN + 15) / 16 * 16;    // stride of one node array (128 B aligned)
  // shared-memory layout, in doubles
  static constexpr int OFF_RAW = 0;                 // [3 slots][6 fields][RS] x,y,z,u,v,w
  static constexpr int OFF_XP = OFF_RAW + 18 * RS;  // [2 planes][3][RS] half-step positions
  static constexpr int OFF_P = OFF_XP + 6 * RS;     // [ZS] P of zone plane p
  static constexpr int OFF_M = OFF_P + ZS;          // [ZS] m of zone plane p
  static constexpr int OFF_G = OFF_M + ZS;          // [9][ZS] g_x, g_y, g_z
  static constexpr int OFF_UH = OFF_G + 9 * ZS;     // [2 planes][3][ZS] u_half
  static constexpr int OFF_PS = OFF_UH + 6 * ZS;    // [2][ZS] psi of x-low, y-low faces
  static constexpr int OFF_RED = OFF_PS + 2 * ZS;   // [32] block dt reduction
  static constexpr int OFF_BAR = OFF_RED + 32;      // 3 mbarriers
  static constexpr int TOTAL = OFF_BAR + 4;
  static constexpr size_t BYTES = sizeof(double) * TOTAL;
  static_assert(BXN >= TX + 3, "TMA box too narrow");
  static_assert(BYN <= 256 && BXN <= 256, "TMA box limit");
};

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
               "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred P1;\n"
      "LAB_WAIT:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
      "@!P1 bra LAB_WAIT;\n"
      "}\n" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void tma_load_3d(double *dst, const CUtensorMap *map, uint64_t *bar,
                                            int c0, int c1, int c2) {
  asm volatile(
      "cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%2, %3, %4}], [%5];" ::"r"(smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(c2), "r"(smem_u32(bar))
      : "memory");
}

__device__ __forceinline__ void flag_error(DevState *st, unsigned bits, int64_t gz) {
  atomicOr(&st->err, bits);
  atomicMin(&st->bad_zone, (unsigned long long)gz);
}

template <int TX, int TY>
__global__ void __launch_bounds__(Tile<TX, TY>::NTHR, 1)
    k_cycle_fused(const __grid_constant__ NodeMaps maps, DomView d, Phys ph, DevState *st,
                  int KZ) {
  using T = Tile<TX, TY>;
  // dynamic shared memory only (no static __shared__ in this kernel), so the window starts
  // 1024-byte aligned and every TMA destination (multiples of 128 B) is aligned
  extern __shared__ __align__(1024) double sm[];
  double *RAW = sm + T::OFF_RAW, *XP = sm + T::OFF_XP, *PS = sm + T::OFF_P, *MS = sm + T::OFF_M;
  double *GX = sm + T::OFF_G, *GY = GX + 3 * T::ZS, *GZ = GY + 3 * T::ZS;
  double *UH = sm + T::OFF_UH, *PSX = sm + T::OFF_PS, *PSY = PSX + T::ZS;
  uint64_t *bar = reinterpret_cast<uint64_t *>(sm + T::OFF_BAR);

  const int t = threadIdx.x;
  const int i0 = blockIdx.x * TX, j0 = blockIdx.y * TY;
  const int k0 = blockIdx.z * KZ;
  const int k1 = min(k0 + KZ, d.n[2]);
  const int n0 = d.n[0], n1 = d.n[1], n2 = d.n[2];
  const bool active = t < T::NZT;
  const int tx = t % T::TXT, ty = t / T::TXT;
  const int li = i0 - 1 + tx, lj = j0 - 1 + ty;  // local zone / node index of this thread

  if ((st->halted | st->done) != 0u) {  // no-op cycle: carry the state over to the next parity
    for (int p = k0; p <= k1; ++p) {
      if (!active || tx < 1 || ty < 1) continue;
      const bool wn = li <= n0 && lj <= n1 && (li < i0 + TX || li == n0) &&
                      (lj < j0 + TY || lj == n1) && (p < k1 || p == n2);
      if (wn) {
        const int64_t id = d.nid(li, lj, p);
        d.xn[id] = d.x[id]; d.yn[id] = d.y[id]; d.zn[id] = d.z[id];
        d.un[id] = d.u[id]; d.vn[id] = d.v[id]; d.wn[id] = d.w[id];
      }
      if (p < k1 && tx <= TX && ty <= TY && li < n0 && lj < n1) {
        const int64_t z = d.zid(li, lj, p);
        d.en[z] = d.e[z];
      }
    }
    return;
  }

  const double dt = st->dt;
  const double hh = 0.5 * dt;
  const int q0 = k0 - 1;  // first node plane of the chunk

  // TMA producer: node plane q -> slot (q-q0)%3, 6 fields, one mbarrier per slot.
  auto issue = [&](int q) {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    const int u = q - q0, s = u % 3;
    double *dst = RAW + s * 6 * T::RS;
    mbar_expect_tx(&bar[s], 6u * T::NN * sizeof(double));
#pragma unroll
    for (int f = 0; f < 6; ++f) tma_load_3d(dst + f * T::RS, &maps.m[f], &bar[s], i0, j0, q + 1);
  };
  auto wait_plane = [&](int q) {
    const int u = q - q0;
    mbar_wait(&bar[u % 3], (uint32_t)((u / 3) & 1));
  };
  auto raw = [&](int q) { return RAW + ((q - q0) % 3) * 6 * T::RS; };
  // X stage: half-step positions of node plane q into XP slot q&1.
  auto form_xp = [&](int q) {
    const double *R = raw(q);
    double *X = XP + (q & 1) * 3 * T::RS;
    for (int n = t; n < T::NN; n += T::NTHR) {
      X[n] = R[n] + hh * R[3 * T::RS + n];
      X[T::RS + n] = R[T::RS + n] + hh * R[4 * T::RS + n];
      X[2 * T::RS + n] = R[2 * T::RS + n] + hh * R[5 * T::RS + n];
    }
  };

  if (t == 0) {
    if (smem_u32(sm) & 127u) __trap();  // TMA destinations must be 128-byte aligned
    for (int s = 0; s < 3; ++s) mbar_init(&bar[s], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    issue(q0);
    issue(q0 + 1);
  }
  __syncthreads();

  // carried per-thread state
  double P_prev = 0.0, im_prev = 0.0, e_prev = 0.0;
  double axp = 0, ayp = 0, azp = 0, bxp = 0, byp = 0, bzp = 0;  // x-low / y-low faces, plane p-1
  double Sx = 0, Sy = 0, Sz = 0, Msum_prev = 0;                   // in-plane node sums, plane p-1
  double psi_zlow = 0.0;
  double dt2min = INFINITY;

  const bool zone_in_storage = active && li <= n0 && lj <= n1;
  const int64_t gxz = d.lo[0] + li, gyz = d.lo[1] + lj;
  const bool zone_xy_exists = zone_in_storage && gxz >= 0 && gxz < d.N[0] && gyz >= 0 &&
                              gyz < d.N[1];
  const bool node_xy = active && tx >= 1 && ty >= 1 && li <= n0 && lj <= n1;
  const bool node_write_xy = node_xy && (li < i0 + TX || li == n0) && (lj < j0 + TY || lj == n1);
  const bool zone_owned_xy = active && tx >= 1 && ty >= 1 && tx <= TX && ty <= TY && li < n0 &&
                             lj < n1;
  const int nidx = ty * T::BXN + tx;  // this thread's node in the node box
  const uint32_t rm = ph.reflect_mask;
  const bool wall_x = (gxz == 0 && (rm & 1u)) || (gxz == d.N[0] && (rm & 2u));
  const bool wall_y = (gyz == 0 && (rm & 4u)) || (gyz == d.N[1] && (rm & 8u));
  const int64_t zrow = (int64_t)(lj + 1) * d.zsx + (li + 1);  // zone id minus plane offset
  const int64_t nrow = (int64_t)(lj + 1) * d.nsx + (li + 1);  // node id minus plane offset

  // zone mass / energy of plane q (prefetched one plane ahead into registers)
  auto load_me = [&](int q, double &m, double &e) {
    m = 0.0;
    e = 0.0;
    const int64_t gz = d.lo[2] + q;
    if (zone_xy_exists && gz >= 0 && gz < d.N[2]) {
      const int64_t zid = (int64_t)(q + 1) * d.zsxy + zrow;
      m = d.m[zid];
      e = d.e[zid];
    }
  };
  double m_nx, e_nx;
  load_me(q0, m_nx, e_nx);

  wait_plane(q0);
  form_xp(q0);

  for (int p = k0 - 1; p <= k1; ++p) {
    // ---------------------------------------------------------------- X
    if (t == 0 && p + 2 <= k1 + 1) issue(p + 2);  // slot of plane p-1, free since step p-1
    const double m = m_nx, e = e_nx;
    if (p + 1 <= k1) load_me(p + 1, m_nx, e_nx);
    wait_plane(p + 1);
    form_xp(p + 1);
    if (active) MS[t] = m;
    __syncthreads();
    // ---------------------------------------------------------------- Z
    const double *Ra = raw(p), *Rb = raw(p + 1);
    double P = 0.0, im = 0.0;
    double ax0 = 0, ay0 = 0, az0 = 0, bx0 = 0, by0 = 0, bz0 = 0, cx0 = 0, cy0 = 0, cz0 = 0;
    if (active) {
      const double *Xa = XP + (p & 1) * 3 * T::RS, *Xb = XP + ((p + 1) & 1) * 3 * T::RS;
      double X[8], Y[8], Z[8];
#pragma unroll
      for (int l = 0; l < 8; ++l) {
        const double *S = (l >> 2) ? Xb : Xa;
        const int n = nidx + ((l >> 1) & 1) * T::BXN + (l & 1);
        X[l] = S[n];
        Y[l] = S[T::RS + n];
        Z[l] = S[2 * T::RS + n];
      }
      double fx[6], fy[6], fz[6];
#pragma unroll
      for (int a = 0; a < 2; ++a) HYDRO_FACE(X, Y, Z, a + 6, a, a + 4, a + 2, fx[a], fy[a], fz[a]);
#pragma unroll
      for (int b = 0; b < 2; ++b)
        HYDRO_FACE(X, Y, Z, 5 + 2 * b, 2 * b, 1 + 2 * b, 2 * b + 4, fx[2 + b], fy[2 + b], fz[2 + b]);
#pragma unroll
      for (int c = 0; c < 2; ++c)
        HYDRO_FACE(X, Y, Z, 3 + 4 * c, 4 * c, 2 + 4 * c, 1 + 4 * c, fx[4 + c], fy[4 + c], fz[4 + c]);
      double V8 = 0.0, DV8 = 0.0;
#pragma unroll
      for (int l = 0; l < 8; ++l) {
        const int a = l & 1, b = (l >> 1) & 1, c = (l >> 2) & 1;
        const double sx = (a ? fx[1] : -fx[0]) + (b ? fx[3] : -fx[2]) + (c ? fx[5] : -fx[4]);
        const double sy = (a ? fy[1] : -fy[0]) + (b ? fy[3] : -fy[2]) + (c ? fy[5] : -fy[4]);
        const double sz = (a ? fz[1] : -fz[0]) + (b ? fz[3] : -fz[2]) + (c ? fz[5] : -fz[4]);
        if (l > 0) V8 += (X[l] - X[0]) * sx + (Y[l] - Y[0]) * sy + (Z[l] - Z[0]) * sz;
        const double *Us = (c ? Rb : Ra) + 3 * T::RS;
        const int n = nidx + b * T::BXN + a;
        DV8 += Us[n] * sx + Us[T::RS + n] * sy + Us[2 * T::RS + n] * sz;
      }
      const double V = V8 * (1.0 / 24.0);
      const double DV = 0.125 * DV8;
      double a2 = 0.0;
#pragma unroll
      for (int f = 0; f < 6; ++f) a2 = fmax(a2, fx[f] * fx[f] + fy[f] * fy[f] + fz[f] * fz[f]);
      // S2-S4 and S6 with branch-free reciprocals; L = 2V/sqrt(a2) enters only through
      // s = L(-D) = -2 DV/sqrt(a2) and through dt^2.
      const double iV = frcp(V);
      im = frcp(m);
      const double rho = m * iV;
      const double epos = fmax(e, 0.0);
      const double ep = e - (hh * (ph.gm1 * rho) * epos) * DV * im;
      const double eppos = fmax(ep, 0.0);
      const double pr = ph.gm1 * rho * eppos;
      const double c2 = ph.ggm1 * eppos;
      const double c = fsqrt(c2);
      double qr = 0.0;
      if (DV < 0.0) {
        const double s = -2.0 * DV * frsqrt(a2);
        qr = s * (ph.q_quad * s + ph.q_lin * c);
      }
      const double sig2a = (c2 + 2.0 * qr) * a2;
      const double V2 = V * V;
      // denominators below 1e-290 mean dt_z^2 > 1e270 V^2: never the minimum, taken as +inf
      const double DV2 = DV * DV;
      const double dtc2 = sig2a > 1e-290 ? (4.0 * ph.cfl * ph.cfl) * V2 * frcp(sig2a) : INFINITY;
      const double dtv2 = DV2 > 1e-290 ? (ph.c_vol * ph.c_vol) * V2 * frcp(DV2) : INFINITY;
      const int64_t gz = d.lo[2] + p;
      const bool exists = zone_xy_exists && gz >= 0 && gz < d.N[2];
      if (exists) {
        P = pr + rho * qr;
        if (p >= k0 && p < k1 && zone_owned_xy) {
          const int64_t gzi = (gz * d.N[1] + gyz) * (int64_t)d.N[0] + gxz;
          if (!(V > 0.0)) flag_error(st, ERR_TANGLED, gzi);
          else if (!isfinite(P)) flag_error(st, ERR_NONFINITE, gzi);
          const double dt2 = fmin(dtc2, dtv2);
          if (dt2 == dt2) dt2min = fmin(dt2min, dt2);
        }
      } else {
        im = 0.0;
      }
      ax0 = fx[0]; ay0 = fy[0]; az0 = fz[0];  // x-low face
      bx0 = fx[2]; by0 = fy[2]; bz0 = fz[2];  // y-low face
      cx0 = fx[4]; cy0 = fy[4]; cz0 = fz[4];  // z-low face (node plane p)
      PS[t] = P;
    }
    __syncthreads();
    // ---------------------------------------------------------------- G
    if (active) {
      const double gxw = (tx > 0) ? 0.125 * (PS[t - 1] - P) : 0.0;
      const double gyw = (ty > 0) ? 0.125 * (PS[t - T::TXT] - P) : 0.0;
      const double gzw = 0.125 * (P_prev - P);
      GX[t] = gxw * ax0; GX[T::ZS + t] = gxw * ay0; GX[2 * T::ZS + t] = gxw * az0;
      GY[t] = gyw * bx0; GY[T::ZS + t] = gyw * by0; GY[2 * T::ZS + t] = gyw * bz0;
      GZ[t] = gzw * cx0; GZ[T::ZS + t] = gzw * cy0; GZ[2 * T::ZS + t] = gzw * cz0;
    }
    __syncthreads();
    // ---------------------------------------------------------------- N
    double *UHc = UH + (p & 1) * 3 * T::ZS;
    if (active && tx >= 1 && ty >= 1) {
      const int tn = t - T::TXT;  // zone (tx, ty-1)
      const double Cx = (GX[tn] + GX[t]) + (GY[t - 1] + GY[t]);
      const double Cy = (GX[T::ZS + tn] + GX[T::ZS + t]) + (GY[T::ZS + t - 1] + GY[T::ZS + t]);
      const double Cz = (GX[2 * T::ZS + tn] + GX[2 * T::ZS + t]) +
                        (GY[2 * T::ZS + t - 1] + GY[2 * T::ZS + t]);
      const double Ms = (MS[tn - 1] + MS[tn]) + (MS[t - 1] + MS[t]);
      if (p >= k0 && node_xy) {
        const double Fx = Sx + Cx + ((GZ[tn - 1] + GZ[tn]) + (GZ[t - 1] + GZ[t]));
        const double Fy = Sy + Cy + ((GZ[T::ZS + tn - 1] + GZ[T::ZS + tn]) +
                                     (GZ[T::ZS + t - 1] + GZ[T::ZS + t]));
        const double Fz = Sz + Cz + ((GZ[2 * T::ZS + tn - 1] + GZ[2 * T::ZS + tn]) +
                                     (GZ[2 * T::ZS + t - 1] + GZ[2 * T::ZS + t]));
        const double rinv = 8.0 * frcp(Msum_prev + Ms);
        double axc = Fx * rinv, ayc = Fy * rinv, azc = Fz * rinv;
        const int64_t g2 = d.lo[2] + p;
        if (wall_x) axc = 0.0;
        if (wall_y) ayc = 0.0;
        if ((g2 == 0 && (rm & 16u)) || (g2 == d.N[2] && (rm & 32u))) azc = 0.0;
        const double u = Ra[3 * T::RS + nidx], v = Ra[4 * T::RS + nidx], w = Ra[5 * T::RS + nidx];
        const double un = u + dt * axc, vn = v + dt * ayc, wn = w + dt * azc;
        const double uh = (u + un) * 0.5, vh = (v + vn) * 0.5, wh = (w + wn) * 0.5;
        UHc[t] = uh;
        UHc[T::ZS + t] = vh;
        UHc[2 * T::ZS + t] = wh;
        if (node_write_xy && (p < k1 || p == n2)) {
          const int64_t id = (int64_t)(p + 1) * d.nsxy + nrow;
          d.xn[id] = Ra[nidx] + dt * uh;
          d.yn[id] = Ra[T::RS + nidx] + dt * vh;
          d.zn[id] = Ra[2 * T::RS + nidx] + dt * wh;
          d.un[id] = un;
          d.vn[id] = vn;
          d.wn[id] = wn;
        }
      }
      Sx = Cx; Sy = Cy; Sz = Cz;
      Msum_prev = Ms;
    }
    __syncthreads();
    // ---------------------------------------------------------------- E
    double psi_zhigh = 0.0;
    if (active && p >= k0) {
      const double *UHp = UH + ((p - 1) & 1) * 3 * T::ZS;
      if (p >= k0 + 1) {
        if (tx >= 1 && tx <= TX + 1 && ty >= 1 && ty <= TY) {  // x-low face of zone plane p-1
          const int t2 = t + T::TXT;
          const double sx = (UHp[t] + UHp[t2]) + (UHc[t] + UHc[t2]);
          const double sy = (UHp[T::ZS + t] + UHp[T::ZS + t2]) + (UHc[T::ZS + t] + UHc[T::ZS + t2]);
          const double sz = (UHp[2 * T::ZS + t] + UHp[2 * T::ZS + t2]) +
                            (UHc[2 * T::ZS + t] + UHc[2 * T::ZS + t2]);
          PSX[t] = axp * sx + ayp * sy + azp * sz;
        }
        if (tx >= 1 && tx <= TX && ty >= 1 && ty <= TY + 1) {  // y-low face of zone plane p-1
          const int t2 = t + 1;
          const double sx = (UHp[t] + UHp[t2]) + (UHc[t] + UHc[t2]);
          const double sy = (UHp[T::ZS + t] + UHp[T::ZS + t2]) + (UHc[T::ZS + t] + UHc[T::ZS + t2]);
          const double sz = (UHp[2 * T::ZS + t] + UHp[2 * T::ZS + t2]) +
                            (UHc[2 * T::ZS + t] + UHc[2 * T::ZS + t2]);
          PSY[t] = bxp * sx + byp * sy + bzp * sz;
        }
      }
      if (tx >= 1 && tx <= TX && ty >= 1 && ty <= TY) {  // z-face at node plane p
        const int t1 = t + 1, t2 = t + T::TXT, t3 = t + T::TXT + 1;
        const double sx = (UHc[t] + UHc[t1]) + (UHc[t2] + UHc[t3]);
        const double sy = (UHc[T::ZS + t] + UHc[T::ZS + t1]) + (UHc[T::ZS + t2] + UHc[T::ZS + t3]);
        const double sz = (UHc[2 * T::ZS + t] + UHc[2 * T::ZS + t1]) +
                          (UHc[2 * T::ZS + t2] + UHc[2 * T::ZS + t3]);
        psi_zhigh = cx0 * sx + cy0 * sy + cz0 * sz;
      }
    }
    __syncthreads();
    if (active && p >= k0 + 1 && zone_owned_xy) {
      const double Wk = 0.125 * P_prev *
                        (((PSX[t + 1] - PSX[t]) + (PSY[t + T::TXT] - PSY[t])) + (psi_zhigh - psi_zlow));
      d.en[(int64_t)p * d.zsxy + zrow] = e_prev - dt * Wk * im_prev;
    }
    psi_zlow = psi_zhigh;
    P_prev = P;
    im_prev = im;
    e_prev = e;
    axp = ax0; ayp = ay0; azp = az0;
    bxp = bx0; byp = by0; bzp = bz0;
  }
  // S9 (block part): dt = sqrt(min dt^2), one atomicMin per block.
  block_min_dt_smem(sqrt(dt2min), &st->dtz_acc, sm + T::OFF_RED);
}

constexpr int FTX = 32, FTY = 12;

// z-chunk length: minimise (waves of blocks) x (planes per block incl. the 2 warm-up planes).
int choose_kz(int tiles, int n2, int sms) {
  int best = n2, best_cost = 1 << 30;
  for (int kz = 4; kz <= n2; ++kz) {
    const int chunks = (n2 + kz - 1) / kz;
    const int waves = (tiles * chunks + sms - 1) / sms;
    const int cost = waves * (kz + 2);
    if (cost < best_cost) {
      best_cost = cost;
      best = kz;
    }
  }
  return std::min(best, n2);
}

}  // namespace

size_t fused_smem_bytes() { return Tile<FTX, FTY>::BYTES; }
int fused_box_y() { return Tile<FTX, FTY>::BYN; }

void launch_cycle_fused(const DomView &d, const NodeMaps &maps, const Phys &ph, DevState *st,
                        cudaStream_t s) {
  using T = Tile<FTX, FTY>;
  static int sms = 0;
  if (!sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaFuncSetAttribute(k_cycle_fused<FTX, FTY>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         (int)T::BYTES);
  }
  const int tx = (d.n[0] + FTX - 1) / FTX, ty = (d.n[1] + FTY - 1) / FTY;
  const int KZ = choose_kz(tx * ty, d.n[2], sms);
  dim3 grid(tx, ty, (d.n[2] + KZ - 1) / KZ);
  k_cycle_fused<FTX, FTY><<<grid, T::NTHR, T::BYTES, s>>>(maps, d, ph, st, KZ);
}

}  // namespace hydro
