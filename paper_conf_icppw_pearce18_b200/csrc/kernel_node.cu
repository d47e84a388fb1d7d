// kernel_node.cu -- node/energy stage of the two-kernel cycle (S5 face form, S7, S8).
//
// Same 2.5-D blocking as kernel_fused.cu (TMA node-plane ring, one-zone ring per tile), but the
// zone physics is not recomputed: P of every zone of the tile and its ring comes from HBM, written
// by the zone stage (kernel_zone.cu).  Per plane the ring zones only form their three low face
// vectors (x-low, y-low, z-low) from the half-step positions; then
//   G  g_f = (P_below - P_above) A_f / 4 per face (the face form of S5),
//   N  node plane p: F = sum of 12 incident g_f, m_p, a, walls, u', u_half, x' (S7),
//   E  zone plane p-1: W = P sum_l B_l.u_half_l in face form, e' = e - dt W / m (S8).
#include <algorithm>
#include <cmath>

#include "fastmath.cuh"
#include "kernels.h"
#include "tma.cuh"
#include "zone_physics.cuh"

namespace hydro {

namespace {

template <int TX, int TY>
struct NTile {
  static constexpr int TXT = TX + 2, TYT = TY + 2;  // zone-stage tile (owned + 1 ring)
  static constexpr int NZT = TXT * TYT;
  static constexpr int NTHR = (NZT + 31) / 32 * 32;
  static constexpr int ZS = NTHR;                   // zone-tile slots
  static constexpr int BXN = FUSED_BOX_X, BYN = TY + 3;  // TMA node box (x padded to 16 B)
  static constexpr int NN = BXN * BYN;
  static constexpr int RS = (NN + 15) / 16 * 16;    // stride of one node array (128 B aligned)
  // shared-memory layout, in doubles; every array is SoA so a warp's LDS.64 is conflict-free
  static constexpr int OFF_RAW = 0;                 // [3 slots][6 fields][RS] x,y,z,u,v,w (TMA)
  static constexpr int OFF_XP = OFF_RAW + 18 * RS;  // [2 planes][3][RS] half-step positions
  static constexpr int OFF_G = OFF_XP + 6 * RS;     // [3 vectors][3][ZS] g_x, g_y, g_z
  static constexpr int OFF_UH = OFF_G + 9 * ZS;     // [2 planes][3][ZS] u_half
  static constexpr int OFF_P = OFF_UH + 6 * ZS;     // [ZS] P of zone plane p
  static constexpr int OFF_M = OFF_P + ZS;          // [ZS] m of zone plane p
  static constexpr int OFF_PS = OFF_M + ZS;         // [2][ZS] psi of x-low, y-low faces
  static constexpr int OFF_RED = OFF_PS + 2 * ZS;   // [32] block dt reduction
  static constexpr int OFF_BAR = OFF_RED + 32;      // 3 mbarriers
  static constexpr int TOTAL = OFF_BAR + 4;
  static constexpr size_t BYTES = sizeof(double) * TOTAL;
  static_assert(BXN >= TX + 3, "TMA box too narrow");
  static_assert(BYN <= 256 && BXN <= 256, "TMA box limit");
  static_assert(BYTES <= 227 * 1024, "shared memory");
};

template <int TX, int TY>
__global__ void __launch_bounds__(NTile<TX, TY>::NTHR, 1)
    k_node_energy(const __grid_constant__ NodeMaps maps, DomView d, Phys ph, DevState *st,
                  int KZ) {
  using T = NTile<TX, TY>;
  // dynamic shared memory only (no static __shared__ in this kernel), so the window starts
  // 1024-byte aligned and every TMA destination (multiples of 128 B) is aligned
  extern __shared__ __align__(1024) double sm[];
  double *RAW = sm + T::OFF_RAW, *XP = sm + T::OFF_XP, *PS = sm + T::OFF_P, *MS = sm + T::OFF_M;
  double *G = sm + T::OFF_G;  // g_x at [0, 3ZS), g_y at [3ZS, 6ZS), g_z at [6ZS, 9ZS)
  double *UH = sm + T::OFF_UH, *PSX = sm + T::OFF_PS, *PSY = PSX + T::ZS;
  uint64_t *bar = reinterpret_cast<uint64_t *>(sm + T::OFF_BAR);

  const int t = threadIdx.x;
  const int i0 = blockIdx.x * TX, j0 = blockIdx.y * TY;
  const int k0 = blockIdx.z * KZ;
  const int k1 = min(k0 + KZ, d.n[2]);
  const int n0 = d.n[0], n1 = d.n[1], n2 = d.n[2];
  const bool active = t < T::NZT;
  const int tc = active ? t : T::NZT - 1;  // padding lanes shadow the last zone (never store)
  const int tx = tc % T::TXT, ty = tc / T::TXT;
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
      X[n] = fma(hh, R[3 * T::RS + n], R[n]);
      X[T::RS + n] = fma(hh, R[4 * T::RS + n], R[T::RS + n]);
      X[2 * T::RS + n] = fma(hh, R[5 * T::RS + n], R[2 * T::RS + n]);
    }
  };
  // 3-vectors in SoA shared arrays: component k of item i at base[k*stride + i]
  auto st3 = [](double *b, int stride, int i, double x, double y, double z) {
    b[i] = x; b[stride + i] = y; b[2 * stride + i] = z;
  };
  auto ld3 = [](const double *b, int stride, int i, double &x, double &y, double &z) {
    x = b[i]; y = b[stride + i]; z = b[2 * stride + i];
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

  const int64_t gxz = d.lo[0] + li, gyz = d.lo[1] + lj;
  const bool zone_xy_exists = active && li <= n0 && lj <= n1 && gxz >= 0 && gxz < d.N[0] &&
                              gyz >= 0 && gyz < d.N[1];
  const bool node_xy = active && tx >= 1 && ty >= 1 && li <= n0 && lj <= n1;
  const bool node_write_xy = node_xy && (li < i0 + TX || li == n0) && (lj < j0 + TY || lj == n1);
  const bool zone_owned_xy = active && tx >= 1 && ty >= 1 && tx <= TX && ty <= TY && li < n0 &&
                             lj < n1;
  const bool ex_x = active && tx >= 1 && tx <= TX + 1 && ty >= 1 && ty <= TY;
  const bool ex_y = active && tx >= 1 && tx <= TX && ty >= 1 && ty <= TY + 1;
  const bool ex_z = active && tx >= 1 && tx <= TX && ty >= 1 && ty <= TY;
  const int nidx = ty * T::BXN + tx;  // this thread's node in the node box
  const uint32_t rm = ph.reflect_mask;
  const bool wall_x = (gxz == 0 && (rm & 1u)) || (gxz == d.N[0] && (rm & 2u));
  const bool wall_y = (gyz == 0 && (rm & 4u)) || (gyz == d.N[1] && (rm & 8u));
  const int64_t zsxy = d.zsxy, nsxy = d.nsxy;
  const double *mg = d.m + (int64_t)(lj + 1) * d.zsx + (li + 1);  // + (q+1)*zsxy
  const double *eg = d.e + (int64_t)(lj + 1) * d.zsx + (li + 1);
  double *eng = d.en + (int64_t)(lj + 1) * d.zsx + (li + 1);
  const int64_t nrow = (int64_t)(lj + 1) * d.nsx + (li + 1);
  const int64_t gz_lo = -d.lo[2], gz_hi = d.N[2] - d.lo[2];  // plane q exists iff in [lo, hi)

  // zone mass / energy of plane q (prefetched one plane ahead into registers)
  const double *Pg = d.P + (int64_t)(lj + 1) * d.zsx + (li + 1);
  double m_nx = 0.0, e_nx = 0.0, P_nx = 0.0;
  if (zone_xy_exists && q0 >= gz_lo && q0 < gz_hi) {
    m_nx = mg[(int64_t)(q0 + 1) * zsxy];
    e_nx = eg[(int64_t)(q0 + 1) * zsxy];
    P_nx = Pg[(int64_t)(q0 + 1) * zsxy];
  }

  wait_plane(q0);
  form_xp(q0);

  for (int p = k0 - 1; p <= k1; ++p) {
    // ---------------------------------------------------------------- X
    if (t == 0 && p + 2 <= k1 + 1) issue(p + 2);  // slot of plane p-1, free since step p-1
    const double m = m_nx, e = e_nx, P_cur = P_nx;
    const bool exists = zone_xy_exists && p >= gz_lo && p < gz_hi;
    {
      const int q = p + 1;
      const bool ok = q <= k1 && zone_xy_exists && q >= gz_lo && q < gz_hi;
      m_nx = ok ? mg[(int64_t)(q + 1) * zsxy] : 0.0;
      e_nx = ok ? eg[(int64_t)(q + 1) * zsxy] : 0.0;
      P_nx = ok ? Pg[(int64_t)(q + 1) * zsxy] : 0.0;
    }
    wait_plane(p + 1);
    form_xp(p + 1);
    MS[t] = m;
    __syncthreads();
    // ---------------------------------------------------------------- Z (faces only)
    const double *Ra = raw(p);
    const double P = P_cur;
    const double im = exists ? frcp(m) : 0.0;
    double ax0, ay0, az0, bx0, by0, bz0, cx0, cy0, cz0;
    {
      const double *Xa = XP + (p & 1) * 3 * T::RS, *Xb = XP + ((p + 1) & 1) * 3 * T::RS;
      double X[8], Y[8], Z[8];
#pragma unroll
      for (int l = 0; l < 7; ++l) {  // corners 0..6 (corner 7 is on no low face)
        const int n = nidx + ((l >> 1) & 1) * T::BXN + (l & 1);
        ld3((l >> 2) ? Xb : Xa, T::RS, n, X[l], Y[l], Z[l]);
      }
      HYDRO_FACE(X, Y, Z, 6, 0, 4, 2, ax0, ay0, az0);  // x-low (AX_0)
      HYDRO_FACE(X, Y, Z, 5, 0, 1, 4, bx0, by0, bz0);  // y-low (AY_0)
      HYDRO_FACE(X, Y, Z, 3, 0, 2, 1, cx0, cy0, cz0);  // z-low (AZ_0, node plane p)
      PS[t] = P;
    }
    __syncthreads();
    // ---------------------------------------------------------------- G
    {
      const double gxw = (tx > 0) ? 0.125 * (PS[tc - 1] - P) : 0.0;
      const double gyw = (ty > 0) ? 0.125 * (PS[tc - T::TXT] - P) : 0.0;
      const double gzw = 0.125 * (P_prev - P);
      st3(G, T::ZS, t, gxw * ax0, gxw * ay0, gxw * az0);
      st3(G + 3 * T::ZS, T::ZS, t, gyw * bx0, gyw * by0, gyw * bz0);
      st3(G + 6 * T::ZS, T::ZS, t, gzw * cx0, gzw * cy0, gzw * cz0);
    }
    __syncthreads();
    // ---------------------------------------------------------------- N
    double *UHc = UH + (p & 1) * 3 * T::ZS;
    const double *GXs = G, *GYs = G + 3 * T::ZS, *GZs = G + 6 * T::ZS;
    if (node_xy) {
      const int tn = tc - T::TXT;  // zone (tx, ty-1)
      double ax_, ay_, az_, bx_, by_, bz_, cx_, cy_, cz_, dx_, dy_, dz_;
      ld3(GXs, T::ZS, tn, ax_, ay_, az_);
      ld3(GXs, T::ZS, tc, bx_, by_, bz_);
      ld3(GYs, T::ZS, tc - 1, cx_, cy_, cz_);
      ld3(GYs, T::ZS, tc, dx_, dy_, dz_);
      const double Cx = (ax_ + bx_) + (cx_ + dx_);
      const double Cy = (ay_ + by_) + (cy_ + dy_);
      const double Cz = (az_ + bz_) + (cz_ + dz_);
      const double Ms = (MS[tn - 1] + MS[tn]) + (MS[tc - 1] + MS[tc]);
      if (p >= k0) {
        ld3(GZs, T::ZS, tn - 1, ax_, ay_, az_);
        ld3(GZs, T::ZS, tn, bx_, by_, bz_);
        ld3(GZs, T::ZS, tc - 1, cx_, cy_, cz_);
        ld3(GZs, T::ZS, tc, dx_, dy_, dz_);
        const double Fx = Sx + Cx + ((ax_ + bx_) + (cx_ + dx_));
        const double Fy = Sy + Cy + ((ay_ + by_) + (cy_ + dy_));
        const double Fz = Sz + Cz + ((az_ + bz_) + (cz_ + dz_));
        const double rinv = 8.0 * frcp(Msum_prev + Ms);
        const int64_t g2 = d.lo[2] + p;
        const bool wall_z = (g2 == 0 && (rm & 16u)) || (g2 == d.N[2] && (rm & 32u));
        const double axc = wall_x ? 0.0 : Fx * rinv;
        const double ayc = wall_y ? 0.0 : Fy * rinv;
        const double azc = wall_z ? 0.0 : Fz * rinv;
        const double u = Ra[3 * T::RS + nidx], v = Ra[4 * T::RS + nidx], w = Ra[5 * T::RS + nidx];
        const double un = u + dt * axc, vn = v + dt * ayc, wn = w + dt * azc;
        const double uh = (u + un) * 0.5, vh = (v + vn) * 0.5, wh = (w + wn) * 0.5;
        st3(UHc, T::ZS, tc, uh, vh, wh);
        if (node_write_xy && (p < k1 || p == n2)) {
          const int64_t id = (int64_t)(p + 1) * nsxy + nrow;
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
    if (p >= k0) {
      const double *UHp = UH + ((p - 1) & 1) * 3 * T::ZS;
      double a0, a1, a2_, b0, b1, b2, c0, c1, c2_, e0, e1, e2;
      if (p >= k0 + 1) {
        if (ex_x) {  // x-low face of zone plane p-1: nodes (tx, ty..ty+1) at planes p-1, p
          const int t2 = tc + T::TXT;
          ld3(UHp, T::ZS, tc, a0, a1, a2_);
          ld3(UHp, T::ZS, t2, b0, b1, b2);
          ld3(UHc, T::ZS, tc, c0, c1, c2_);
          ld3(UHc, T::ZS, t2, e0, e1, e2);
          PSX[t] = axp * ((a0 + b0) + (c0 + e0)) + ayp * ((a1 + b1) + (c1 + e1)) +
                   azp * ((a2_ + b2) + (c2_ + e2));
        }
        if (ex_y) {  // y-low face of zone plane p-1: nodes (tx..tx+1, ty) at planes p-1, p
          const int t2 = tc + 1;
          ld3(UHp, T::ZS, tc, a0, a1, a2_);
          ld3(UHp, T::ZS, t2, b0, b1, b2);
          ld3(UHc, T::ZS, tc, c0, c1, c2_);
          ld3(UHc, T::ZS, t2, e0, e1, e2);
          PSY[t] = bxp * ((a0 + b0) + (c0 + e0)) + byp * ((a1 + b1) + (c1 + e1)) +
                   bzp * ((a2_ + b2) + (c2_ + e2));
        }
      }
      if (ex_z) {  // z-face at node plane p: nodes (tx..tx+1, ty..ty+1)
        ld3(UHc, T::ZS, tc, a0, a1, a2_);
        ld3(UHc, T::ZS, tc + 1, b0, b1, b2);
        ld3(UHc, T::ZS, tc + T::TXT, c0, c1, c2_);
        ld3(UHc, T::ZS, tc + T::TXT + 1, e0, e1, e2);
        psi_zhigh = cx0 * ((a0 + b0) + (c0 + e0)) + cy0 * ((a1 + b1) + (c1 + e1)) +
                    cz0 * ((a2_ + b2) + (c2_ + e2));
      }
    }
    __syncthreads();
    if (p >= k0 + 1 && zone_owned_xy) {
      const double Wk = 0.125 * P_prev *
                        (((PSX[t + 1] - PSX[t]) + (PSY[t + T::TXT] - PSY[t])) + (psi_zhigh - psi_zlow));
      eng[(int64_t)p * zsxy] = e_prev - dt * Wk * im_prev;
    }
    psi_zlow = psi_zhigh;
    P_prev = P;
    im_prev = im;
    e_prev = e;
    axp = ax0; ayp = ay0; azp = az0;
    bxp = bx0; byp = by0; bzp = bz0;
  }
}

constexpr int NTX = 32, NTY = 12;

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

int node_box_y() { return NTile<NTX, NTY>::BYN; }

void launch_node_energy(const DomView &d, const NodeMaps &maps, const Phys &ph, DevState *st,
                        cudaStream_t s) {
  using T = NTile<NTX, NTY>;
  static int sms = 0;
  if (!sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaFuncSetAttribute(k_node_energy<NTX, NTY>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         (int)T::BYTES);
  }
  const int tx = (d.n[0] + NTX - 1) / NTX, ty = (d.n[1] + NTY - 1) / NTY;
  const int KZ = choose_kz(tx * ty, d.n[2], sms);
  dim3 grid(tx, ty, (d.n[2] + KZ - 1) / KZ);
  k_node_energy<NTX, NTY><<<grid, T::NTHR, T::BYTES, s>>>(maps, d, ph, st, KZ);
}

}  // namespace hydro
