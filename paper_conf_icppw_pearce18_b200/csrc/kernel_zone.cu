// kernel_zone.cu -- zone stage of the two-kernel cycle (S1-S4, S6): P and dt_z for every zone.
//
// Every zone of the domain and its ghost ring (local [-1, n] per axis) is computed exactly once:
// half-step positions x_p = x + dt/2 u (S1), face and corner vectors, V, DV (S2), the energy
// predictor and EOS (S3), the artificial viscosity and P = p + q (S4), and dt_z (S6, owned zones
// only, reduced per block and combined with one atomicMin).  P is written to HBM (8 B/zone) for
// the node/energy kernel (kernel_cycle.cu).  A 32x8 block marches its share of z-columns; node
// planes stream in by TMA into a 5-slot ring three planes ahead of use, x_p is formed once per
// node into a 4-slot ring ordered by per-slot mbarriers (HYDRO_ZONE_XPBAR; the older variant
// orders a 3-slot ring with one __syncthreads per plane).  No redundant compute: this is the
// point of the split versus the one-kernel variant (k_cycle<..., FUSED>), which recomputes a
// zone ring per tile.
#include <algorithm>
#include <cmath>
#include <cstdlib>

#include "fastmath.cuh"
#include "kernels.h"
#include "tma.cuh"
#include "zone_physics.cuh"

namespace hydro {

namespace {

#ifndef HYDRO_ZONE_MINB
#define HYDRO_ZONE_MINB 2
#endif
#ifndef HYDRO_ZONE_BY
#define HYDRO_ZONE_BY 8
#endif
constexpr int ZBX = 32, ZBY = HYDRO_ZONE_BY;           // zones per block (x, y)
constexpr int ZNX = ZONE_BOX_X, ZNY = ZBY + 1;         // TMA node box (x padded to 16 B)
constexpr int ZNN = ZNX * ZNY;
constexpr int ZRS = (ZNN + 15) / 16 * 16;              // stride of one node array (128 B)
// HYDRO_ZONE_XPBAR (default 1): the x_p ring is ordered by per-slot mbarriers (every thread
// arrives after forming its share of plane q, a thread waits for plane p+1 only before it
// computes zone plane p) instead of one __syncthreads per plane, so a thread may run up to one
// plane ahead of the slowest; that needs 4 x_p slots and a 5-slot TMA ring (a slot is refilled
// only once every thread has finished the zone plane that last read it).
#ifndef HYDRO_ZONE_XPBAR
#define HYDRO_ZONE_XPBAR 1
#endif
#if HYDRO_ZONE_XPBAR
constexpr int ZRING = 5;                               // TMA ring: planes issued 3 ahead
constexpr int ZXP = 4;                                 // x_p ring
#else
constexpr int ZRING = 4;                               // TMA ring: planes issued 3 ahead
constexpr int ZXP = 3;
#endif
constexpr int ZOFF_RAW = 0;                            // [ZRING slots][6 fields][ZRS]
constexpr int ZOFF_XP = ZOFF_RAW + ZRING * 6 * ZRS;    // [ZXP slots][3][ZRS]
constexpr int ZOFF_RED = ZOFF_XP + ZXP * 3 * ZRS;      // [32]
constexpr int ZOFF_BAR = ZOFF_RED + 32;                // ZRING + ZXP mbarriers
constexpr int ZTOTAL = ZOFF_BAR + ZRING + ZXP;
constexpr size_t ZBYTES = ZTOTAL * sizeof(double);
static_assert(ZNX >= ZBX + 2, "zone-kernel TMA box too narrow (33 nodes + 1 alignment shift)");

// Work split (persistent, SM-count-sized grid).  The zone columns (32x8 tiles, tcols along x,
// all planes [zlo.z, zhi.z) along z) are linearised column-major into W = ncols * nplanes units;
// CTA b of G takes the contiguous range [b W / G, (b+1) W / G) and marches it as one or two
// column segments (a range may cross a column boundary), so every CTA does the same number of
// planes (plus one pipeline warm-up plane per segment) and the grid is exactly one wave.
// GROUP: the units of ALL domains of this GPU are concatenated (ZoneTask table, u0 = prefix), so
// one launch covers every domain and small domains share the SMs instead of each running a
// short, tail-dominated grid.  sched_kz > 0 (single domain only) selects the chunked schedule
// instead (CTA b = column b % ncols, chunk b / ncols of sched_kz planes), kept for A/B.
template <bool GROUP>
__global__ void __launch_bounds__(ZBX *ZBY, HYDRO_ZONE_MINB)
    k_zone_stage(const __grid_constant__ NodeMaps maps1, const __grid_constant__ DomView d1,
                 const __grid_constant__ ZoneTask task1, const DomView *views,
                 const NodeMaps *mapsg, const ZoneTask *tasks, int64_t Wtot, int sched_kz,
                 Phys ph, DevState *st) {
  extern __shared__ __align__(1024) double sm[];
  double *RAW = sm + ZOFF_RAW, *XP = sm + ZOFF_XP;
  uint64_t *bar = reinterpret_cast<uint64_t *>(sm + ZOFF_BAR);
  uint64_t *xbar = bar + ZRING;  // x_p ring (HYDRO_ZONE_XPBAR)
  pdl_wait_and_trigger();
  if ((st->halted | st->done) != 0u) return;

  const int t = threadIdx.x;
  const int tx = t % ZBX, ty = t / ZBX;
  int64_t r0, r1;
  if (!GROUP && sched_kz > 0) {
    const int nplanes = task1.zhi[2] - task1.zlo[2];
    const int ncols = (int)(task1.units / nplanes);
    const int64_t col = blockIdx.x % ncols, ch = blockIdx.x / ncols;  // adjacent CTAs: same z
    r0 = col * nplanes + ch * sched_kz;
    r1 = col * nplanes + min((int)(ch + 1) * sched_kz, nplanes);
  } else {
    r0 = Wtot * blockIdx.x / gridDim.x;
    r1 = Wtot * (blockIdx.x + 1) / gridDim.x;
  }
  const double dt = st->dt;
  const double hh = 0.5 * dt;
  const double hgm1 = hh * ph.gm1;
  const double cfl4 = 4.0 * ph.cfl * ph.cfl, cv2 = ph.c_vol * ph.c_vol;
  double dt2min = INFINITY;
  uint32_t ubase = 0;  // planes this CTA consumed in earlier segments (mbarrier phase continuity)

  if (t == 0) {
    if (smem_u32(sm) & 127u) __trap();
    for (int s = 0; s < ZRING; ++s) mbar_init(&bar[s], 1);
    for (int s = 0; s < ZXP; ++s) mbar_init(&xbar[s], ZBX * ZBY);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();

  int ti = 0;  // current task (GROUP)
  for (int64_t r = r0; r < r1;) {
    if (GROUP)
      while (r >= tasks[ti].u0 + tasks[ti].units) ++ti;
    const ZoneTask &T = GROUP ? tasks[ti] : task1;
    const DomView &d = GROUP ? views[T.slot] : d1;
    const NodeMaps &maps = GROUP ? mapsg[T.slot] : maps1;
    const int n0 = d.n[0], n1 = d.n[1], n2 = d.n[2];
    const int3 zlo = make_int3(T.zlo[0], T.zlo[1], T.zlo[2]);
    const int3 zhi = make_int3(T.zhi[0], T.zhi[1], T.zhi[2]);
    const int tcols = T.tcols;
    const int nplanes = zhi.z - zlo.z;
    const int64_t rl = r - T.u0, rl1 = min(r1, T.u0 + T.units) - T.u0;  // task-local units
    // unit order: z-blocks of zblk planes, within a block column-major (zblk = nplanes: plain
    // column-major), so CTAs that run at the same time march neighbouring columns over the same
    // z range and the node-box rows the columns share are L2 hits
    const int zblk = T.zblk;
    const int64_t bsz = (int64_t)(T.units / nplanes) * zblk;  // units of a full z-block
    const int zb = (int)(rl / bsz);
    const int lb = min(zblk, nplanes - zb * zblk);
    const int64_t rem = rl - (int64_t)zb * bsz;
    const int col = (int)(rem / lb);
    const int zk0 = zlo.z + zb * zblk + (int)(rem - (int64_t)col * lb);
    const int zk1 = zlo.z + zb * zblk + (int)min((int64_t)lb, rl1 - (int64_t)zb * bsz - (int64_t)col * lb);
    r = T.u0 + (int64_t)zb * bsz + (int64_t)col * lb + (zk1 - zlo.z - zb * zblk);
    const int gz_lo = -(int)d.lo[2], gz_hi = d.N[2] - (int)d.lo[2];
    // this segment's zones: local [zi0, zi0+32) x [zj0, zj0+8) x [zk0, zk1) inside [zlo, zhi):
    // the owned zones plus the ghost ring where a neighbour domain exists (ghost zones beyond
    // the physical boundary do not exist; their P stays 0)
    const int zi0 = zlo.x + (col % tcols) * ZBX, zj0 = zlo.y + (col / tcols) * ZBY;
    const int li = zi0 + tx, lj = zj0 + ty;
    // TMA needs a 16-byte-aligned box start in x: start at the even storage column at or below
    // the tile's first node column and shift the shared-memory index by xoff
    const int xoff = (zi0 + 1) & 1, cx = zi0 + 1 - xoff;

    // node plane q (local) -> ring slot (ubase + q - zk0) % ZRING
    auto issue = [&](int q) {
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      const int s = (ubase + (uint32_t)(q - zk0)) % ZRING;
      double *dst = RAW + s * 6 * ZRS;
      mbar_expect_tx(&bar[s], 6u * ZNN * sizeof(double));
#pragma unroll
      for (int f = 0; f < 6; ++f)
        tma_load_3d(dst + f * ZRS, &maps.m[f], &bar[s], cx, zj0 + 1, q + 1);
    };
    auto wait_plane = [&](int q) {
      const uint32_t u = ubase + (uint32_t)(q - zk0);
      mbar_wait(&bar[u % ZRING], (u / ZRING) & 1u);
    };
    auto xp_slot = [&](int q) {
#if HYDRO_ZONE_XPBAR
      return XP + ((ubase + (uint32_t)(q - zk0)) % ZXP) * 3 * ZRS;
#else
      return XP + ((q - zk0) % 3) * 3 * ZRS;
#endif
    };
    auto form_xp = [&](int q) {
      const double *R = RAW + ((ubase + (uint32_t)(q - zk0)) % ZRING) * 6 * ZRS;
      double *X = xp_slot(q);
      for (int n = t; n < ZNN; n += ZBX * ZBY) {
        X[n] = fma(hh, R[3 * ZRS + n], R[n]);
        X[ZRS + n] = fma(hh, R[4 * ZRS + n], R[ZRS + n]);
        X[2 * ZRS + n] = fma(hh, R[5 * ZRS + n], R[2 * ZRS + n]);
      }
#if HYDRO_ZONE_XPBAR
      mbar_arrive(&xbar[(ubase + (uint32_t)(q - zk0)) % ZXP]);
#endif
    };
#if HYDRO_ZONE_XPBAR
    auto xp_wait = [&](int q) {
      const uint32_t u = ubase + (uint32_t)(q - zk0);
      mbar_wait(&xbar[u % ZXP], (u / ZXP) & 1u);
    };
    if (t == 0)
      for (int q = zk0; q < zk0 + 3 && q <= zk1; ++q) issue(q);
    wait_plane(zk0);
    form_xp(zk0);
    wait_plane(zk0 + 1);  // a segment has >= 1 zone plane: node planes zk0 .. zk1 >= zk0 + 1
    form_xp(zk0 + 1);
    xp_wait(zk0);
#else
    if (t == 0)
      for (int q = zk0; q < zk0 + ZRING - 1 && q <= zk1; ++q) issue(q);
    wait_plane(zk0);
    form_xp(zk0);
#endif

    const bool in_xy = li < zhi.x && lj < zhi.y;
    const int64_t gx = d.lo[0] + li, gy = d.lo[1] + lj;
    const bool exists_xy = in_xy && gx >= 0 && gx < d.N[0] && gy >= 0 && gy < d.N[1];
    const bool owned_xy = li >= 0 && lj >= 0 && li < n0 && lj < n1;
    const int nidx = ty * ZNX + tx + xoff;
    // 32-bit storage indices (a domain's storage is below 2^31 elements, checked at create)
    const int zrow = (lj + 1) * (int)d.zsx + (li + 1), zsxy = (int)d.zsxy;

    // Values handed from plane p to plane p+1: the zone's m, e, 1/m (prefetched one plane
    // ahead) and its z-high face (= the z-low face of the zone above).  Two sets alternate (the
    // body runs twice per trip with the roles swapped), so no registers are copied between planes.
    struct Carry { double m, e, zx, zy, zz, za2; };
    Carry S0 = {}, S1 = {};
    if (exists_xy && zk0 >= gz_lo && zk0 < gz_hi) {
      S0.m = d.m[(zk0 + 1) * zsxy + zrow];
      S0.e = d.e[(zk0 + 1) * zsxy + zrow];
    }

    auto body = [&](const int p, const Carry &cu, Carry &nx) {
      const double m = cu.m, e = cu.e;
      const bool exists = exists_xy && p >= gz_lo && p < gz_hi;
      {
        const int q = p + 1;
        const bool ok = q < zk1 && exists_xy && q >= gz_lo && q < gz_hi;
        nx.m = ok ? d.m[(q + 1) * zsxy + zrow] : 0.0;
        nx.e = ok ? d.e[(q + 1) * zsxy + zrow] : 0.0;
      }
#if HYDRO_ZONE_XPBAR
      // every thread has formed x_p of plane p+1, so every thread has finished zone plane
      // p-2: the TMA slot of node plane p-2 and the x_p slot of plane p-2 are free
      xp_wait(p + 1);
      if (t == 0 && p + 3 <= zk1) issue(p + 3);
      if (p + 2 <= zk1) {
        wait_plane(p + 2);
        form_xp(p + 2);
      }
#else
      wait_plane(p + 1);
      form_xp(p + 1);
      __syncthreads();
      if (t == 0 && p + ZRING - 1 <= zk1) issue(p + ZRING - 1);  // slot of plane p-1 (done)
#endif
      const double *Xa = xp_slot(p), *Xb = xp_slot(p + 1);
      const double *Ua = RAW + ((ubase + (uint32_t)(p - zk0)) % ZRING) * 6 * ZRS + 3 * ZRS;
      const double *Ub = RAW + ((ubase + (uint32_t)(p + 1 - zk0)) % ZRING) * 6 * ZRS + 3 * ZRS;
      double X[8], Y[8], Z[8];
#pragma unroll
      for (int l = 0; l < 8; ++l) {
        const double *S = (l >> 2) ? Xb : Xa;
        const int n = nidx + ((l >> 1) & 1) * ZNX + (l & 1);
        X[l] = S[n];
        Y[l] = S[ZRS + n];
        Z[l] = S[2 * ZRS + n];
      }
      double fx[6], fy[6], fz[6];
#pragma unroll
      for (int a = 0; a < 2; ++a) HYDRO_FACE(X, Y, Z, a + 6, a, a + 4, a + 2, fx[a], fy[a], fz[a]);
#pragma unroll
      for (int b = 0; b < 2; ++b)
        HYDRO_FACE(X, Y, Z, 5 + 2 * b, 2 * b, 1 + 2 * b, 2 * b + 4, fx[2 + b], fy[2 + b],
                   fz[2 + b]);
      // z-low face = the z-high face this thread formed for the zone below (same nodes, bits)
      double za2 = cu.za2;
      if (p == zk0) {
        HYDRO_FACE(X, Y, Z, 3, 0, 2, 1, fx[4], fy[4], fz[4]);
        za2 = fx[4] * fx[4] + fy[4] * fy[4] + fz[4] * fz[4];
      } else {
        fx[4] = cu.zx; fy[4] = cu.zy; fz[4] = cu.zz;
      }
      HYDRO_FACE(X, Y, Z, 7, 4, 6, 5, fx[5], fy[5], fz[5]);
      nx.zx = fx[5]; nx.zy = fy[5]; nx.zz = fz[5];
      // corner vectors S_l = s(a)AX_a + (s(b)AY_b + s(c)AZ_c): the (b, c) pair sums once
      double qx[4], qy[4], qz[4];
#pragma unroll
      for (int bc = 0; bc < 4; ++bc) {
        const int b = bc & 1, c = bc >> 1;
        qx[bc] = (b ? fx[3] : -fx[2]) + (c ? fx[5] : -fx[4]);
        qy[bc] = (b ? fy[3] : -fy[2]) + (c ? fy[5] : -fy[4]);
        qz[bc] = (b ? fz[3] : -fz[2]) + (c ? fz[5] : -fz[4]);
      }
      double V8 = 0.0, DV8 = 0.0;
#pragma unroll
      for (int l = 0; l < 8; ++l) {
        const int a = l & 1, b = (l >> 1) & 1, c = (l >> 2) & 1, bc = l >> 1;
        const double sx = (a ? fx[1] : -fx[0]) + qx[bc];
        const double sy = (a ? fy[1] : -fy[0]) + qy[bc];
        const double sz = (a ? fz[1] : -fz[0]) + qz[bc];
        if (l > 0) V8 += (X[l] - X[0]) * sx + (Y[l] - Y[0]) * sy + (Z[l] - Z[0]) * sz;
        const double *Us = c ? Ub : Ua;
        const int n = nidx + b * ZNX + a;
        DV8 += Us[n] * sx + Us[ZRS + n] * sy + Us[2 * ZRS + n] * sz;
      }
      const double V = V8 * (1.0 / 24.0);
      const double DV = 0.125 * DV8;
      // max squared face area; the z-high face's square is handed to the zone above
      const double zh2 = fx[5] * fx[5] + fy[5] * fy[5] + fz[5] * fz[5];
      nx.za2 = zh2;
      // (compare-select, not fmax: fp64 fmax costs a NaN-handling sequence; areas are finite)
      double a2 = zh2 > za2 ? zh2 : za2;
#pragma unroll
      for (int f = 0; f < 4; ++f) {
        const double v = fx[f] * fx[f] + fy[f] * fy[f] + fz[f] * fz[f];
        a2 = v > a2 ? v : a2;
      }
      // S2-S4, S6 (see kernel_cycle.cu for the algebra): L = 2V/sqrt(a2) enters through
      // s = -2 DV/sqrt(a2) and dt^2 = V^2 min(4 cfl^2/(a2 sigma^2), c_vol^2/DV^2).
      const double iV = frcp(V);
      const double rho = m * iV;
      const double epos = e > 0.0 ? e : 0.0;
      // e_p = e - (hh p~ DV) / m with p~ = gm1 (m / V) e+: the mass cancels, so the zone's 1/m
      // is not needed here (within rounding of the oracle's order)
      const double ep = e - (hgm1 * epos) * DV * iV;
      const double eppos = ep > 0.0 ? ep : 0.0;
      const double pr = ph.gm1 * rho * eppos;
      const double c2 = ph.ggm1 * eppos;
      double qr = 0.0;
      if (DV < 0.0) {
        const double c = fsqrt(c2);
        const double s = -2.0 * DV * frsqrt(a2);
        qr = s * (ph.q_quad * s + ph.q_lin * c);
      }
      const double P = exists ? pr + rho * qr : 0.0;
      if (in_xy) d.P[(p + 1) * zsxy + zrow] = P;
      if (exists && owned_xy && p >= 0 && p < n2) {
        const double V2 = V * V;
        const double n1c = cfl4 * V2, d1c = (c2 + 2.0 * qr) * a2;
        const double n2c = cv2 * V2, d2c = DV * DV;
        const bool ok1 = d1c > 1e-290, ok2 = d2c > 1e-290;
        const bool pick1 = ok1 && (!ok2 || n1c * d2c < n2c * d1c);
        const double num = pick1 ? n1c : n2c, den = pick1 ? d1c : d2c;
        const double dt2 = (ok1 || ok2) ? num * frcp(den) : INFINITY;
        dt2min = dt2 < dt2min ? dt2 : dt2min;
        if (!(V > 0.0) || !isfinite(P)) {
          const int64_t gzi = ((d.lo[2] + p) * d.N[1] + gy) * (int64_t)d.N[0] + gx;
          flag_error_zone(st, (V > 0.0) ? ERR_NONFINITE : ERR_TANGLED, gzi);
        }
      }
    };
    for (int p = zk0; p < zk1; p += 2) {
      body(p, S0, S1);
      if (p + 1 >= zk1) break;
      body(p + 1, S1, S0);
    }
    ubase += (uint32_t)(zk1 + 1 - zk0);  // node planes zk0..zk1 went through the ring
    __syncthreads();  // every read of this segment's ring and XP slots is done
  }
  block_min_dt_smem(sqrt(dt2min), &st->dtz_acc, sm + ZOFF_RED);
}


// Tiling of one domain's zone stage: ghost ring only on sides with a neighbouring domain whose
// ring bit is set (ring zones owned by a domain of this GPU get their P by a copy instead).
ZoneTask zone_task(const DomView &d, int slot, uint8_t ring) {
  ZoneTask T = {};
  T.slot = slot;
  for (int a = 0; a < 3; ++a) {
    T.zlo[a] = (d.lo[a] > 0 && (ring >> (2 * a) & 1u)) ? -1 : 0;
    T.zhi[a] = (d.lo[a] + d.n[a] < d.N[a] && (ring >> (2 * a + 1) & 1u)) ? d.n[a] + 1 : d.n[a];
  }
  T.tcols = (T.zhi[0] - T.zlo[0] + ZBX - 1) / ZBX;
  const int ty = (T.zhi[1] - T.zlo[1] + ZBY - 1) / ZBY;
  T.units = (int64_t)T.tcols * ty * (T.zhi[2] - T.zlo[2]);
  T.u0 = 0;
  T.zblk = T.zhi[2] - T.zlo[2];
  static const int zb_env = getenv("HYDRO_ZONE_ZBLK") ? atoi(getenv("HYDRO_ZONE_ZBLK")) : 0;
  if (zb_env > 0) T.zblk = std::min(T.zblk, zb_env);
  return T;
}

int zone_slots() {  // per device: the shared-memory opt-in is a per-device attribute
  static int slots_dev[64] = {};
  int dev = 0;
  cudaGetDevice(&dev);
  int &slots = slots_dev[dev < 0 ? 0 : (dev >= 64 ? 63 : dev)];
  if (!slots) {
    int sms = 0, per_sm = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    for (auto k : {k_zone_stage<false>, k_zone_stage<true>})
      cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)ZBYTES);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_zone_stage<false>, ZBX * ZBY,
                                                  ZBYTES);
    slots = sms * std::max(per_sm, 1);
  }
  return slots;
}

}  // namespace

int zone_box_y() { return ZNY; }

void launch_zone_stage(const DomView &d, const NodeMaps &maps, uint8_t ring, const Phys &ph,
                       DevState *st, cudaStream_t s) {
  const int slots = zone_slots();
  ZoneTask T = zone_task(d, 0, ring);
  // Default: the persistent linearised split (measured 67 vs 70 us for the best chunking at
  // 128^3).  HYDRO_KZ_ZONE=k: the chunked schedule with k planes per CTA (A/B measurement).
  static const int kz_env = getenv("HYDRO_KZ_ZONE") ? atoi(getenv("HYDRO_KZ_ZONE")) : 0;
  const int nz = T.zhi[2] - T.zlo[2];
  int G, kz = 0;
  if (kz_env > 0) {
    kz = std::min(kz_env, nz);
    G = (int)(T.units / nz) * ((nz + kz - 1) / kz);
    T.zblk = nz;  // the chunked schedule indexes units column-major
  } else {
    G = (int)std::min<int64_t>(slots, T.units);
  }
  launch_pdl(k_zone_stage<false>, dim3(G), dim3(ZBX * ZBY), ZBYTES, s, maps, d, T,
             (const DomView *)nullptr, (const NodeMaps *)nullptr, (const ZoneTask *)nullptr,
             T.units, kz, ph, st);
}

void zone_group_tasks(const DomView *views_host, const uint8_t *rings, int n, ZoneTask *out,
                      int64_t *Wtot) {
  int64_t u = 0;
  for (int i = 0; i < n; ++i) {
    out[i] = zone_task(views_host[i], i, rings[i]);
    out[i].u0 = u;
    u += out[i].units;
  }
  *Wtot = u;
}

void launch_zone_stage_group(const DomView *views_dev, const NodeMaps *maps_dev,
                             const ZoneTask *tasks_dev, int64_t Wtot, const Phys &ph,
                             DevState *st, cudaStream_t s) {
  const int G = (int)std::min<int64_t>(zone_slots(), Wtot);
  DomView d0 = {};
  NodeMaps m0 = {};
  ZoneTask t0 = {};
  launch_pdl(k_zone_stage<true>, dim3(G), dim3(ZBX * ZBY), ZBYTES, s, m0, d0, t0, views_dev,
             maps_dev, tasks_dev, Wtot, 0, ph, st);
}

}  // namespace hydro
