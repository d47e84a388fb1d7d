// kernel_cycle.cu -- the node/energy side of the cycle (S5 face form, S7, S8), either with the
// zone physics recomputed in the same kernel (FUSED: the whole cycle S1-S8 in ONE kernel) or
// with P read from HBM as written by the zone-stage kernel (kernel_zone.cu).
//
// Blocking.  A block owns a TX x TY column of zones of one domain and marches it
// through a z-chunk [k0, k1) (2.5-D blocking).  Thread (tx, ty) stands for zone and node
// (i0-1+tx, j0-1+ty): the tile plus a one-zone ring, which is recomputed instead of exchanged.
// Node planes stream in through TMA (one box per field, mbarrier completion) into a 3-slot ring
// two planes ahead of use.  Per zone plane p, separated by __syncthreads:
//   X  own node of plane p+1: x_p = x + dt/2 u (S1), kept in registers and shared;
//   Z  zone plane p: FUSED -- faces, corner vectors, V, DV, predictor, EOS, q, P, dt_z^2
//      (S2-S4, S6); otherwise P comes from HBM and only the three low faces are formed;
//   G  per-face force vectors g_f = (P_below - P_above) A_f / 4 of each zone's low faces (S5 in
//      face form: sum_z P_z B_z,l regrouped by faces);
//   N  node plane p: F = sum of the 12 incident g_f (4 own, 5 read), m_p, a, reflecting walls,
//      u', u_half, x' (S7), written to HBM; u_half and its two-plane sum are shared;
//   E  zone plane p-1: psi_f = A_f . (sum of u_half over the face), W = P/8 sum_f +-psi_f,
//      e' = e - dt W / m (S8), written to HBM.
// No tensor cores: nothing here is a dense contraction (BASELINE.json north_star).
#include <algorithm>
#include <climits>
#include <cmath>
#include <cstdlib>

#include "fastmath.cuh"
#include "kernels.h"
#include "tma.cuh"
#include "zone_physics.cuh"

namespace hydro {

namespace {

template <int TX, int TY>
struct CTile {
  static constexpr int TXT = TX + 2, TYT = TY + 2;  // zone-stage tile (owned + 1 ring)
  // One row pitch PX for the threads, the node box and the zone box (TX + 3 node columns rounded
  // up to a 16-byte TMA row): neighbour offsets are the same in every array and a warp's LDS.64
  // over consecutive threads touches consecutive words (no bank conflicts at row wraps).
  static constexpr int PX = FUSED_BOX_X;
  static constexpr int NZT = PX * TYT;              // thread slots of the tile rows
  static constexpr int NTHR = (NZT + 31) / 32 * 32;
  static constexpr int ZS = NTHR;                   // zone-tile slots
  static constexpr int BXN = FUSED_BOX_X, BYN = TY + 3;  // TMA node box (x padded to 16 B)
  static constexpr int NN = BXN * BYN;
  static constexpr int RS = (NN + 15) / 16 * 16;    // stride of one node array (128 B aligned)
  static constexpr int ZBX = PX, ZBY = TYT;         // TMA zone box = the zone tile (+ pad)
  static constexpr int ZN = ZBX * ZBY;
  static constexpr int ZRS = (ZN + 15) / 16 * 16;
  // shared memory, in doubles; SoA everywhere so a warp's LDS.64 is conflict-free
// Phase-barrier arrivals: every thread arrives (release) on its own.  The warp-elected variant
// (__syncwarp, then lane 0 arrives; HYDRO_ARRIVE_ALL=0) is correct under the PTX memory model
// (bar.warp.sync orders the lanes' stores before lane 0's cumulative release) and measured
// equally fast, but compute-sanitizer racecheck does not follow that chain and reports every
// phase as a hazard; per-thread arrivals are racecheck-clean at the same speed (94.2 vs 94.3 us).
#ifndef HYDRO_ARRIVE_ALL
#define HYDRO_ARRIVE_ALL 1
#endif
#ifndef HYDRO_MN8_TMA
#define HYDRO_MN8_TMA 1
#endif
  static constexpr int NF = HYDRO_MN8_TMA ? 7 : 6;  // node fields: x,y,z,u,v,w[, 8/nodal mass]
  static constexpr int OFF_RAW = 0;                 // [3 slots][NF fields][RS] (TMA)
  static constexpr int OFF_ZR = OFF_RAW + 3 * NF * RS;  // [3 slots][3 fields][ZRS] m, e, P (TMA)
  static constexpr int OFF_XP = OFF_ZR + 9 * ZRS;   // [2 planes][3][RS] half-step positions
  // PAD doubles after XP and UH: the padding lanes (t >= NZT) run the unconditional corner and
  // u_half neighbour loads up to PX + 1 entries past their array; the pad keeps those dead reads
  // inside dead memory instead of the next array (racecheck-clean)
  static constexpr int PAD = 64;
  static constexpr int OFF_G = OFF_XP + 6 * RS + PAD;  // [3 vectors][3][ZS] g_x, g_y, g_z
  static constexpr int OFF_UH = OFF_G + 9 * ZS;     // [3][ZS] u_half of node plane p
  static constexpr int OFF_P = OFF_UH + 3 * ZS + PAD;  // [ZS] P of zone plane p (FUSED)
  static constexpr int OFF_PS = OFF_P + ZS;         // [2][ZS] psi of x-low, y-low faces
  static constexpr int OFF_RED = OFF_PS + 2 * ZS;   // [32] block dt reduction
  static constexpr int OFF_BAR = OFF_RED + 32;      // 3 TMA mbarriers + 3 phase mbarriers
  static constexpr int TOTAL = OFF_BAR + 8;
  static constexpr size_t BYTES = sizeof(double) * TOTAL;
  static_assert(BXN >= TX + 3 && BXN == PX, "TMA box too narrow");
  static_assert(BYN <= 256 && BXN <= 256, "TMA box limit");
  static_assert((ZBX * 8) % 16 == 0, "TMA zone box rows must be 16-byte multiples");
  static_assert(ZRS >= ZS - 32 && ZN <= ZS, "zone tile fits the thread tile");
  static_assert(BYTES <= 227 * 1024, "shared memory");
  static_assert(9 * ZS * sizeof(double) >= (64 * 8 + 2) * sizeof(int), "fused-halo table");
};

// GROUP: one chunked launch over all domains of this GPU; CTA b belongs to the NodeTask whose
// [cta0, cta0 + ctas) contains b (adjacent CTAs: adjacent columns of one domain, same z-chunk).
template <int TX, int TY, bool FUSED, bool GROUP>
__global__ void __launch_bounds__(CTile<TX, TY>::NTHR, 1)
    k_cycle(const __grid_constant__ NodeMaps maps1, const __grid_constant__ DomView d1, Phys ph,
            DevState *st, int tcols1, int ncols1, int sched_kz1, int fold_finalize,
            const NodeTask *tasks, int ntasks, const DomView *views, const NodeMaps *mapsg,
            const PushSlab *push1, int npush1) {
  using T = CTile<TX, TY>;
  // dynamic shared memory only (no static __shared__), so the window is 1024-byte aligned
  extern __shared__ __align__(1024) double sm[];
  double *RAW = sm + T::OFF_RAW, *ZR = sm + T::OFF_ZR, *XP = sm + T::OFF_XP, *PSF = sm + T::OFF_P;
  double *GX = sm + T::OFF_G, *GY = GX + 3 * T::ZS, *GZ = GY + 3 * T::ZS;
  double *UH = sm + T::OFF_UH, *PSX = sm + T::OFF_PS, *PSY = PSX + T::ZS;
  uint64_t *bar = reinterpret_cast<uint64_t *>(sm + T::OFF_BAR);
  constexpr int ZS = T::ZS, RS = T::RS, TXT = T::TXT, ZRS = T::ZRS, PX = T::PX;

  pdl_wait_and_trigger();
  int task_i = 0;
  if (GROUP)
    while (task_i + 1 < ntasks && (int)blockIdx.x >= tasks[task_i + 1].cta0) ++task_i;
  const DomView &d = GROUP ? views[tasks[task_i].slot] : d1;
  const NodeMaps &maps = GROUP ? mapsg[tasks[task_i].slot] : maps1;
  const int ncols = GROUP ? tasks[task_i].ncols : ncols1;
  const int tcols = GROUP ? tasks[task_i].tcols : tcols1;
  const int sched_kz = GROUP ? tasks[task_i].kz : sched_kz1;
  const int bid = GROUP ? (int)blockIdx.x - tasks[task_i].cta0 : (int)blockIdx.x;
  const PushSlab *push = GROUP ? push1 + tasks[task_i].push0 : push1;
  const int npush = GROUP ? tasks[task_i].npush : npush1;
  const int t = threadIdx.x;
  const int n0 = d.n[0], n1 = d.n[1], n2 = d.n[2];
  // lanes: zone/node (tx, ty) for tx < TXT; tx == TXT forms the box's last node column; the
  // rest (tx == PX-1 and the padding warp's tail) form the box's last node row
  const int tc = t;
  const int tx = t % PX, ty = t / PX;
  const bool active = t < T::NZT && tx < TXT;

  // Work split (persistent, SM-count-sized grid; same scheme as kernel_zone.cu): the tile
  // columns (TX x TY, all n2 zone planes) are linearised column-major into ncols * n2 units and
  // CTA b takes [b W / G, (b+1) W / G), marched as one or two column segments.  sched_kz > 0:
  // the chunked schedule (CTA b = column b / chunks, chunk b % chunks), for A/B measurement.
  int64_t r0, r1;
  int unit = bid, nunits = 0;  // chunked schedule: this CTA's (column, chunk) unit
  if (sched_kz > 0) {
    nunits = ncols * ((n2 + sched_kz - 1) / sched_kz);
    const int64_t col = bid % ncols, ch = bid / ncols;  // adjacent CTAs: same z
    r0 = col * n2 + ch * sched_kz;
    r1 = col * n2 + min((int)(ch + 1) * sched_kz, n2);
  } else {
    const int64_t W = (int64_t)ncols * n2;
    r0 = W * blockIdx.x / gridDim.x;
    r1 = W * (blockIdx.x + 1) / gridDim.x;
  }
  const bool halted = (st->halted | st->done) != 0u;
  if (!halted && t == 0) {
    if (smem_u32(sm) & 127u) __trap();  // TMA destinations must be 128-byte aligned
    for (int s = 0; s < 3; ++s) mbar_init(&bar[s], 1);
    for (int s = 3; s < 6; ++s)  // one arrival per warp (HYDRO_ARRIVE_ALL: per thread)
      mbar_init(&bar[s], HYDRO_ARRIVE_ALL ? T::NTHR : T::NTHR / 32);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  double dt2min = INFINITY;

  // Fused halo: after a column segment, the CTA stores the part of every
  // neighbour's ghost slab that it has just written (nodes of planes [k0, k1), plus n2 on the
  // last chunk; zones of planes [k0, k1)) into the neighbour's next-parity arrays, reading the
  // values back from its own freshly written (L2-resident) output.  Replaces the separate
  // intra-GPU copy / peer push kernel: the exchange overlaps the other CTAs' compute.  Warp 0
  // clips the (<= 32) slabs against the segment in parallel, one lane per slab, and scans the
  // item counts into a table in the (now idle) g-vector smem; then every (slab, kind, element)
  // item is one independent load/store for some thread.
  auto push_halo = [&](int i0, int j0, int k0, int k1) {
    int *tab = reinterpret_cast<int *>(sm + T::OFF_G);  // [64 items][8]: end, lo x3, ext x2, slab, kind
    if (t < 32) {
      // this segment's output: nodes [i0, wn1) x [j0, wn1) x [k0, wn1), zones [.., wz1); the last
      // tile in x / y also writes the domain's last node (F_NWR), the last chunk node plane n2
      const int wn1[3] = {n0 <= i0 + TX ? n0 + 1 : i0 + TX, n1 <= j0 + TY ? n1 + 1 : j0 + TY,
                          k1 == n2 ? n2 + 1 : k1};
      const int wz1[3] = {min(i0 + TX, n0), min(j0 + TY, n1), k1};
      const int w0[3] = {i0, j0, k0};
      int cnt[2] = {0, 0}, lo[2][3] = {}, ext[2][3] = {}, rem = 0;
      if (t < npush) {
        const PushSlab &S = push[t];
        rem = S.remote;
#pragma unroll
        for (int c = 0; c < 2; ++c) {
          int n = 1;
#pragma unroll
          for (int a = 0; a < 3; ++a) {
            lo[c][a] = max(c ? S.zlo[a] : S.nlo[a], w0[a]);
            ext[c][a] = min(c ? S.zhi[a] : S.nhi[a], c ? wz1[a] : wn1[a]) - lo[c][a];
            n = ext[c][a] > 0 ? n * ext[c][a] : 0;
          }
          cnt[c] = n;
        }
      }
      int incl = cnt[0] + cnt[1];  // inclusive warp scan of the per-slab item counts
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const int v = __shfl_up_sync(0xffffffffu, incl, o);
        if (t >= o) incl += v;
      }
      const int excl = incl - cnt[0] - cnt[1];
#pragma unroll
      for (int c = 0; c < 2; ++c) {
        int *r = tab + (2 * t + c) * 8;
        r[0] = excl + cnt[0] + (c ? cnt[1] : 0);  // end of the item range
        r[1] = lo[c][0]; r[2] = lo[c][1]; r[3] = lo[c][2];
        r[4] = ext[c][0]; r[5] = ext[c][1];
        r[6] = t; r[7] = c;
      }
      const bool any_remote = __any_sync(0xffffffffu, rem && (cnt[0] + cnt[1]) > 0);
      if (t == 31) {
        tab[64 * 8] = incl;
        tab[64 * 8 + 1] = any_remote;
      }
    }
    __syncthreads();
    const int total = tab[64 * 8];
    const int nsx = (int)d.nsx, nsxy2 = (int)d.nsxy, zsx = (int)d.zsx, zsxy2 = (int)d.zsxy;
    // two items per thread in flight: both items' loads, then both items' stores
    struct Item { int kind, si; int64_t di; const PushSlab *S; };
    auto locate = [&](int e) {
      int a = 0, b = 63;  // first item whose end exceeds e
      while (a < b) {
        const int m = (a + b) >> 1;
        if (tab[m * 8] > e) b = m;
        else a = m + 1;
      }
      const int *r = tab + a * 8;
      const int rem = e - (a ? tab[(a - 1) * 8] : 0);
      const int i = r[1] + rem % r[4], q = rem / r[4];
      const int j = r[2] + q % r[5], k = r[3] + q / r[5];
      Item it;
      it.kind = r[7];
      it.S = push + r[6];
      if (it.kind == 0) {
        it.si = (k + 1) * nsxy2 + (j + 1) * nsx + (i + 1);
        it.di = __ldg(&it.S->nbase) + (int64_t)k * __ldg(&it.S->nsxy) +
                (int64_t)j * __ldg(&it.S->nsx) + i;
      } else {
        it.si = (k + 1) * zsxy2 + (j + 1) * zsx + (i + 1);
        it.di = __ldg(&it.S->zbase) + (int64_t)k * __ldg(&it.S->zsxy) +
                (int64_t)j * __ldg(&it.S->zsx) + i;
      }
      return it;
    };
    auto load = [&](const Item &it, double &v0, double &v1, double &v2, double &v3, double &v4,
                    double &v5) {
      if (it.kind == 0) {
        v0 = d.xn[it.si]; v1 = d.yn[it.si]; v2 = d.zn[it.si];
        v3 = d.un[it.si]; v4 = d.vn[it.si]; v5 = d.wn[it.si];
      } else {
        v0 = d.en[it.si];
      }
    };
    auto store = [&](const Item &it, double v0, double v1, double v2, double v3, double v4,
                     double v5) {
      const long long *dst = (const long long *)it.S->dst;
      if (it.kind == 0) {
        ((double *)__ldg(dst + 0))[it.di] = v0;
        ((double *)__ldg(dst + 1))[it.di] = v1;
        ((double *)__ldg(dst + 2))[it.di] = v2;
        ((double *)__ldg(dst + 3))[it.di] = v3;
        ((double *)__ldg(dst + 4))[it.di] = v4;
        ((double *)__ldg(dst + 5))[it.di] = v5;
      } else {
        ((double *)__ldg(dst + 6))[it.di] = v0;
      }
    };
    for (int e0 = t; e0 < total; e0 += 2 * T::NTHR) {
      const bool two = e0 + T::NTHR < total;
      const Item A = locate(e0);
      const Item B = locate(two ? e0 + T::NTHR : e0);
      double a0 = 0, a1 = 0, a2 = 0, a3 = 0, a4 = 0, a5 = 0;
      double b0 = 0, b1 = 0, b2 = 0, b3 = 0, b4 = 0, b5 = 0;
      load(A, a0, a1, a2, a3, a4, a5);
      load(B, b0, b1, b2, b3, b4, b5);
      store(A, a0, a1, a2, a3, a4, a5);
      if (two) store(B, b0, b1, b2, b3, b4, b5);
    }
    if (total && tab[64 * 8 + 1]) __threadfence_system();  // peer stores before the mailbox flag
    __syncthreads();  // the table region is the next segment's g-vector array
  };
  uint32_t ubase = 0;  // TMA planes consumed in earlier segments (ring slot / phase continuity)
  uint32_t pbase = 0;  // plane iterations run in earlier segments (phase-barrier parity)

  for (int64_t r = r0;;) {
  if (r >= r1) {
    // chunked schedule on a persistent grid (fewer CTAs than units): the next unit is
    // unit + gridDim.x, so the CTAs running at any time still hold consecutive units (adjacent
    // columns at the same z-chunk: shared ring rows stay L2 hits)
    if (sched_kz <= 0 || GROUP) break;
    unit += gridDim.x;
    if (unit >= nunits) break;
    const int64_t c = unit % ncols, ch = unit / ncols;
    r = c * n2 + ch * sched_kz;
    r1 = c * n2 + min((int)(ch + 1) * sched_kz, n2);
  }
  const int col = (int)(r / n2);
  const int k0 = (int)(r - (int64_t)col * n2);
  const int k1 = (int)min((int64_t)n2, r1 - (int64_t)col * n2);
  r = (int64_t)col * n2 + k1;
  const int i0 = (col % tcols) * TX, j0 = (col / tcols) * TY;
  const int li = i0 - 1 + tx, lj = j0 - 1 + ty;  // local zone / node index of this thread

  if (halted) {  // no-op cycle: carry the state over to the next parity
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
    if (!FUSED && npush) {
      __syncthreads();  // the whole segment's output is written
      push_halo(i0, j0, k0, k1);
    }
    continue;
  }

  const double dt = st->dt;
  const double hh = 0.5 * dt;
  const int q0 = k0 - 1;  // first node plane of the chunk

  // TMA producer: node plane q and zone plane q (m, e, and P unless FUSED) -> slot (q-q0)%3,
  // one mbarrier per slot.  Zone plane q lies between node planes q and q+1.
  constexpr int NZF = FUSED ? 2 : 3;
  auto issue = [&](int q) {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    const uint32_t u = ubase + (uint32_t)(q - q0), s = u % 3;
    double *dst = RAW + s * T::NF * RS;
    double *zdst = ZR + s * 3 * ZRS;
    mbar_expect_tx(&bar[s], ((unsigned)T::NF * T::NN + (unsigned)NZF * T::ZN) * sizeof(double));
#pragma unroll
    for (int f = 0; f < T::NF; ++f) tma_load_3d(dst + f * RS, &maps.m[f], &bar[s], i0, j0, q + 1);
#pragma unroll
    for (int f = 0; f < NZF; ++f)  // FUSED: m, e; else 1/m (z[3]), e, P
      tma_load_3d(zdst + f * ZRS, &maps.z[(FUSED || f) ? f : 3], &bar[s], i0, j0, q + 1);
  };
  auto wait_plane = [&](int q) {
    const uint32_t u = ubase + (uint32_t)(q - q0);
    mbar_wait(&bar[u % 3], (u / 3) & 1u);
  };
  auto raw = [&](int q) { return RAW + ((ubase + (uint32_t)(q - q0)) % 3) * T::NF * RS; };
  auto zraw = [&](int q) { return ZR + ((ubase + (uint32_t)(q - q0)) % 3) * 3 * ZRS; };
  // X stage: half-step positions of node plane q into XP slot q&1.  Thread t forms its own
  // node (tx, ty) -- returned in registers -- and the box's last column / row are shared out.
  const int nidx = t;  // this thread's node in the node box (pitch PX)
  const bool xown = t < T::NZT && tx <= TXT;  // forms x_p of its own node
  const int hrow = tx == PX - 1 ? ty : (t >= T::NZT ? T::TYT + (t - T::NZT) : -1);
  constexpr int NHELP = T::TYT + (T::NTHR - T::NZT);  // lanes forming the last node row
  auto form_xp = [&](int q, double &px, double &py, double &pz) {
    const double *R = raw(q);
    double *X = XP + (q & 1) * 3 * RS;
    px = fma(hh, R[3 * RS + nidx], R[nidx]);
    py = fma(hh, R[4 * RS + nidx], R[RS + nidx]);
    pz = fma(hh, R[5 * RS + nidx], R[2 * RS + nidx]);
    if (xown) {
      X[nidx] = px;
      X[RS + nidx] = py;
      X[2 * RS + nidx] = pz;
    }
    // the box's last node row (TYT), columns 0..TXT
    for (int e = hrow; e >= 0 && e <= TXT; e += NHELP) {
      const int n = T::TYT * PX + e;
      X[n] = fma(hh, R[3 * RS + n], R[n]);
      X[RS + n] = fma(hh, R[4 * RS + n], R[RS + n]);
      X[2 * RS + n] = fma(hh, R[5 * RS + n], R[2 * RS + n]);
    }
  };
  auto st3 = [](double *b, int i, double x, double y, double z) {
    b[i] = x; b[ZS + i] = y; b[2 * ZS + i] = z;
  };
  auto ld3 = [](const double *b, int i, double &x, double &y, double &z) {
    x = b[i]; y = b[ZS + i]; z = b[2 * ZS + i];
  };

  if (t == 0) {
    issue(q0);
    issue(q0 + 1);
    if (q0 + 2 <= k1 + 1) issue(q0 + 2);
  }

  // Values one plane hands to the next.  Two sets alternate (the loop body runs twice per trip
  // with the roles swapped), so nothing is copied between iterations: iteration p reads plane
  // p-1's set `pv` and overwrites `cu`, which until then holds plane p-2 (the pending E2).
  struct Carry {
    double P, im, e;                // zone: P, 1/m, e
    double ax, ay, az, bx, by, bz;  // zone: x-low and y-low face vectors
    double Sx, Sy, Sz;              // node: sum of the 4 in-plane face forces of this zone plane
    double uh, vh, wh;              // node: own u_half
    double nxu, nxv, nxw;           // u_half of node (tx+1, ty)
    double nyu, nyv, nyw;           // u_half of node (tx, ty+1)
    double psiz;                    // psi of the z-face at this node plane
    double part;                    // E2 partial sum of the zone plane (set one plane later)
  };
  struct XP3 { double x, y, z; };  // own node's half-step position
  Carry S0 = {}, S1 = {};

  // Per-thread constants, kept in few registers (32-bit indices: a domain's storage is below
  // 2^31 elements, checked at create) so the compiler does not rematerialise them per plane.
  const int gxz = (int)d.lo[0] + li, gyz = (int)d.lo[1] + lj;
  const uint32_t rm = ph.reflect_mask;
  enum : uint32_t { F_ZEX = 1, F_NODE = 2, F_NWR = 4, F_OWN = 8, F_EXX = 16, F_EXY = 32,
                    F_EXZ = 64, F_WX = 128, F_WY = 256 };
  uint32_t fl = 0;
  {
    const bool in_t = active && tx >= 1 && ty >= 1;
    if (active && li <= n0 && lj <= n1 && gxz >= 0 && gxz < d.N[0] && gyz >= 0 && gyz < d.N[1])
      fl |= F_ZEX;
    if (in_t && li <= n0 && lj <= n1) {
      fl |= F_NODE;
      if ((li < i0 + TX || li == n0) && (lj < j0 + TY || lj == n1)) fl |= F_NWR;
    }
    if (in_t && tx <= TX && ty <= TY && li < n0 && lj < n1) fl |= F_OWN;
    if (in_t && tx <= TX + 1 && ty <= TY) fl |= F_EXX;
    if (in_t && tx <= TX && ty <= TY + 1) fl |= F_EXY;
    if (in_t && tx <= TX && ty <= TY) fl |= F_EXZ;
    if ((gxz == 0 && (rm & 1u)) || (gxz == d.N[0] && (rm & 2u))) fl |= F_WX;
    if ((gyz == 0 && (rm & 4u)) || (gyz == d.N[1] && (rm & 8u))) fl |= F_WY;
  }
  const int zsxy = (int)d.zsxy, nsxy = (int)d.nsxy;
  const int zoff = (lj + 1) * (int)d.zsx + (li + 1);  // zone id = (q+1)*zsxy + zoff
  const int nrow = (lj + 1) * (int)d.nsx + (li + 1);  // node id = (q+1)*nsxy + nrow
  const int gz_lo = -(int)d.lo[2], gz_hi = d.N[2] - (int)d.lo[2];  // plane q exists iff in range
  const int wz_lo = (rm & 16u) ? gz_lo : INT_MIN, wz_hi = (rm & 32u) ? gz_hi : INT_MIN;
  const double cfl4 = 4.0 * ph.cfl * ph.cfl, cv2 = ph.c_vol * ph.c_vol;

  // Software pipeline (3 barriers per plane, 4 when FUSED): iteration p runs
  //   phase 1: E2 of zone plane p-2 and the zone/face stage of plane p,
  //   phase 2: the node stage of node plane p,
  //   phase 3: x_p of node plane p+2 and E1 of zone plane p-1.
  XP3 XA, XB;  // own node's x_p at planes p and p+1 (x_p of plane p+2 replaces plane p's)
  wait_plane(q0);
  form_xp(q0, XA.x, XA.y, XA.z);
  wait_plane(q0 + 1);
  form_xp(q0 + 1, XB.x, XB.y, XB.z);
  __syncthreads();

  // Split phase barriers (node/energy kernel): a warp arrives once its shared-memory writes of a
  // phase are done, runs work that does not read them, then waits.  Every barrier completes once
  // per plane, so plane p waits on parity (p - q0) & 1.  The fused kernel uses __syncthreads.
  enum { B_G = 3, B_U = 4, B_P = 5 };
  auto arrive = [&](int b) {
    if (HYDRO_ARRIVE_ALL) {
      mbar_arrive(&bar[b]);
    } else {
      __syncwarp();
      if ((t & 31) == 0) mbar_arrive(&bar[b]);
    }
  };
  auto await = [&](int b, int p) { mbar_wait(&bar[b], (pbase + (uint32_t)(p - q0)) & 1u); };
  auto energy2 = [&](int zp, const Carry &c) {  // E2 of zone plane zp from its carry set
    if (fl & F_OWN) {
      const double Wk = 0.125 * c.P * ((PSX[t + 1] + PSY[t + PX]) + c.part);
      d.en[(zp + 1) * zsxy + zoff] = c.e - dt * Wk * c.im;
    }
  };

  auto body = [&](const int p, Carry &pv, Carry &cu, XP3 &xa, const XP3 &xb) {
    // (HYDRO_MN8_TMA=0) 8 / nodal mass from global memory, read early so its latency hides
    const double rinv_g = (!HYDRO_MN8_TMA && (fl & F_NODE) && p >= k0)
                              ? __ldg(d.mn8 + (p + 1) * nsxy + nrow) : 0.0;
    // ---------------------------------------------------------------- phase 1: E2(p-2), Z(p)
    if (FUSED && p >= k0 + 2) energy2(p - 2, cu);  // cu still holds zone plane p-2
    const bool exists = (fl & F_ZEX) && p >= gz_lo && p < gz_hi;
    // zone plane p (TMA): m and e are 0 on zones outside the mesh (never written), P too
    double *MS = zraw(p), *ES = MS + ZRS, *PS = FUSED ? PSF : MS + 2 * ZRS;
    const double m = MS[tc], e = ES[tc];
    double P = FUSED ? 0.0 : PS[tc];
    const double *Ra = raw(p);
    const double *Xa = XP + (p & 1) * 3 * RS, *Xb = XP + ((p + 1) & 1) * 3 * RS;
    if (!FUSED && p > q0) await(B_P, p - 1);  // x_p(p+1) and psi of the previous plane
    double im;
    double ax0, ay0, az0, bx0, by0, bz0, cx0, cy0, cz0;
    if (FUSED) {
      const double *Rb = raw(p + 1);
      double X[8], Y[8], Z[8];
      X[0] = xa.x; Y[0] = xa.y; Z[0] = xa.z;
      X[4] = xb.x; Y[4] = xb.y; Z[4] = xb.z;
#pragma unroll
      for (int l = 0; l < 8; ++l) {
        if (l == 0 || l == 4) continue;
        const int n = nidx + ((l >> 1) & 1) * T::BXN + (l & 1);
        const double *S = (l >> 2) ? Xb : Xa;
        X[l] = S[n]; Y[l] = S[RS + n]; Z[l] = S[2 * RS + n];
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
        const double *Us = (c ? Rb : Ra) + 3 * RS;
        const int n = nidx + b * T::BXN + a;
        DV8 += Us[n] * sx + Us[RS + n] * sy + Us[2 * RS + n] * sz;
      }
      const double V = V8 * (1.0 / 24.0);
      const double DV = 0.125 * DV8;
      double a2 = fx[0] * fx[0] + fy[0] * fy[0] + fz[0] * fz[0];
#pragma unroll
      for (int f = 1; f < 6; ++f) {
        const double v = fx[f] * fx[f] + fy[f] * fy[f] + fz[f] * fz[f];
        a2 = v > a2 ? v : a2;
      }
      // S2-S4 and S6: L = 2V/sqrt(a2) enters only through s = L(-D) = -2 DV/sqrt(a2) and
      // dt^2 = V^2 min(4 cfl^2/(a2 sigma^2), c_vol^2/DV^2) (one reciprocal)
      const double iV = frcp(V);
      im = frcp(m);
      const double rho = m * iV;
      const double epos = e > 0.0 ? e : 0.0;
      const double ep = e - (hh * (ph.gm1 * rho) * epos) * DV * im;
      const double eppos = ep > 0.0 ? ep : 0.0;
      const double pr = ph.gm1 * rho * eppos;
      const double c2 = ph.ggm1 * eppos;
      double qr = 0.0;
      if (DV < 0.0) {  // S4: compression only (sign(D) = sign(DV) for V > 0)
        const double c = fsqrt(c2);
        const double s = -2.0 * DV * frsqrt(a2);
        qr = s * (ph.q_quad * s + ph.q_lin * c);
      }
      P = exists ? pr + rho * qr : 0.0;
      if (exists && p >= k0 && p < k1 && (fl & F_OWN)) {
        const double V2 = V * V;
        const double n1c = cfl4 * V2, d1c = (c2 + 2.0 * qr) * a2;
        const double n2c = cv2 * V2, d2c = DV * DV;
        const bool ok1 = d1c > 1e-290, ok2 = d2c > 1e-290;  // else dt_z^2 > 1e270 V^2: +inf
        const bool pick1 = ok1 && (!ok2 || n1c * d2c < n2c * d1c);
        const double num = pick1 ? n1c : n2c, den = pick1 ? d1c : d2c;
        const double dt2 = (ok1 || ok2) ? num * frcp(den) : INFINITY;
        dt2min = dt2 < dt2min ? dt2 : dt2min;
        if (!(V > 0.0) || !isfinite(P)) {
          const int64_t gzi = ((d.lo[2] + p) * d.N[1] + gyz) * (int64_t)d.N[0] + gxz;  // global
          flag_error_zone(st, (V > 0.0) ? ERR_NONFINITE : ERR_TANGLED, gzi);
        }
      }
      ax0 = fx[0]; ay0 = fy[0]; az0 = fz[0];  // x-low face
      bx0 = fx[2]; by0 = fy[2]; bz0 = fz[2];  // y-low face
      cx0 = fx[4]; cy0 = fy[4]; cz0 = fz[4];  // z-low face (node plane p)
      PS[t] = P;
      __syncthreads();
    } else {
      double X[7], Y[7], Z[7];  // corners 0..6 (corner 7 lies on no low face)
      X[0] = xa.x; Y[0] = xa.y; Z[0] = xa.z;
      X[4] = xb.x; Y[4] = xb.y; Z[4] = xb.z;
#pragma unroll
      for (int l = 1; l < 7; ++l) {
        if (l == 4) continue;
        const int n = nidx + ((l >> 1) & 1) * T::BXN + (l & 1);
        const double *S = (l >> 2) ? Xb : Xa;
        X[l] = S[n]; Y[l] = S[RS + n]; Z[l] = S[2 * RS + n];
      }
      HYDRO_FACE(X, Y, Z, 6, 0, 4, 2, ax0, ay0, az0);  // x-low (AX_0)
      HYDRO_FACE(X, Y, Z, 5, 0, 1, 4, bx0, by0, bz0);  // y-low (AY_0)
      HYDRO_FACE(X, Y, Z, 3, 0, 2, 1, cx0, cy0, cz0);  // z-low (AZ_0, node plane p)
      im = m;  // the ring's first field is 1/m here (0 outside the mesh)
    }
    if (FUSED) im = exists ? im : 0.0;
    // ---------------------------------------------------------------- G
    const double gxw = (tx > 0) ? 0.125 * (PS[tc - 1] - P) : 0.0;
    const double gyw = (ty > 0) ? 0.125 * (PS[tc - PX] - P) : 0.0;
    const double gzw = 0.125 * (pv.P - P);
    st3(GX, t, gxw * ax0, gxw * ay0, gxw * az0);
    st3(GY, t, gyw * bx0, gyw * by0, gyw * bz0);
    st3(GZ, t, gzw * cx0, gzw * cy0, gzw * cz0);
    if (FUSED) {
      __syncthreads();
    } else {
      arrive(B_G);
      if (p >= k0 + 2) energy2(p - 2, cu);  // cu still holds zone plane p-2
      await(B_G, p);
    }
    cu.P = P; cu.im = im; cu.e = e;
    cu.ax = ax0; cu.ay = ay0; cu.az = az0;
    cu.bx = bx0; cu.by = by0; cu.bz = bz0;
    // ---------------------------------------------------------------- N
    double uh = 0.0, vh = 0.0, wh = 0.0;
    double Cx = 0.0, Cy = 0.0, Cz = 0.0;
    if (fl & F_NODE) {
      const int tn = tc - PX;  // zone (tx, ty-1)
      double a0, a1, a2_, b0, b1, b2;
      ld3(GX, tn, a0, a1, a2_);      // g_x of zone (tx, ty-1)
      ld3(GY, tc - 1, b0, b1, b2);   // g_y of zone (tx-1, ty)
      // own faces' g enter fused (g = w A, not re-read): same value to within one rounding
      Cx = fma(gxw, ax0, a0) + fma(gyw, bx0, b0);
      Cy = fma(gxw, ay0, a1) + fma(gyw, by0, b1);
      Cz = fma(gxw, az0, a2_) + fma(gyw, bz0, b2);
      if (p >= k0) {
        double c0, c1, c2_;
        ld3(GZ, tn - 1, a0, a1, a2_);
        ld3(GZ, tn, b0, b1, b2);
        ld3(GZ, tc - 1, c0, c1, c2_);
        const double Fx = pv.Sx + Cx + ((a0 + b0) + fma(gzw, cx0, c0));
        const double Fy = pv.Sy + Cy + ((a1 + b1) + fma(gzw, cy0, c1));
        const double Fz = pv.Sz + Cz + ((a2_ + b2) + fma(gzw, cz0, c2_));
        const double rinv =  // 8 / nodal mass (constant d.mn8)
            HYDRO_MN8_TMA ? Ra[6 * RS + nidx] : rinv_g;
        const bool wall_z = p == wz_lo || p == wz_hi;
        const double axc = (fl & F_WX) ? 0.0 : Fx * rinv;
        const double ayc = (fl & F_WY) ? 0.0 : Fy * rinv;
        const double azc = wall_z ? 0.0 : Fz * rinv;
        const double u = Ra[3 * RS + nidx], v = Ra[4 * RS + nidx], w = Ra[5 * RS + nidx];
        const double un = u + dt * axc, vn = v + dt * ayc, wn = w + dt * azc;
        uh = (u + un) * 0.5;
        vh = (v + vn) * 0.5;
        wh = (w + wn) * 0.5;
        st3(UH, tc, uh, vh, wh);
        if ((fl & F_NWR) && (p < k1 || p == n2)) {
          const int id = (p + 1) * nsxy + nrow;
          d.xn[id] = fma(hh, un, xa.x);  // x + dt u_half = x_p + dt/2 u' (reading R21)
          d.yn[id] = fma(hh, vn, xa.y);
          d.zn[id] = fma(hh, wn, xa.z);
          d.un[id] = un;
          d.vn[id] = vn;
          d.wn[id] = wn;
        }
      }
    }
    cu.Sx = Cx; cu.Sy = Cy; cu.Sz = Cz;  // every set member is written every plane (short ranges)
    cu.uh = uh; cu.vh = vh; cu.wh = wh;
    // ---------------------------------------------------------------- phase 3: X(p+2), E1(p-1)
    if (FUSED) {
      __syncthreads();
      if (t == 0 && p + 3 <= k1 + 1) issue(p + 3);  // slot of plane p, free after N(p)
    } else {
      arrive(B_U);
    }
    if (p + 2 <= k1 + 1) {  // x_p of plane p+2 into the registers of plane p (Z(p) done)
      wait_plane(p + 2);
      form_xp(p + 2, xa.x, xa.y, xa.z);
    }
    if (!FUSED) {
      await(B_U, p);
      if (t == 0 && p + 3 <= k1 + 1) issue(p + 3);  // slot of plane p, free after N(p)
    }
    {
      // E1 runs on every plane and lane (results of planes < k0+1 and of lanes whose faces do not
      // matter are never read): u_half of nodes (tx+1, ty), (tx, ty+1), (tx+1, ty+1) on plane p;
      // with the values of plane p-1 they give the neighbours' two-plane sums
      const double vsx = pv.uh + uh, vsy = pv.vh + vh, vsz = pv.wh + wh;  // own two-plane sum
      double a0, a1, a2_, b0, b1, b2, c0, c1, c2_;
      ld3(UH, tc + 1, a0, a1, a2_);
      ld3(UH, tc + PX, b0, b1, b2);
      ld3(UH, tc + PX + 1, c0, c1, c2_);
      // x-low face of zone plane p-1: nodes (tx, ty..ty+1), planes p-1, p
      const double psx = pv.ax * (vsx + (pv.nyu + b0)) + pv.ay * (vsy + (pv.nyv + b1)) +
                         pv.az * (vsz + (pv.nyw + b2));
      // y-low face of zone plane p-1: nodes (tx..tx+1, ty), planes p-1, p
      const double psy = pv.bx * (vsx + (pv.nxu + a0)) + pv.by * (vsy + (pv.nxv + a1)) +
                         pv.bz * (vsz + (pv.nxw + a2_));
      PSX[t] = psx;
      PSY[t] = psy;
      // z-face at node plane p: nodes (tx..tx+1, ty..ty+1)
      const double psi_zhigh = cx0 * ((uh + a0) + (b0 + c0)) + cy0 * ((vh + a1) + (b1 + c1)) +
                               cz0 * ((wh + a2_) + (b2 + c2_));
      cu.nxu = a0; cu.nxv = a1; cu.nxw = a2_;
      cu.nyu = b0; cu.nyv = b1; cu.nyw = b2;
      // E2 of zone plane p-1 runs in the next phase 1: W = P/8 (psi_xhi - psi_x + psi_yhi - psi_y
      // + psi_zhi - psi_zlo) with the high-face psi read from the neighbours
      pv.part = ((psi_zhigh - pv.psiz) - psx) - psy;
      cu.psiz = psi_zhigh;
    }
    if (FUSED) __syncthreads();
    else arrive(B_P);
    if (p == k1 && k1 >= k0 + 1) {  // the last pending E2 (zone plane k1-1)
      if (!FUSED) await(B_P, p);
      energy2(k1 - 1, pv);
    }
  };
  for (int p = k0 - 1; p <= k1; p += 2) {
    body(p, S0, S1, XA, XB);
    if (p + 1 > k1) break;
    body(p + 1, S1, S0, XB, XA);
  }
  ubase += (uint32_t)(k1 + 2 - q0);  // node planes q0 .. k1+1 went through the TMA ring
  pbase += (uint32_t)(k1 + 1 - q0);  // iterations p = q0 .. k1 completed each phase barrier
  __syncthreads();                   // the next segment reuses the rings
  if (!FUSED && npush) push_halo(i0, j0, k0, k1);
  }
  if (FUSED) block_min_dt_smem(sqrt(dt2min), &st->dtz_acc, sm + T::OFF_RED);
  if (fold_finalize)  // single-domain, single-rank cycle: S9 here instead of a separate launch
    finalize_if_last_block(st, ph, reinterpret_cast<unsigned int *>(sm + T::OFF_RED));
}

// Node-stage tile: 32 x CTY zones (+ ring).  Two heights are compiled, 12 (512 threads) and 11
// (480 threads); node_tile_ty picks one per domain from the wave-quantisation model below
// (measured: 128^3 85.3 vs 89.7 us with TY = 11, weak 384^3 slabs 499.7 vs 473.8 with TY = 12).
// The grouped launch and the one-kernel variant use CTY.
constexpr int CTX = 32, CTY = 12, CTY_ALT = 11;
// one-kernel variant's tile height (HYDRO_FUSED_TY at build time; default CTY): smaller tiles
// give each thread more registers (NTHR threads at one CTA per SM)
#ifndef HYDRO_FUSED_TY
#define HYDRO_FUSED_TY 12
#endif
constexpr int FTY = HYDRO_FUSED_TY;

// z-chunk length of the chunked schedule: minimise (waves of CTAs) x (planes per CTA incl. the
// 2 warm-up planes + a fixed per-chunk overhead of 1.4 plane-equivalents: pipeline fill and
// drain, prologue).  The overhead term was fitted on the B200 at 128^3 (44 tile columns:
// kz = 43 / 22 / 13 / 8 -> 89.5 / 97.3 / 95.0 / 109.8 us, i.e. 1 / 2 / 3 / 5 waves); without it
// the model ties kz = 13 (3 waves x 15 planes) with kz = 43 (1 wave x 45) and took the slower.
int64_t chunk_cost(int64_t ctas, int kz, int sms) {
  return ((ctas + sms - 1) / sms) * (10 * (int64_t)(kz + 2) + 14);
}

int choose_kz(int tiles, int n2, int sms) {
  int best = n2;
  int64_t best_cost = INT64_MAX;
  for (int kz = 4; kz <= n2; ++kz) {
    const int64_t cost = chunk_cost((int64_t)tiles * ((n2 + kz - 1) / kz), kz, sms);
    if (cost < best_cost) {
      best_cost = cost;
      best = kz;
    }
  }
  return std::min(best, n2);
}

// The shared-memory opt-in is a per-device function attribute: cached per device ordinal.
int cur_device() {
  int dev = 0;
  cudaGetDevice(&dev);
  return dev < 0 ? 0 : (dev >= 64 ? 63 : dev);
}

template <bool FUSED, int TY>
void set_smem() {
  static bool done_dev[64] = {};
  bool &done = done_dev[cur_device()];
  if (!done) {
    using T = CTile<CTX, TY>;
    cudaFuncSetAttribute(k_cycle<CTX, TY, FUSED, false>,
                         cudaFuncAttributeMaxDynamicSharedMemorySize, (int)T::BYTES);
    if constexpr (!FUSED && TY == CTY)
      cudaFuncSetAttribute(k_cycle<CTX, CTY, false, true>,
                           cudaFuncAttributeMaxDynamicSharedMemorySize, (int)T::BYTES);
    done = true;
  }
}

int num_sms() {
  static int sms_dev[64] = {};
  const int dev = cur_device();
  int &sms = sms_dev[dev];
  if (!sms) cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  return sms;
}

// Modelled node-stage cost of one domain with tile height TY: best chunking's
// chunk_cost x threads per CTA (per-plane time ~ CTA size at one CTA per SM).
template <int TY>
int64_t tile_cost(int n0, int n1, int n2, int sms) {
  const int tiles = ((n0 + CTX - 1) / CTX) * ((n1 + TY - 1) / TY);
  const int kz = choose_kz(tiles, n2, sms);
  return chunk_cost((int64_t)tiles * ((n2 + kz - 1) / kz), kz, sms) * CTile<CTX, TY>::NTHR;
}

template <bool FUSED, int TY>
void launch(const DomView &d, const NodeMaps &maps, const Phys &ph, DevState *st, int fold,
            const PushSlab *push, int npush, cudaStream_t s) {
  using T = CTile<CTX, TY>;
  set_smem<FUSED, TY>();
  const int sms = num_sms();
  const int tx = (d.n[0] + CTX - 1) / CTX, ty = (d.n[1] + TY - 1) / TY;
  // Default: the chunked schedule (CTAs adjacent in x, y at the same z-chunk, so the tile rings
  // that neighbouring CTAs both read are L2 hits; measured faster here than the persistent
  // linearised split, which spreads concurrent CTAs over z: 94 vs 110 us at 128^3).
  // HYDRO_KZ_NODE / HYDRO_KZ_FUSED = k: chunks of k planes; = -1: the persistent split.
  static const int kz_env = getenv(FUSED ? "HYDRO_KZ_FUSED" : "HYDRO_KZ_NODE")
                                ? atoi(getenv(FUSED ? "HYDRO_KZ_FUSED" : "HYDRO_KZ_NODE")) : 0;
  // HYDRO_NODE_PERSIST=0: one CTA per (column, chunk) unit instead of an SM-count grid that
  // walks the units (A/B)
  static const int persist = getenv("HYDRO_NODE_PERSIST") ? atoi(getenv("HYDRO_NODE_PERSIST")) : 1;
  const int ncols = tx * ty;
  int G, kz = 0;
  if (kz_env >= 0) {
    kz = kz_env > 0 ? std::min(kz_env, d.n[2]) : choose_kz(ncols, d.n[2], sms);
    G = ncols * ((d.n[2] + kz - 1) / kz);
    if (persist && !FUSED) G = std::min(G, sms);
  } else {
    G = (int)std::min<int64_t>(sms, (int64_t)ncols * d.n[2]);
  }
  launch_pdl(k_cycle<CTX, TY, FUSED, false>, dim3(G), dim3(T::NTHR), T::BYTES, s, maps, d, ph,
             st, tx, ncols, kz, fold, (const NodeTask *)nullptr, 0, (const DomView *)nullptr,
             (const NodeMaps *)nullptr, push, npush);
}

}  // namespace

size_t fused_smem_bytes() { return CTile<CTX, FTY>::BYTES; }
int fused_box_y() { return CTile<CTX, FTY>::BYN; }
int node_box_y(int ty) { return ty + 3; }  // CTile<CTX, ty>::BYN
int cycle_zone_box_x() { return CTile<CTX, CTY>::ZBX; }
int cycle_zone_box_y(int ty) {
  return ty + 2;  // CTile<CTX, ty>::ZBY
}

int node_tile_ty(int n0, int n1, int n2) {
  // read per call (host side, at create): tests force either height within one process
  const int force = getenv("HYDRO_NODE_TY") ? atoi(getenv("HYDRO_NODE_TY")) : 0;
  if (force == CTY || force == CTY_ALT) return force;
  const int sms = num_sms();
  return tile_cost<CTY_ALT>(n0, n1, n2, sms) < tile_cost<CTY>(n0, n1, n2, sms) ? CTY_ALT : CTY;
}

void launch_cycle_fused(const DomView &d, const NodeMaps &maps, const Phys &ph, DevState *st,
                        int fold_finalize, cudaStream_t s) {
  launch<true, FTY>(d, maps, ph, st, fold_finalize, nullptr, 0, s);
}
int fused_tile_ty() { return FTY; }

void launch_node_energy(const DomView &d, const NodeMaps &maps, const Phys &ph, DevState *st,
                        int fold_finalize, const PushSlab *push, int npush, int ty,
                        cudaStream_t s) {
  if (ty == CTY_ALT)
    launch<false, CTY_ALT>(d, maps, ph, st, fold_finalize, push, npush, s);
  else
    launch<false, CTY>(d, maps, ph, st, fold_finalize, push, npush, s);
}

int node_group_tasks(const DomView *views_host, int n, NodeTask *out) {
  // one z-chunk length for all domains: minimise (waves of all CTAs) x (chunk + 2 warm-up
  // planes) over the concatenated grid, as choose_kz does for one domain
  const int sms = num_sms();
  int nzmax = 1;
  for (int i = 0; i < n; ++i) nzmax = std::max(nzmax, views_host[i].n[2]);
  int best = nzmax;
  int64_t best_cost = INT64_MAX;
  for (int kz = 4; kz <= nzmax; ++kz) {
    int64_t ctas = 0;
    for (int i = 0; i < n; ++i) {
      const DomView &d = views_host[i];
      const int cols = ((d.n[0] + CTX - 1) / CTX) * ((d.n[1] + CTY - 1) / CTY);
      ctas += (int64_t)cols * ((d.n[2] + kz - 1) / kz);
    }
    const int64_t cost = chunk_cost(ctas, kz, sms);
    if (cost < best_cost) {
      best_cost = cost;
      best = kz;
    }
  }
  int cta = 0;
  for (int i = 0; i < n; ++i) {
    const DomView &d = views_host[i];
    NodeTask &T = out[i];
    T.slot = i;
    T.tcols = (d.n[0] + CTX - 1) / CTX;
    T.ncols = T.tcols * ((d.n[1] + CTY - 1) / CTY);
    T.kz = std::min(best, d.n[2]);
    T.cta0 = cta;
    T.push0 = 0;
    T.npush = 0;  // filled by the runtime when the fused halo is on
    cta += T.ncols * ((d.n[2] + T.kz - 1) / T.kz);
  }
  return cta;
}

void launch_node_energy_group(const NodeTask *tasks_dev, int ntasks, int nctas,
                              const DomView *views_dev, const NodeMaps *maps_dev, const Phys &ph,
                              DevState *st, const PushSlab *push, cudaStream_t s) {
  using T = CTile<CTX, CTY>;
  set_smem<false, CTY>();
  DomView d0 = {};
  NodeMaps m0 = {};
  launch_pdl(k_cycle<CTX, CTY, false, true>, dim3(nctas), dim3(T::NTHR), T::BYTES, s, m0, d0,
             ph, st, 0, 0, 0, 0, tasks_dev, ntasks, views_dev, maps_dev, push, 0);
}

}  // namespace hydro
