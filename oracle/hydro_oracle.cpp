// hydro_oracle.cpp -- TEST INFRASTRUCTURE ONLY (see hydro_oracle.h).
//
// A plain, slow, obviously-correct single-threaded fp64 implementation of one explicit
// staggered-grid Lagrangian hydro cycle on a domain-decomposed structured 3-D mesh.
//
// Sources.  PAPER.md fixes the workload (3-D Sedov blast wave, L637-642; "80 kernels" of hydro,
// L672), the block-structured mesh split into domains owned by ranks that exchange a halo
// (L307-310, L525-557), and the hierarchical split (L559-572).  The paper never states the
// hydro equations, so the cycle below is SURVEY.md §8c "SG" (single-geometry-pass compatible
// predictor), restated in DESIGN.md §3 together with every reading R1-R18 it relies on.  The
// step labels S1..S9 are those of SURVEY.md §8c.3; each function says which step it is.
//
// Decomposition: every domain keeps one ghost layer of zones and nodes.  Interface nodes are
// owned by both neighbours and are recomputed by each from identical inputs, so a decomposed
// run is bitwise equal to an undecomposed one (pinned by tests).
//
// Nothing here is blocked, fused or reordered beyond the summation orders written in §8c.
#include "hydro_oracle.h"

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstring>
#include <limits>
#include <string>
#include <vector>

namespace {

thread_local std::string g_err;

const double INF = std::numeric_limits<double>::infinity();
const double THIRD = 1.0 / 3.0;  // reading R3: the constant as a double

inline double sgn(int bit, double v) { return bit ? v : -v; }  // s(0)=-1, s(1)=+1 (exact)

// Face vector, 0.5 * (a x b), component order of SURVEY.md §8c.2.
inline void cross_half(const double a[3], const double b[3], double o[3]) {
  o[0] = 0.5 * (a[1] * b[2] - a[2] * b[1]);
  o[1] = 0.5 * (a[2] * b[0] - a[0] * b[2]);
  o[2] = 0.5 * (a[0] * b[1] - a[1] * b[0]);
}
inline void sub3(const double a[3], const double b[3], double o[3]) {
  o[0] = a[0] - b[0];
  o[1] = a[1] - b[1];
  o[2] = a[2] - b[2];
}
inline double dot3(const double a[3], const double b[3]) {
  return (a[0] * b[0] + a[1] * b[1]) + a[2] * b[2];
}

// S2 geometry (readings R2, R3, R4).
//   AX(a): x-face at i+a, AY(b): y-face at j+b, AZ(c): z-face at k+c, oriented +x/+y/+z.
//   B_l = 0.25*((s(a)AX_a + s(b)AY_b) + s(c)AZ_c);  V = THIRD * sum_{l=1..7} (X_l-X_0).B_l;
//   L = V / sqrt(max_faces |A|^2).
void geometry(const double X[8][3], double B[8][3], double *V, double *L) {
  double AX[2][3], AY[2][3], AZ[2][3], d1[3], d2[3];
  for (int a = 0; a < 2; ++a) {  // X(i+a,j+1,k+1)-X(i+a,j,k)  x  X(i+a,j,k+1)-X(i+a,j+1,k)
    sub3(X[a + 6], X[a], d1);
    sub3(X[a + 4], X[a + 2], d2);
    cross_half(d1, d2, AX[a]);
  }
  for (int b = 0; b < 2; ++b) {  // X(i+1,j+b,k+1)-X(i,j+b,k)  x  X(i+1,j+b,k)-X(i,j+b,k+1)
    sub3(X[1 + 2 * b + 4], X[2 * b], d1);
    sub3(X[1 + 2 * b], X[2 * b + 4], d2);
    cross_half(d1, d2, AY[b]);
  }
  for (int c = 0; c < 2; ++c) {  // X(i+1,j+1,k+c)-X(i,j,k+c)  x  X(i,j+1,k+c)-X(i+1,j,k+c)
    sub3(X[3 + 4 * c], X[4 * c], d1);
    sub3(X[2 + 4 * c], X[1 + 4 * c], d2);
    cross_half(d1, d2, AZ[c]);
  }
  for (int l = 0; l < 8; ++l) {
    const int a = l & 1, b = (l >> 1) & 1, c = (l >> 2) & 1;
    for (int d = 0; d < 3; ++d)
      B[l][d] = 0.25 * ((sgn(a, AX[a][d]) + sgn(b, AY[b][d])) + sgn(c, AZ[c][d]));
  }
  double s = 0.0, r[3];
  for (int l = 1; l < 8; ++l) {
    sub3(X[l], X[0], r);
    const double t = dot3(r, B[l]);
    s = (l == 1) ? t : s + t;
  }
  *V = THIRD * s;
  const double *faces[6] = {AX[0], AX[1], AY[0], AY[1], AZ[0], AZ[1]};
  double a2max = 0.0;
  for (int f = 0; f < 6; ++f) {
    const double a2 = dot3(faces[f], faces[f]);
    a2max = (f == 0) ? a2 : std::max(a2max, a2);
  }
  *L = *V / std::sqrt(a2max);
}

struct Params {
  double gamma, gm1, ggm1, q_lin, q_quad, cfl, c_vol;
  double hg;  // hourglass coefficient kappa (reading R17; 0 = off)
  int q_kind = 0;  // 0 scalar q (reading R7), 1 monotone q (reading R24)
};

// f1 / reading R24: the zone's strain rate along each logical direction d (0 = xi, 1 = eta,
// 2 = zeta): face-centre differences dx_d = (mean of the 4 corners with bit d = 1) - (mean with
// bit d = 0), du_d likewise for the velocities (corner sums in ascending l, first term
// initialising); L_d = |dx_d|; eps_d = (du_d . dx_d) / (dx_d . dx_d).
void strain(const double X[8][3], const double U[8][3], double eps[3], double L[3]) {
  for (int d = 0; d < 3; ++d) {
    double xs[2][3], us[2][3];
    bool first[2] = {true, true};
    for (int l = 0; l < 8; ++l) {
      const int side = (l >> d) & 1;
      for (int k = 0; k < 3; ++k) {
        xs[side][k] = first[side] ? X[l][k] : xs[side][k] + X[l][k];
        us[side][k] = first[side] ? U[l][k] : us[side][k] + U[l][k];
      }
      first[side] = false;
    }
    double dx[3], du[3];
    for (int k = 0; k < 3; ++k) {
      dx[k] = 0.25 * (xs[1][k] - xs[0][k]);
      du[k] = 0.25 * (us[1][k] - us[0][k]);
    }
    const double L2 = dot3(dx, dx);
    eps[d] = dot3(du, dx) / L2;
    L[d] = std::sqrt(L2);
  }
}

// Reading R24: monotonic limiter of direction d from the strain rates of the zone (e0) and of its
// two neighbours along d (em, ep): phi = max(0, min(1/2 (rm + rp), 2 rm, 2 rp, 1)) with
// r = e_neighbour / e0 (the MC-type limiter of Christensen / LULESH); phi = 1 when e0 = 0.
double mono_limiter(double em, double e0, double ep) {
  if (e0 == 0.0) return 1.0;
  const double rm = em / e0, rp = ep / e0;
  double phi = 0.5 * (rm + rp);
  phi = std::min(phi, 2.0 * rm);
  phi = std::min(phi, 2.0 * rp);
  phi = std::min(phi, 1.0);
  return std::max(phi, 0.0);
}

struct ZoneOut {
  double rho, ep, p, c, q, P, dtz, V, L, D;
};

// S2 (DV, rho, D) + S3 (predictor, EOS) + S4 (q, P) + S6 (dt_z) for one zone
// (readings R5-R8).  X are the half-step positions x_p, U the velocities u^n.
// phi (reading R24, q_kind 1): the zone's three limiter values; nullptr for the scalar q.
void zone_state(const double X[8][3], const double U[8][3], double m, double e, double hh,
                const Params &pr, double B[8][3], ZoneOut *o, const double *phi = nullptr) {
  double V, L;
  geometry(X, B, &V, &L);
  double DV = 0.0;
  for (int l = 0; l < 8; ++l) {
    const double t = dot3(U[l], B[l]);
    DV = (l == 0) ? t : DV + t;
  }
  const double inv = 1.0 / V;
  const double rho = m * inv;
  const double D = DV * inv;
  // S3
  const double epos = std::max(e, 0.0);
  const double pt = (pr.gm1 * rho) * epos;
  const double ep = e - ((hh * pt) * DV) / m;
  const double eppos = std::max(ep, 0.0);
  const double p = (pr.gm1 * rho) * eppos;
  const double c = std::sqrt(pr.ggm1 * eppos);
  // S4
  double qr = 0.0;
  if (D < 0.0 && !phi) {
    const double s = L * (-D);
    qr = s * ((pr.q_quad * s) + (pr.q_lin * c));
  } else if (D < 0.0) {  // reading R24: per direction, limited by the neighbours' strain rates
    double eps[3], Ld[3];
    strain(X, U, eps, Ld);
    for (int d = 0; d < 3; ++d) {
      const double dv = Ld[d] * std::max(-eps[d], 0.0);
      const double t = ((pr.q_quad * dv) * dv) * (1.0 - phi[d] * phi[d]) +
                       ((pr.q_lin * c) * dv) * (1.0 - phi[d]);
      qr = (d == 0) ? t : qr + t;
    }
  }
  const double q = rho * qr;
  const double P = p + q;
  // S6
  const double sig = std::sqrt(c * c + 2.0 * qr);
  const double dtc = (sig > 0.0) ? (pr.cfl * L) / sig : INF;
  const double dtv = (D != 0.0) ? pr.c_vol / std::fabs(D) : INF;
  o->rho = rho;
  o->ep = ep;
  o->p = p;
  o->c = c;
  o->q = q;
  o->P = P;
  o->dtz = std::min(dtc, dtv);
  o->V = V;
  o->L = L;
  o->D = D;
}

// S5 addition, SURVEY §8f row f1 / reading R17: viscous hourglass control in
// the Flanagan-Belytschko form, added to the corner forces f_l = P B_l (so it is still a corner
// force: momentum and, through the compatible S8 update, total energy stay conserved).
//   base vectors on the reference cube, corner l = a+2b+4c, xi = 2a-1, eta = 2b-1, zeta = 2c-1:
//     h1 = eta*zeta, h2 = zeta*xi, h3 = xi*eta, h4 = xi*eta*zeta;
//   M_dk = sum_l B_ld X_lk  (= V delta_dk when B is the exact gradient of V: affine hexes),
//   H_ak = sum_l h_al X_lk,  C = H M^-1,
//   gamma_al = h_al - sum_d C_ad B_ld   (sum_l gamma_al = 0 and sum_l gamma_al X_lk = 0 exactly
//                                        in real arithmetic: linear velocity fields are immune),
//   g_ad = sum_l gamma_al U_ld,
//   f_hg_ld = -kappa rho c V^(2/3) sum_a gamma_al g_ad.
// X: half-step positions, U: u^n, B/V/rho/c: the zone's S2-S3 values (same as for P).
void hourglass(const double X[8][3], const double U[8][3], const double B[8][3], double V,
               double rho, double c, double kappa, double F[8][3]) {
  double h[4][8];
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
      double sum = 0.0;
      for (int l = 0; l < 8; ++l) sum = (l == 0) ? B[l][d] * X[l][k] : sum + B[l][d] * X[l][k];
      M[d][k] = sum;
    }
  for (int a = 0; a < 4; ++a)
    for (int k = 0; k < 3; ++k) {
      double sum = 0.0;
      for (int l = 0; l < 8; ++l) sum = (l == 0) ? h[a][l] * X[l][k] : sum + h[a][l] * X[l][k];
      H[a][k] = sum;
    }
  // M^-1 by the adjugate: Minv[k][d] = cof(M)[d][k] / det M
  double cof[3][3];
  for (int r = 0; r < 3; ++r)
    for (int q = 0; q < 3; ++q) {
      const int r1 = (r + 1) % 3, r2 = (r + 2) % 3, q1 = (q + 1) % 3, q2 = (q + 2) % 3;
      cof[r][q] = M[r1][q1] * M[r2][q2] - M[r1][q2] * M[r2][q1];
    }
  const double det = (M[0][0] * cof[0][0] + M[0][1] * cof[0][1]) + M[0][2] * cof[0][2];
  double Minv[3][3];
  for (int k = 0; k < 3; ++k)
    for (int d = 0; d < 3; ++d) Minv[k][d] = cof[d][k] / det;
  double C[4][3];
  for (int a = 0; a < 4; ++a)
    for (int d = 0; d < 3; ++d)
      C[a][d] = (H[a][0] * Minv[0][d] + H[a][1] * Minv[1][d]) + H[a][2] * Minv[2][d];
  double gam[4][8];
  for (int a = 0; a < 4; ++a)
    for (int l = 0; l < 8; ++l)
      gam[a][l] = h[a][l] - ((C[a][0] * B[l][0] + C[a][1] * B[l][1]) + C[a][2] * B[l][2]);
  double g[4][3];
  for (int a = 0; a < 4; ++a)
    for (int d = 0; d < 3; ++d) {
      double sum = 0.0;
      for (int l = 0; l < 8; ++l)
        sum = (l == 0) ? gam[a][l] * U[l][d] : sum + gam[a][l] * U[l][d];
      g[a][d] = sum;
    }
  const double v13 = std::cbrt(V);
  const double coef = -(((kappa * rho) * c) * (v13 * v13));
  for (int l = 0; l < 8; ++l)
    for (int d = 0; d < 3; ++d) {
      double sum = 0.0;
      for (int a = 0; a < 4; ++a) sum = (a == 0) ? gam[a][l] * g[a][d] : sum + gam[a][l] * g[a][d];
      F[l][d] = coef * sum;
    }
}

// ----------------------------------------------------------------------------------------
// Domains.  Owned zones [lo, lo+n) per axis (global).  Local zone index i in [-1, n] and node
// index i in [-1, n+1]; storage offset +1.  Only entries that exist in the global mesh are
// ever read.
struct Domain {
  int64_t lo[3], n[3], zs[3], ns[3];
  std::vector<double> x[3], u[3], xn[3], un[3], xp[3], uh[3];
  std::vector<double> m, e, en, P, B;  // B: 24 per zone
  std::vector<double> HG;              // hourglass corner forces, 24 per zone (kappa > 0 only)
  std::vector<double> eps[3];          // strain rates of the owned zones (monotone q only, R24)
  std::vector<uint8_t> zex, nex;       // exists in the global mesh

  int64_t zid(int64_t i, int64_t j, int64_t k) const {
    return ((k + 1) * zs[1] + (j + 1)) * zs[0] + (i + 1);
  }
  int64_t nid(int64_t i, int64_t j, int64_t k) const {
    return ((k + 1) * ns[1] + (j + 1)) * ns[0] + (i + 1);
  }
};

}  // namespace

struct orc_ctx {
  orc_config cfg;
  std::vector<int64_t> cuts[3];
  int64_t N[3];
  Params pr;
  std::vector<Domain> dom;
  int ndx, ndy, ndz;
  std::vector<int32_t> zown[3], nown[3];  // per axis: owning domain coordinate (lowest)
  double t, dt, dtzmin;
  double dt_floor;  // reading R23: 0 = none
  int64_t cycle;
  int failed;
  int64_t bad_zone;

  int dom_index(int a, int b, int c) const { return (c * ndy + b) * ndx + a; }
};

namespace {

bool exists_zone(const orc_ctx *h, const int64_t g[3]) {
  for (int a = 0; a < 3; ++a)
    if (g[a] < 0 || g[a] >= h->N[a]) return false;
  return true;
}
bool exists_node(const orc_ctx *h, const int64_t g[3]) {
  for (int a = 0; a < 3; ++a)
    if (g[a] < 0 || g[a] > h->N[a]) return false;
  return true;
}

// Initial node position, reading R1: o + (L*i)/n.
double init_coord(const orc_ctx *h, int a, int64_t g) {
  return h->cfg.origin[a] + (h->cfg.extent[a] * (double)g) / (double)h->N[a];
}

int64_t gnode(const orc_ctx *h, const int64_t g[3]) {
  return (g[2] * (h->N[1] + 1) + g[1]) * (h->N[0] + 1) + g[0];
}
int64_t gzone(const orc_ctx *h, const int64_t g[3]) {
  return (g[2] * h->N[1] + g[1]) * h->N[0] + g[0];
}

void gather_corners(const Domain &D, const std::vector<double> *pos, const std::vector<double> *vel,
                    int64_t i, int64_t j, int64_t k, double X[8][3], double U[8][3]) {
  for (int l = 0; l < 8; ++l) {
    const int64_t id = D.nid(i + (l & 1), j + ((l >> 1) & 1), k + ((l >> 2) & 1));
    for (int d = 0; d < 3; ++d) {
      X[l][d] = pos[d][id];
      U[l][d] = vel[d][id];
    }
  }
}

// S2-S6 at the initial state with no predictor (hh = 0): zone masses and dt^0 (SURVEY §8c.3
// "Start-up").
void init_domain(orc_ctx *h, Domain &D) {
  const orc_config &c = h->cfg;
  int64_t tot_z = D.zs[0] * D.zs[1] * D.zs[2], tot_n = D.ns[0] * D.ns[1] * D.ns[2];
  for (int d = 0; d < 3; ++d) {
    D.x[d].assign(tot_n, 0.0);
    D.u[d].assign(tot_n, 0.0);
    D.xn[d].assign(tot_n, 0.0);
    D.un[d].assign(tot_n, 0.0);
    D.xp[d].assign(tot_n, 0.0);
    D.uh[d].assign(tot_n, 0.0);
  }
  D.m.assign(tot_z, 0.0);
  D.e.assign(tot_z, 0.0);
  D.en.assign(tot_z, 0.0);
  D.P.assign(tot_z, 0.0);
  D.B.assign(tot_z * 24, 0.0);
  if (h->pr.hg > 0.0) D.HG.assign(tot_z * 24, 0.0);
  D.zex.assign(tot_z, 0);
  D.nex.assign(tot_n, 0);
  for (int64_t k = -1; k <= D.n[2] + 1; ++k)
    for (int64_t j = -1; j <= D.n[1] + 1; ++j)
      for (int64_t i = -1; i <= D.n[0] + 1; ++i) {
        const int64_t g[3] = {D.lo[0] + i, D.lo[1] + j, D.lo[2] + k};
        if (!exists_node(h, g)) continue;
        const int64_t id = D.nid(i, j, k);
        D.nex[id] = 1;
        if (c.init_kind == ORC_INIT_SEDOV) {
          for (int d = 0; d < 3; ++d) D.x[d][id] = init_coord(h, d, g[d]);
        } else {
          const int64_t gi = gnode(h, g);
          for (int d = 0; d < 3; ++d) {
            D.x[d][id] = c.user[d][gi];
            D.u[d][id] = c.user[3 + d][gi];
          }
        }
      }
  for (int64_t k = -1; k <= D.n[2]; ++k)
    for (int64_t j = -1; j <= D.n[1]; ++j)
      for (int64_t i = -1; i <= D.n[0]; ++i) {
        const int64_t g[3] = {D.lo[0] + i, D.lo[1] + j, D.lo[2] + k};
        if (!exists_zone(h, g)) continue;
        const int64_t id = D.zid(i, j, k);
        D.zex[id] = 1;
        double X[8][3], U[8][3], B[8][3], V, L;
        gather_corners(D, D.x, D.u, i, j, k, X, U);
        geometry(X, B, &V, &L);
        if (c.init_kind == ORC_INIT_SEDOV) {
          D.m[id] = c.rho0 * V;
          D.e[id] = (g[0] == 0 && g[1] == 0 && g[2] == 0) ? c.sedov_energy / D.m[id] : c.e0;
        } else if (c.init_kind == ORC_INIT_USER) {
          const int64_t gi = gzone(h, g);
          D.m[id] = c.user[6][gi] * V;
          D.e[id] = c.user[7][gi];
        } else {
          const int64_t gi = gzone(h, g);
          D.m[id] = c.user[6][gi];
          D.e[id] = c.user[7][gi];
        }
      }
}

// Ghost exchange: every ghost node / zone that exists globally takes the value of its owner
// (lowest owning domain index; interface copies are bitwise identical anyway).
void exchange(orc_ctx *h, bool nodes_new) {
  for (size_t di = 0; di < h->dom.size(); ++di) {
    Domain &D = h->dom[di];
    for (int64_t k = -1; k <= D.n[2] + 1; ++k)
      for (int64_t j = -1; j <= D.n[1] + 1; ++j)
        for (int64_t i = -1; i <= D.n[0] + 1; ++i) {
          const bool owned = i >= 0 && i <= D.n[0] && j >= 0 && j <= D.n[1] && k >= 0 &&
                             k <= D.n[2];
          if (owned) continue;
          const int64_t g[3] = {D.lo[0] + i, D.lo[1] + j, D.lo[2] + k};
          if (!exists_node(h, g)) continue;
          const int o = h->dom_index(h->nown[0][g[0]], h->nown[1][g[1]], h->nown[2][g[2]]);
          const Domain &S = h->dom[o];
          const int64_t sid = S.nid(g[0] - S.lo[0], g[1] - S.lo[1], g[2] - S.lo[2]);
          const int64_t id = D.nid(i, j, k);
          for (int d = 0; d < 3; ++d) {
            if (nodes_new) {
              D.xn[d][id] = S.xn[d][sid];
              D.un[d][id] = S.un[d][sid];
            } else {
              D.x[d][id] = S.x[d][sid];
              D.u[d][id] = S.u[d][sid];
            }
          }
        }
    for (int64_t k = -1; k <= D.n[2]; ++k)
      for (int64_t j = -1; j <= D.n[1]; ++j)
        for (int64_t i = -1; i <= D.n[0]; ++i) {
          const bool owned = i >= 0 && i < D.n[0] && j >= 0 && j < D.n[1] && k >= 0 &&
                             k < D.n[2];
          if (owned) continue;
          const int64_t g[3] = {D.lo[0] + i, D.lo[1] + j, D.lo[2] + k};
          if (!exists_zone(h, g)) continue;
          const int o = h->dom_index(h->zown[0][g[0]], h->zown[1][g[1]], h->zown[2][g[2]]);
          const Domain &S = h->dom[o];
          const int64_t sid = S.zid(g[0] - S.lo[0], g[1] - S.lo[1], g[2] - S.lo[2]);
          if (nodes_new)
            D.en[D.zid(i, j, k)] = S.en[sid];
          else
            D.e[D.zid(i, j, k)] = S.e[sid];
        }
  }
}

void fail(orc_ctx *h, int code, int64_t zone) {
  if (!h->failed) h->failed = code;
  if (zone >= 0 && (h->bad_zone < 0 || zone < h->bad_zone)) h->bad_zone = zone;
}

// Reading R24: the strain rates eps_d of every domain's owned zones at positions (x^n or x_p)
// and velocities u^n.  Neighbour values are then read from the owning domain by global index,
// so a ghost-ring zone's limiter sees exactly what its owner's does (decomposition-invariant).
void strain_pass(const orc_ctx *h, bool half_step) {
  for (const Domain &Dc : h->dom) {
    Domain &D = const_cast<Domain &>(Dc);  // a per-pass cache, also filled by get_fields
    const size_t tot_z = D.zex.size();
    for (int d = 0; d < 3; ++d) D.eps[d].assign(tot_z, 0.0);
    for (int64_t k = 0; k < D.n[2]; ++k)
      for (int64_t j = 0; j < D.n[1]; ++j)
        for (int64_t i = 0; i < D.n[0]; ++i) {
          double X[8][3], U[8][3], eps[3], L[3];
          gather_corners(D, half_step ? D.xp : D.x, D.u, i, j, k, X, U);
          strain(X, U, eps, L);
          for (int d = 0; d < 3; ++d) D.eps[d][D.zid(i, j, k)] = eps[d];
        }
  }
}

double eps_global(const orc_ctx *h, const int64_t g[3], int d) {
  const Domain &S = h->dom[h->dom_index(h->zown[0][g[0]], h->zown[1][g[1]], h->zown[2][g[2]])];
  return S.eps[d][S.zid(g[0] - S.lo[0], g[1] - S.lo[1], g[2] - S.lo[2])];
}

// Reading R24: limiter values of global zone g.  A neighbour outside the mesh mirrors the zone
// at a reflecting wall (ratio 1) and has zero strain at a free boundary.
void mono_phi(const orc_ctx *h, const int64_t g[3], double phi[3]) {
  for (int d = 0; d < 3; ++d) {
    const double e0 = eps_global(h, g, d);
    int64_t gm[3] = {g[0], g[1], g[2]}, gp[3] = {g[0], g[1], g[2]};
    gm[d] -= 1;
    gp[d] += 1;
    const double em = exists_zone(h, gm) ? eps_global(h, gm, d)
                      : ((h->cfg.reflect_mask >> (2 * d)) & 1u) ? e0 : 0.0;
    const double ep = exists_zone(h, gp) ? eps_global(h, gp, d)
                      : ((h->cfg.reflect_mask >> (2 * d + 1)) & 1u) ? e0 : 0.0;
    phi[d] = mono_limiter(em, e0, ep);
  }
}

// One cycle S1..S9 over all domains, then the ghost exchange.
void cycle(orc_ctx *h) {
  const double dt = h->dt;
  const double hh = 0.5 * dt;  // S1
  const orc_config &c = h->cfg;
  double dtmin = INF;
  // S1: half-step positions for every existing local node (owned and ghost).
  for (Domain &D : h->dom) {
    const size_t nn = D.nex.size();
    for (size_t id = 0; id < nn; ++id) {
      if (!D.nex[id]) continue;
      for (int d = 0; d < 3; ++d) D.xp[d][id] = D.x[d][id] + hh * D.u[d][id];
    }
  }
  if (h->pr.q_kind == 1) strain_pass(h, true);  // R24: strain rates at the half step
  // S2-S6 for every existing local zone (owned and ghost); dt_z over owned zones.
  for (Domain &D : h->dom) {
    for (int64_t k = -1; k <= D.n[2]; ++k)
      for (int64_t j = -1; j <= D.n[1]; ++j)
        for (int64_t i = -1; i <= D.n[0]; ++i) {
          const int64_t id = D.zid(i, j, k);
          if (!D.zex[id]) continue;
          double X[8][3], U[8][3], B[8][3], phi[3];
          ZoneOut o;
          gather_corners(D, D.xp, D.u, i, j, k, X, U);
          if (h->pr.q_kind == 1) {
            const int64_t gg[3] = {D.lo[0] + i, D.lo[1] + j, D.lo[2] + k};
            mono_phi(h, gg, phi);
          }
          zone_state(X, U, D.m[id], D.e[id], hh, h->pr, B, &o,
                     h->pr.q_kind == 1 ? phi : nullptr);
          std::memcpy(&D.B[id * 24], B, sizeof(B));
          D.P[id] = o.P;  // S5 f_l = P*B_l is formed where it is used (same bits)
          if (h->pr.hg > 0.0) {  // f1: f_l = P*B_l + f_hg_l
            double Fh[8][3];
            hourglass(X, U, B, o.V, o.rho, o.c, h->pr.hg, Fh);
            std::memcpy(&D.HG[id * 24], Fh, sizeof(Fh));
          }
          const bool owned = i >= 0 && i < D.n[0] && j >= 0 && j < D.n[1] && k >= 0 &&
                             k < D.n[2];
          if (!owned) continue;
          const int64_t g[3] = {D.lo[0] + i, D.lo[1] + j, D.lo[2] + k};
          if (!(o.V > 0.0)) fail(h, ORC_ETANGLED, gzone(h, g));
          else if (!std::isfinite(o.P)) fail(h, ORC_ENONFINITE, gzone(h, g));
          dtmin = std::min(dtmin, o.dtz);
        }
  }
  // S7: nodal force gather, mass, acceleration, reflecting walls, velocity/position update.
  for (Domain &D : h->dom) {
    for (int64_t k = 0; k <= D.n[2]; ++k)
      for (int64_t j = 0; j <= D.n[1]; ++j)
        for (int64_t i = 0; i <= D.n[0]; ++i) {
          double F[3] = {0.0, 0.0, 0.0}, msum = 0.0;
          bool first = true;
          for (int lp = 0; lp < 8; ++lp) {
            const int ap = lp & 1, bp = (lp >> 1) & 1, cp = (lp >> 2) & 1;
            const int64_t zid = D.zid(i - 1 + ap, j - 1 + bp, k - 1 + cp);
            if (!D.zex[zid]) continue;
            const double *Bz = &D.B[zid * 24 + (7 - lp) * 3];
            const double P = D.P[zid];
            double f[3] = {P * Bz[0], P * Bz[1], P * Bz[2]};
            if (h->pr.hg > 0.0)
              for (int d = 0; d < 3; ++d) f[d] = f[d] + D.HG[zid * 24 + (7 - lp) * 3 + d];
            for (int d = 0; d < 3; ++d) F[d] = first ? f[d] : F[d] + f[d];
            msum = first ? D.m[zid] : msum + D.m[zid];
            first = false;
          }
          const double mp = 0.125 * msum;
          const double rinv = 1.0 / mp;
          double acc[3] = {F[0] * rinv, F[1] * rinv, F[2] * rinv};
          const int64_t g[3] = {D.lo[0] + i, D.lo[1] + j, D.lo[2] + k};
          for (int d = 0; d < 3; ++d) {
            if (g[d] == 0 && (c.reflect_mask >> (2 * d) & 1u)) acc[d] = 0.0;
            if (g[d] == h->N[d] && (c.reflect_mask >> (2 * d + 1) & 1u)) acc[d] = 0.0;
          }
          const int64_t id = D.nid(i, j, k);
          for (int d = 0; d < 3; ++d) {
            const double un = D.u[d][id] + dt * acc[d];
            const double uh = (D.u[d][id] + un) * 0.5;
            D.un[d][id] = un;
            D.uh[d][id] = uh;
            D.xn[d][id] = D.x[d][id] + dt * uh;
          }
        }
  }
  // S8: compatible internal-energy update for owned zones.
  for (Domain &D : h->dom) {
    for (int64_t k = 0; k < D.n[2]; ++k)
      for (int64_t j = 0; j < D.n[1]; ++j)
        for (int64_t i = 0; i < D.n[0]; ++i) {
          const int64_t id = D.zid(i, j, k);
          const double P = D.P[id];
          double W = 0.0;
          for (int l = 0; l < 8; ++l) {
            const int64_t nid = D.nid(i + (l & 1), j + ((l >> 1) & 1), k + ((l >> 2) & 1));
            const double *Bl = &D.B[id * 24 + l * 3];
            double f[3] = {P * Bl[0], P * Bl[1], P * Bl[2]};
            if (h->pr.hg > 0.0)
              for (int d = 0; d < 3; ++d) f[d] = f[d] + D.HG[id * 24 + l * 3 + d];
            const double uh[3] = {D.uh[0][nid], D.uh[1][nid], D.uh[2][nid]};
            const double t = dot3(f, uh);
            W = (l == 0) ? t : W + t;
          }
          D.en[id] = D.e[id] - (dt * W) / D.m[id];
        }
  }
  // S9: time and the next dt.
  const double tn = h->t + dt;
  double dtn = std::min(std::min(c.dt_growth * dt, c.dt_max), dtmin);
  if (c.t_stop > 0.0) dtn = std::min(dtn, c.t_stop - tn);
  // Ghost exchange of the new state, then the new state becomes current.
  exchange(h, true);
  for (Domain &D : h->dom) {
    for (int d = 0; d < 3; ++d) {
      D.x[d].swap(D.xn[d]);
      D.u[d].swap(D.un[d]);
    }
    D.e.swap(D.en);
  }
  h->t = tn;
  h->dtzmin = dtmin;
  h->dt = dtn;
  h->cycle += 1;
  const bool stop = c.t_stop > 0.0 && tn >= c.t_stop;
  if (!(std::isfinite(dtn) && dtn > 0.0) && !stop) fail(h, ORC_ENONFINITE, -1);
  // Reading R23: dt collapse.  The zone dt minimum of this cycle fell below the floor: the run
  // halts (state = the one after this cycle), a global condition, so no bad zone is named.
  if (!stop && dtmin < h->dt_floor) fail(h, ORC_EDTMIN, -1);
}

bool valid_config(const orc_config *c) {
  for (int a = 0; a < 3; ++a) {
    if (c->n[a] < 1 || c->ndom[a] < 1 || c->extent[a] <= 0.0) return false;
    if (c->cuts[a]) {
      if (c->cuts[a][0] != 0 || c->cuts[a][c->ndom[a]] != c->n[a]) return false;
      for (int d = 0; d < c->ndom[a]; ++d)
        if (c->cuts[a][d + 1] - c->cuts[a][d] < 1) return false;
    } else if (c->ndom[a] > c->n[a]) {
      return false;
    }
  }
  if (!(c->gamma > 1.0) || c->q_lin < 0.0 || c->q_quad < 0.0 || !(c->cfl > 0.0) ||
      !(c->c_vol > 0.0) || !(c->dt_growth > 0.0) || !(c->dt_max > 0.0) || !(c->hg_coef >= 0.0) ||
      c->q_kind < 0 || c->q_kind > 1)
    return false;
  if (c->init_kind != ORC_INIT_SEDOV) {
    for (int f = 0; f < 8; ++f)
      if (!c->user[f]) return false;
  }
  return true;
}

}  // namespace

extern "C" {

const char *orc_last_error(void) { return g_err.c_str(); }

void orc_zone_strain(const double X[8][3], const double U[8][3], double eps[3], double L[3]) {
  strain(X, U, eps, L);
}

double orc_mono_limiter(double em, double e0, double ep) { return mono_limiter(em, e0, ep); }

void orc_zone_hourglass(const double X[8][3], const double U[8][3], const double B[8][3],
                        double V, double rho, double c, double kappa, double F[8][3]) {
  hourglass(X, U, B, V, rho, c, kappa, F);
}

void orc_zone_geometry(const double X[8][3], double B[8][3], double *V, double *L) {
  geometry(X, B, V, L);
}

void orc_zone_state(const double X[8][3], const double U[8][3], double m, double e, double hh,
                    double gamma, double q_lin, double q_quad, double cfl, double c_vol,
                    double out[8]) {
  Params pr{gamma, gamma - 1.0, gamma * (gamma - 1.0), q_lin, q_quad, cfl, c_vol, 0.0};
  double B[8][3];
  ZoneOut o;
  zone_state(X, U, m, e, hh, pr, B, &o);
  out[0] = o.rho;
  out[1] = o.ep;
  out[2] = o.p;
  out[3] = o.c;
  out[4] = o.q;
  out[5] = o.P;
  out[6] = o.dtz;
  out[7] = o.V;
}

int orc_create(const orc_config *cfg, orc_ctx **out) {
  if (!cfg || !out) return ORC_EINVAL;
  *out = nullptr;
  if (!valid_config(cfg)) {
    g_err = "invalid config";
    return ORC_EINVAL;
  }
  orc_ctx *h = new orc_ctx();
  h->cfg = *cfg;
  h->failed = 0;
  h->bad_zone = -1;
  for (int a = 0; a < 3; ++a) {
    h->N[a] = cfg->n[a];
    h->cuts[a].resize(cfg->ndom[a] + 1);
    for (int d = 0; d <= cfg->ndom[a]; ++d)
      h->cuts[a][d] = cfg->cuts[a] ? cfg->cuts[a][d] : (cfg->n[a] * d) / cfg->ndom[a];
    // owner tables (lowest domain coordinate containing the index)
    h->zown[a].assign(h->N[a], 0);
    h->nown[a].assign(h->N[a] + 1, 0);
    for (int64_t g = 0; g < h->N[a]; ++g) {
      int d = 0;
      while (!(h->cuts[a][d] <= g && g < h->cuts[a][d + 1])) ++d;
      h->zown[a][g] = d;
    }
    for (int64_t g = 0; g <= h->N[a]; ++g) {
      int d = 0;
      while (!(h->cuts[a][d] <= g && g <= h->cuts[a][d + 1])) ++d;
      h->nown[a][g] = d;
    }
  }
  h->ndx = cfg->ndom[0];
  h->ndy = cfg->ndom[1];
  h->ndz = cfg->ndom[2];
  h->pr = Params{cfg->gamma, cfg->gamma - 1.0, cfg->gamma * (cfg->gamma - 1.0), cfg->q_lin,
                 cfg->q_quad, cfg->cfl, cfg->c_vol, cfg->hg_coef, cfg->q_kind};
  h->dom.resize((size_t)h->ndx * h->ndy * h->ndz);
  for (int c = 0; c < h->ndz; ++c)
    for (int b = 0; b < h->ndy; ++b)
      for (int a = 0; a < h->ndx; ++a) {
        Domain &D = h->dom[h->dom_index(a, b, c)];
        const int idx[3] = {a, b, c};
        for (int ax = 0; ax < 3; ++ax) {
          D.lo[ax] = h->cuts[ax][idx[ax]];
          D.n[ax] = h->cuts[ax][idx[ax] + 1] - D.lo[ax];
          D.zs[ax] = D.n[ax] + 2;
          D.ns[ax] = D.n[ax] + 3;
        }
        init_domain(h, D);
      }
  // dt^0: S2-S6 at x^0, e^0 with no predictor.
  double dtmin = INF;
  if (h->pr.q_kind == 1) strain_pass(h, false);
  for (Domain &D : h->dom)
    for (int64_t k = 0; k < D.n[2]; ++k)
      for (int64_t j = 0; j < D.n[1]; ++j)
        for (int64_t i = 0; i < D.n[0]; ++i) {
          const int64_t id = D.zid(i, j, k);
          double X[8][3], U[8][3], B[8][3], phi[3];
          ZoneOut o;
          gather_corners(D, D.x, D.u, i, j, k, X, U);
          if (h->pr.q_kind == 1) {
            const int64_t gg[3] = {D.lo[0] + i, D.lo[1] + j, D.lo[2] + k};
            mono_phi(h, gg, phi);
          }
          zone_state(X, U, D.m[id], D.e[id], 0.0, h->pr, B, &o,
                     h->pr.q_kind == 1 ? phi : nullptr);
          dtmin = std::min(dtmin, o.dtz);
          if (!(o.V > 0.0)) {
            const int64_t g[3] = {D.lo[0] + i, D.lo[1] + j, D.lo[2] + k};
            fail(h, ORC_ETANGLED, gzone(h, g));
          }
        }
  h->t = cfg->t0;
  h->cycle = 0;
  h->dtzmin = dtmin;
  h->dt = (cfg->dt_first > 0.0) ? cfg->dt_first
                                 : std::min(std::min(cfg->dt_init, cfg->dt_max), dtmin);
  // reading R23: the floor is relative to dt^0 (before the t_stop clamp) unless given
  h->dt_floor = cfg->dt_floor > 0.0 ? cfg->dt_floor
                : (cfg->dt_floor == 0.0 && std::isfinite(h->dt)) ? 1e-6 * h->dt : 0.0;
  if (cfg->t_stop > 0.0) h->dt = std::min(h->dt, cfg->t_stop - h->t);
  if (h->failed) {
    const int code = h->failed;
    g_err = "initial mesh is tangled";
    delete h;
    return code;
  }
  *out = h;
  return ORC_OK;
}

int orc_step(orc_ctx *h, int32_t ncycles, orc_info *info) {
  if (!h) return ORC_EINVAL;
  if (h->failed) return ORC_ESTATE;
  for (int32_t n = 0; n < ncycles; ++n) {
    if (h->cfg.t_stop > 0.0 && h->t >= h->cfg.t_stop) break;
    cycle(h);
    if (h->failed) break;
  }
  orc_info_get(h, info);
  return h->failed ? h->failed : ORC_OK;
}

int orc_info_get(const orc_ctx *h, orc_info *info) {
  if (!h) return ORC_EINVAL;
  if (info) {
    info->t = h->t;
    info->dt = h->dt;
    info->cycle = h->cycle;
    info->dt_min_zone = h->dtzmin;
    info->bad_zone = h->bad_zone;
  }
  return ORC_OK;
}

// Output fields (SURVEY §8c.3 "Outputs"): x, u; V, rho, p, c, q by S2-S4 at (x, u) with
// e_p = e (hh = 0); e; m.
int orc_get_fields(const orc_ctx *h, uint32_t mask, double *const *out) {
  if (!h || !out) return ORC_EINVAL;
  if (h->pr.q_kind == 1) strain_pass(h, false);  // R24 limiter inputs at (x, u)
  for (size_t di = 0; di < h->dom.size(); ++di) {
    const Domain &D = h->dom[di];
    for (int64_t k = 0; k <= D.n[2]; ++k)
      for (int64_t j = 0; j <= D.n[1]; ++j)
        for (int64_t i = 0; i <= D.n[0]; ++i) {
          const int64_t g[3] = {D.lo[0] + i, D.lo[1] + j, D.lo[2] + k};
          if (h->dom_index(h->nown[0][g[0]], h->nown[1][g[1]], h->nown[2][g[2]]) != (int)di)
            continue;
          const int64_t gi = gnode(h, g), id = D.nid(i, j, k);
          for (int d = 0; d < 3; ++d) {
            if (mask & (1u << d)) out[d][gi] = D.x[d][id];
            if (mask & (1u << (3 + d))) out[3 + d][gi] = D.u[d][id];
          }
        }
    for (int64_t k = 0; k < D.n[2]; ++k)
      for (int64_t j = 0; j < D.n[1]; ++j)
        for (int64_t i = 0; i < D.n[0]; ++i) {
          const int64_t g[3] = {D.lo[0] + i, D.lo[1] + j, D.lo[2] + k};
          const int64_t gi = gzone(h, g), id = D.zid(i, j, k);
          double X[8][3], U[8][3], B[8][3], phi[3];
          ZoneOut o;
          gather_corners(D, D.x, D.u, i, j, k, X, U);
          if (h->pr.q_kind == 1) mono_phi(h, g, phi);
          zone_state(X, U, D.m[id], D.e[id], 0.0, h->pr, B, &o,
                     h->pr.q_kind == 1 ? phi : nullptr);
          if (mask & ORC_F_RHO) out[6][gi] = o.rho;
          if (mask & ORC_F_E) out[7][gi] = D.e[id];
          if (mask & ORC_F_P) out[8][gi] = o.p;
          if (mask & ORC_F_Q) out[9][gi] = o.q;
          if (mask & ORC_F_C) out[10][gi] = o.c;
          if (mask & ORC_F_VOL) out[11][gi] = o.V;
          if (mask & ORC_F_MASS) out[12][gi] = D.m[id];
        }
  }
  return ORC_OK;
}

void orc_destroy(orc_ctx *h) { delete h; }

}  // extern "C"
