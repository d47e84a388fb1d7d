// layout.cpp -- see layout.h.  Host C++ only (no CUDA), so the layout can be built and tested on
// a machine without a GPU.
#include "layout.h"

#include <algorithm>
#include <cmath>
#include <limits>
#include <numeric>

namespace hydro {

std::vector<int32_t> lpt_assign(const std::vector<int64_t> &cost, int32_t nranks,
                                const double *weight) {
  // Domains in order (-cost, id); each goes to argmin_g (load_g + c)/w_g, ties -> lowest g.
  std::vector<int32_t> order(cost.size());
  std::iota(order.begin(), order.end(), 0);
  std::stable_sort(order.begin(), order.end(),
                   [&](int32_t a, int32_t b) { return cost[a] > cost[b]; });
  std::vector<double> load(nranks, 0.0);
  std::vector<int32_t> owner(cost.size(), 0);
  for (int32_t d : order) {
    int32_t best = 0;
    double bestv = std::numeric_limits<double>::infinity();
    for (int32_t g = 0; g < nranks; ++g) {
      const double w = weight ? weight[g] : 1.0;
      const double v = (load[g] + (double)cost[d]) / w;
      if (v < bestv) {
        bestv = v;
        best = g;
      }
    }
    owner[d] = best;
    load[best] += (double)cost[d];
  }
  return owner;
}

int layout_build(const hydro_config *cfg, Layout *L, std::string *err) {
  if (!cfg) {
    *err = "cfg is NULL";
    return HYDRO_EINVAL;
  }
  if (cfg->nranks < 1 || cfg->rank < 0 || cfg->rank >= cfg->nranks) {
    *err = "rank/nranks out of range";
    return HYDRO_EINVAL;
  }
  L->nranks = cfg->nranks;
  for (int a = 0; a < 3; ++a) {
    L->N[a] = cfg->n[a];
    L->nd[a] = cfg->ndom[a];
    if (cfg->n[a] < 1 || cfg->ndom[a] < 1) {
      *err = "mesh and domain counts must be >= 1";
      return HYDRO_EINVAL;
    }
    L->cuts[a].resize(cfg->ndom[a] + 1);
    for (int d = 0; d <= cfg->ndom[a]; ++d)
      L->cuts[a][d] = cfg->cuts[a] ? cfg->cuts[a][d] : (cfg->n[a] * d) / cfg->ndom[a];
    if (L->cuts[a][0] != 0 || L->cuts[a][cfg->ndom[a]] != cfg->n[a]) {
      *err = "cuts must start at 0 and end at n";
      return HYDRO_EINVAL;
    }
    for (int d = 0; d < cfg->ndom[a]; ++d)
      if (L->cuts[a][d + 1] <= L->cuts[a][d]) {
        *err = "cuts must be strictly increasing (every domain >= 1 zone)";
        return HYDRO_EINVAL;
      }
  }
  const int nd = L->nd[0] * L->nd[1] * L->nd[2];
  L->dom.assign(nd, DomainBox{});
  std::vector<int64_t> cost(nd);
  for (int c = 0; c < L->nd[2]; ++c)
    for (int b = 0; b < L->nd[1]; ++b)
      for (int a = 0; a < L->nd[0]; ++a) {
        DomainBox &D = L->dom[L->dom_index(a, b, c)];
        const int idx[3] = {a, b, c};
        for (int ax = 0; ax < 3; ++ax) {
          D.idx[ax] = idx[ax];
          D.lo[ax] = L->cuts[ax][idx[ax]];
          D.n[ax] = L->cuts[ax][idx[ax] + 1] - D.lo[ax];
        }
        cost[L->dom_index(a, b, c)] = D.n[0] * D.n[1] * D.n[2];
      }
  if (cfg->dom_to_rank) {
    for (int d = 0; d < nd; ++d) {
      if (cfg->dom_to_rank[d] < 0 || cfg->dom_to_rank[d] >= cfg->nranks) {
        *err = "dom_to_rank entry out of range";
        return HYDRO_EINVAL;
      }
      L->dom[d].rank = cfg->dom_to_rank[d];
    }
  } else {
    if (cfg->rank_weight)
      for (int g = 0; g < cfg->nranks; ++g)
        if (!(cfg->rank_weight[g] > 0.0)) {
          *err = "rank weights must be > 0";
          return HYDRO_EINVAL;
        }
    std::vector<int32_t> own = lpt_assign(cost, cfg->nranks, cfg->rank_weight);
    for (int d = 0; d < nd; ++d) L->dom[d].rank = own[d];
  }
  // Halo pairs: the ghost region of a domain (its zone box grown by one layer, its node box
  // [lo, lo+n] grown by one node, minus the owned part) splits into 26 slabs, one per direction;
  // slab `dir` lies entirely inside the owned part of the neighbour in that direction because
  // the cuts form a tensor-product grid.  Slabs across the physical boundary have no source.
  L->pairs.clear();
  for (int d = 0; d < nd; ++d) {
    const DomainBox &D = L->dom[d];
    for (int dz = -1; dz <= 1; ++dz)
      for (int dy = -1; dy <= 1; ++dy)
        for (int dx = -1; dx <= 1; ++dx) {
          if (!dx && !dy && !dz) continue;
          const int dd[3] = {dx, dy, dz};
          int s[3];
          bool ok = true;
          for (int ax = 0; ax < 3; ++ax) {
            s[ax] = D.idx[ax] + dd[ax];
            if (s[ax] < 0 || s[ax] >= L->nd[ax]) ok = false;
          }
          if (!ok) continue;
          HaloPair P;
          P.dst = d;
          P.src = L->dom_index(s[0], s[1], s[2]);
          P.dir = (dx + 1) + 3 * (dy + 1) + 9 * (dz + 1);
          for (int ax = 0; ax < 3; ++ax) {
            const int64_t lo = D.lo[ax], n = D.n[ax];
            if (dd[ax] < 0) {
              P.zlo[ax] = lo - 1; P.zhi[ax] = lo;
              P.nlo[ax] = lo - 1; P.nhi[ax] = lo;
            } else if (dd[ax] == 0) {
              P.zlo[ax] = lo; P.zhi[ax] = lo + n;
              P.nlo[ax] = lo; P.nhi[ax] = lo + n + 1;
            } else {
              P.zlo[ax] = lo + n; P.zhi[ax] = lo + n + 1;
              P.nlo[ax] = lo + n + 1; P.nhi[ax] = lo + n + 2;
            }
          }
          L->pairs.push_back(P);
        }
  }
  return HYDRO_OK;
}

std::vector<int64_t> layout_serialise(const Layout &L) {
  std::vector<int64_t> w;
  w.push_back(1);
  w.push_back((int64_t)L.dom.size());
  w.push_back(L.nranks);
  w.push_back((int64_t)L.pairs.size());
  for (int a = 0; a < 3; ++a) w.push_back(L.N[a]);
  for (const DomainBox &D : L.dom) {
    for (int a = 0; a < 3; ++a) w.push_back(D.lo[a]);
    for (int a = 0; a < 3; ++a) w.push_back(D.n[a]);
    w.push_back(D.rank);
  }
  for (const HaloPair &P : L.pairs) {
    w.push_back(P.dst);
    w.push_back(P.src);
    w.push_back(P.dir);
    for (int a = 0; a < 3; ++a) w.push_back(P.nlo[a]);
    for (int a = 0; a < 3; ++a) w.push_back(P.nhi[a]);
    for (int a = 0; a < 3; ++a) w.push_back(P.zlo[a]);
    for (int a = 0; a < 3; ++a) w.push_back(P.zhi[a]);
  }
  return w;
}

void comm_plan(const Layout &L, int32_t rank, std::vector<PlanEntry> *sends,
               std::vector<PlanEntry> *recvs, bool self_all) {
  sends->clear();
  recvs->clear();
  for (size_t i = 0; i < L.pairs.size(); ++i) {
    const HaloPair &P = L.pairs[i];
    const int32_t rd = L.dom[P.dst].rank, rs = L.dom[P.src].rank;
    if (rd == rs && !(self_all && rd == rank)) continue;  // same rank: intra-GPU copy kernel
    int64_t nn = 1, nz = 1;
    for (int a = 0; a < 3; ++a) {
      nn *= P.nhi[a] - P.nlo[a];
      nz *= P.zhi[a] - P.zlo[a];
    }
    if (rs == rank) sends->push_back(PlanEntry{(int32_t)i, rd, 6 * nn + nz});
    if (rd == rank) recvs->push_back(PlanEntry{(int32_t)i, rs, 6 * nn + nz});
  }
}

}  // namespace hydro

using namespace hydro;

extern "C" {

int hydro_layout_export(const hydro_config *cfg, int64_t *buf, size_t *len) {
  if (!len) return HYDRO_EINVAL;
  Layout L;
  std::string err;
  const int rc = layout_build(cfg, &L, &err);
  if (rc != HYDRO_OK) return rc;
  std::vector<int64_t> w = layout_serialise(L);
  const size_t cap = *len;
  *len = w.size();
  if (buf && cap >= w.size()) std::copy(w.begin(), w.end(), buf);
  return (buf && cap < w.size()) ? HYDRO_EINVAL : HYDRO_OK;
}

int hydro_comm_plan_export(const hydro_config *cfg, int64_t *buf, size_t *len) {
  if (!len) return HYDRO_EINVAL;
  Layout L;
  std::string err;
  const int rc = layout_build(cfg, &L, &err);
  if (rc != HYDRO_OK) return rc;
  std::vector<PlanEntry> snd, rcv;
  comm_plan(L, cfg->rank, &snd, &rcv);
  std::vector<int64_t> w{(int64_t)snd.size(), (int64_t)rcv.size()};
  for (const auto *v : {&snd, &rcv})
    for (const PlanEntry &e : *v) {
      const HaloPair &P = L.pairs[e.pair];
      w.insert(w.end(), {e.pair, e.peer, e.count, P.dst, P.src, P.dir});
    }
  const size_t cap = *len;
  *len = w.size();
  if (buf && cap >= w.size()) std::copy(w.begin(), w.end(), buf);
  return (buf && cap < w.size()) ? HYDRO_EINVAL : HYDRO_OK;
}

int hydro_rebalance_plan(const hydro_config *cfg, const double *busy, double beta,
                         double min_gain, int32_t *new_map, double *weights, double *predicted) {
  if (!cfg || !busy || !new_map || !(beta >= 0.0) || !(min_gain >= 0.0)) return HYDRO_EINVAL;
  Layout L;
  std::string err;
  const int rc = layout_build(cfg, &L, &err);
  if (rc != HYDRO_OK) return rc;
  const int nd = (int)L.dom.size(), G = cfg->nranks;
  for (int g = 0; g < G; ++g)
    if (!(busy[g] > 0.0) || !std::isfinite(busy[g])) return HYDRO_EINVAL;
  // domain cost: owned zones + beta * ghost elements (the surface term)
  std::vector<double> ghost(nd, 0.0);
  for (const HaloPair &P : L.pairs) {
    int64_t nn = 1, nz = 1;
    for (int a = 0; a < 3; ++a) {
      nn *= P.nhi[a] - P.nlo[a];
      nz *= P.zhi[a] - P.zlo[a];
    }
    ghost[P.dst] += (double)(nn + nz);
  }
  std::vector<int64_t> cost(nd);
  for (int d = 0; d < nd; ++d) {
    const double c = (double)(L.dom[d].n[0] * L.dom[d].n[1] * L.dom[d].n[2]) + beta * ghost[d];
    cost[d] = (int64_t)std::llround(c);
  }
  // measured speeds ("We measured the respective contributions ... and
  // adjusted the split"): w_g = load_g / busy_g under the current map; a rank with no domain
  // keeps the mean speed of the others
  std::vector<double> load(G, 0.0), w(G, 0.0);
  for (int d = 0; d < nd; ++d) load[L.dom[d].rank] += (double)cost[d];
  double wsum = 0.0;
  int nw = 0;
  for (int g = 0; g < G; ++g)
    if (load[g] > 0.0) {
      w[g] = load[g] / busy[g];
      wsum += w[g];
      ++nw;
    }
  if (nw == 0) return HYDRO_EINVAL;
  for (int g = 0; g < G; ++g)
    if (!(load[g] > 0.0)) w[g] = wsum / nw;
  double mean = 0.0;
  for (int g = 0; g < G; ++g) mean += w[g];
  mean /= G;
  for (int g = 0; g < G; ++g) w[g] /= mean;
  std::vector<int32_t> own = lpt_assign(cost, G, w.data());
  // predicted makespans in the speed model (before = the measured map, after = LPT)
  std::vector<double> l0(G, 0.0), l1(G, 0.0);
  for (int d = 0; d < nd; ++d) {
    l0[L.dom[d].rank] += (double)cost[d];
    l1[own[d]] += (double)cost[d];
  }
  double before = 0.0, after = 0.0;
  for (int g = 0; g < G; ++g) {
    before = std::max(before, l0[g] / w[g]);
    after = std::max(after, l1[g] / w[g]);
  }
  const bool move = after < before * (1.0 - min_gain);  // migration only for a real gain
  for (int d = 0; d < nd; ++d) new_map[d] = move ? own[d] : L.dom[d].rank;
  if (weights)
    for (int g = 0; g < G; ++g) weights[g] = w[g];
  if (predicted) {
    predicted[0] = before;
    predicted[1] = move ? after : before;
  }
  return HYDRO_OK;
}

int hydro_weighted_slabs(int64_t nplanes, int32_t nparts, const double *w, int64_t *out) {
  if (nparts < 1 || nplanes < nparts || !out) return HYDRO_EINVAL;
  double W = 0.0;
  for (int g = 0; g < nparts; ++g) {
    const double wg = w ? w[g] : 1.0;
    if (!(wg > 0.0)) return HYDRO_EINVAL;
    W += wg;
  }
  std::vector<double> rem(nparts);
  int64_t used = 0;
  for (int g = 0; g < nparts; ++g) {
    const double exact = (double)nplanes * (w ? w[g] : 1.0) / W;
    out[g] = (int64_t)std::floor(exact);
    rem[g] = exact - (double)out[g];
    used += out[g];
  }
  // remaining planes to the largest fractional remainders, ties -> lowest g
  std::vector<int32_t> order(nparts);
  std::iota(order.begin(), order.end(), 0);
  std::stable_sort(order.begin(), order.end(), [&](int a, int b) { return rem[a] > rem[b]; });
  for (int64_t k = 0; used < nplanes; ++k, ++used) out[order[k % nparts]] += 1;
  // whole-plane granularity: every part gets at least one plane, taken from the largest parts
  for (int g = 0; g < nparts; ++g) {
    while (out[g] < 1) {
      int big = 0;
      for (int h = 1; h < nparts; ++h)
        if (out[h] > out[big]) big = h;
      out[big] -= 1;
      out[g] += 1;
    }
  }
  return HYDRO_OK;
}

int hydro_decompose_hierarchical(const int64_t n[3], int32_t ngpu, int32_t dpg, int32_t ndom[3],
                                 int64_t *const cuts[3], int32_t *dom_to_rank) {
  if (!n || ngpu < 1 || dpg < 1 || !ndom || !cuts || !dom_to_rank) return HYDRO_EINVAL;
  // Step 1 (Fig. 10a): ngpu = gx*gy*gz blocks minimising the interface area; ties prefer fewer
  // cuts in x (x is kept whole where possible, L587), then fewer in y.
  int best[3] = {0, 0, 0};
  double best_area = std::numeric_limits<double>::infinity();
  for (int gx = 1; gx <= ngpu; ++gx) {
    if (ngpu % gx) continue;
    for (int gy = 1; gy <= ngpu / gx; ++gy) {
      if ((ngpu / gx) % gy) continue;
      const int gz = ngpu / gx / gy;
      if (gx > n[0] || gy * dpg > n[1] || gz > n[2]) continue;
      const double area = (double)(gx - 1) * n[1] * n[2] + (double)(gy - 1) * n[0] * n[2] +
                          (double)(gz - 1) * n[0] * n[1];
      if (area < best_area) {  // strict: first found (smallest gx, then gy) wins ties
        best_area = area;
        best[0] = gx; best[1] = gy; best[2] = gz;
      }
    }
  }
  if (!best[0]) return HYDRO_EINVAL;
  // Step 2 (Fig. 10b): each GPU block split into dpg slabs along y.
  ndom[0] = best[0];
  ndom[1] = best[1] * dpg;
  ndom[2] = best[2];
  for (int a = 0; a < 3; a += 2)
    for (int d = 0; d <= best[a]; ++d) cuts[a][d] = (n[a] * d) / best[a];
  for (int by = 0; by < best[1]; ++by) {
    const int64_t y0 = (n[1] * by) / best[1], y1 = (n[1] * (by + 1)) / best[1];
    for (int s = 0; s < dpg; ++s) cuts[1][by * dpg + s] = y0 + ((y1 - y0) * s) / dpg;
  }
  cuts[1][best[1] * dpg] = n[1];
  for (int c = 0; c < ndom[2]; ++c)
    for (int b = 0; b < ndom[1]; ++b)
      for (int a = 0; a < ndom[0]; ++a)
        dom_to_rank[(c * ndom[1] + b) * ndom[0] + a] = (c * best[1] + b / dpg) * best[0] + a;
  return HYDRO_OK;
}

}  // extern "C"
