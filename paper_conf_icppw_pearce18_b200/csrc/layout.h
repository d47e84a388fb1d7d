// layout.h -- host-side integer layout: domain boxes, domain->rank assignment and halo maps.
//
// PAPER.md L525-557 (§6.1): spatial decomposition into domains, each owned by one rank, with a
// halo exchange between neighbouring domains.  L559-572: hierarchical decomposition (per GPU,
// then a single-dimension split).  L589-603 (§6.2): weighted decomposition, initial guess from
// FLOPS, then measured and adjusted.  DESIGN.md §5 gives the exact rules (readings R14, R19).
#pragma once
#include <cstdint>
#include <string>
#include <vector>

#include "../../include/hydro.h"

namespace hydro {

struct DomainBox {
  int64_t lo[3];  // first owned zone (global)
  int64_t n[3];   // owned zones per axis
  int32_t idx[3]; // position in the domain grid
  int32_t rank;   // owning rank
};

// One ghost slab of domain `dst` filled from domain `src` (its neighbour in direction `dir`,
// encoded (dx+1) + 3(dy+1) + 9(dz+1)).  Boxes are half-open, in global node / zone indices.
struct HaloPair {
  int32_t dst, src, dir;
  int64_t nlo[3], nhi[3];
  int64_t zlo[3], zhi[3];
};

struct Layout {
  int64_t N[3];
  int32_t nd[3];
  std::vector<int64_t> cuts[3];
  std::vector<DomainBox> dom;
  std::vector<HaloPair> pairs;
  int32_t nranks;

  int dom_index(int a, int b, int c) const { return (c * nd[1] + b) * nd[0] + a; }
};

// Returns HYDRO_OK or HYDRO_EINVAL with a message in *err.
int layout_build(const hydro_config *cfg, Layout *out, std::string *err);

// LPT (longest processing time first) weighted assignment, reading R19 / SURVEY §8c.6.
std::vector<int32_t> lpt_assign(const std::vector<int64_t> &cost, int32_t nranks,
                                const double *weight);

// Serialisation used by hydro_layout_export.
std::vector<int64_t> layout_serialise(const Layout &L);

// Inter-rank halo plan of one rank: the slabs it sends (it owns the source domain) and receives
// (it owns the destination domain), in global pair order so that both ends of every rank pair
// enumerate their messages identically (NCCL send/recv match in issue order).
struct PlanEntry {
  int32_t pair;   // index into Layout::pairs
  int32_t peer;   // remote rank
  int64_t count;  // doubles: 6 node fields over the node slab + e over the zone slab
};
// self_all: also plan the pairs whose two domains are on this rank (as messages to itself;
// the one-rank NCCL test world, HYDRO_FLAG_COMM_SELF)
void comm_plan(const Layout &L, int32_t rank, std::vector<PlanEntry> *sends,
               std::vector<PlanEntry> *recvs, bool self_all = false);

}  // namespace hydro
