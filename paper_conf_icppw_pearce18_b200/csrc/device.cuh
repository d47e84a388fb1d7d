// device.cuh -- device-side data layout and per-zone physics shared by the CUDA kernels.
//
// Layout in HBM.  Every domain owns one allocation holding SoA fp64 arrays,
// x fastest, with one ghost layer:
//   nodes  local index i in [-1, n+1] per axis -> (k+1)*nsxy + (j+1)*nsx + (i+1)
//   zones  local index i in [-1, n]   per axis -> (k+1)*zsxy + (j+1)*zsx + (i+1)
// Node state x,y,z,u,v,w and zone energy e are double-buffered (parity 0/1: a cycle reads one
// and writes the other, so no tile ever reads a value another tile already advanced); zone
// mass m is constant.  Ghost entries beyond the physical boundary are never advanced: their
// nodes keep the extrapolated lattice position and u = 0, their zones m = e = 0, so any stencil
// that touches them reads finite numbers and masks them out.
#pragma once
#include <cstdint>

namespace hydro {

struct DomView {
  int64_t lo[3];   // first owned zone, global
  int32_t n[3];    // owned zones per axis
  int32_t N[3];    // global zones per axis
  int64_t nsx, nsxy, zsx, zsxy;
  int64_t nnode, nzone;  // storage sizes
  const double *x, *y, *z, *u, *v, *w;  // node state at t^n (parity p)
  double *xn, *yn, *zn, *un, *vn, *wn;  // node state at t^{n+1} (parity 1-p)
  const double *e;                      // zone energy at t^n
  double *en;                           // zone energy at t^{n+1}
  const double *m;                      // zone mass (constant)
  double *P;                            // split pipeline: zone P scratch
  double *B;                            // split pipeline: 24 corner-vector components per zone
  double *aux;                          // 5 zone arrays: rho, p, q, c, vol (get_fields)
  int32_t dom;                          // global domain index
  int32_t pad_;

  __host__ __device__ int64_t nid(int i, int j, int k) const {
    return (int64_t)(k + 1) * nsxy + (int64_t)(j + 1) * nsx + (i + 1);
  }
  __host__ __device__ int64_t zid(int i, int j, int k) const {
    return (int64_t)(k + 1) * zsxy + (int64_t)(j + 1) * zsx + (i + 1);
  }
};

struct Phys {
  double gamma, gm1, ggm1, q_lin, q_quad, cfl, c_vol;
  double dt_growth, dt_max, t_stop;
  uint32_t reflect_mask;
  uint32_t pad_;
};

// Device-resident scalar state of a run (one per rank).  Kernels read t, dt from here so a
// captured CUDA graph replays every cycle without host involvement.
struct DevState {
  double t, dt;
  double dtz_last;              // global min_z dt_z of the last cycle
  unsigned long long dtz_acc;   // running min of dt_z (bits of a non-negative double)
  unsigned long long cycle;
  unsigned long long bad_zone;  // lowest failing global zone index (~0 = none)
  unsigned int err;             // error bits raised during the current cycle
  unsigned int halted;          // != 0: run stopped with these error bits
  unsigned int done;            // t >= t_stop
  unsigned int pad_;
};

enum : unsigned int { ERR_TANGLED = 1u, ERR_NONFINITE = 2u };

}  // namespace hydro
