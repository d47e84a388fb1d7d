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
  double *mn8;                          // node: 8 / (sum of the <= 8 zone masses around it),
                                        // constant (Lagrangian masses, S7); see k_nodal_mass
  double *mi;                           // zone: 1 / m (0 outside the mesh), constant
  double *eps;                          // monotone q (R24): 3 zone planes of strain rates of
                                        // the owned zones (scratch; nullptr unless q_kind 1)
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
  int32_t q_kind;  // 0 scalar q (reading R7), 1 monotone q (reading R24; split / STRICT paths)
  double hg;  // hourglass kappa (split path only; 0 = off)
};

// Reading R24 (monotone q): where the strain rate of any global zone lives.  Single rank: every
// domain is on this GPU.  Owner of global zone g = domain (zown0[g0], zown1[g1], zown2[g2]).
struct MonoMap {
  const int32_t *zown[3];  // per axis: domain coordinate of each global zone index
  const int32_t *slot;     // global domain -> local slot
  const DomView *views;    // local views (current parity; eps is parity-free)
  int32_t ndx, ndy;
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
  unsigned int blocks_done;     // CTAs of the last cycle kernel that finished (folded finalize)
  unsigned long long xchg;      // peer-transport exchange epoch (peer.cu)
  double dt_floor;              // reading R23: min_z dt_z below this halts the run (0 = none)
};

enum : unsigned int { ERR_TANGLED = 1u, ERR_NONFINITE = 2u, ERR_DTMIN = 4u };

// S9: t' = t + dt, dt' = min(min(growth*dt, dt_max), min_z dt_z), t_stop clamp;
// dt-collapse check (reading R23); latch the cycle's error bits so later cycles become no-ops (the state stays the one after the
// failing cycle, as in the oracle).  Run by one thread after every kernel of the cycle.
// PDL (kernels.h launch_pdl): wait for the preceding kernel's completion and memory flush, then
// let the next kernel launch.  No-ops when the kernel was launched without the attribute.
__device__ __forceinline__ void pdl_wait_and_trigger() {
  asm volatile("griddepcontrol.wait;" ::: "memory");
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}

__device__ __forceinline__ void finalize_cycle(DevState *st, const Phys &ph) {
  if (st->halted | st->done) return;
  const double dtmin = __longlong_as_double((long long)st->dtz_acc);
  const double dt = st->dt;
  const double tn = st->t + dt;
  double dtn = fmin(fmin(ph.dt_growth * dt, ph.dt_max), dtmin);
  const bool stop = ph.t_stop > 0.0 && tn >= ph.t_stop;
  if (ph.t_stop > 0.0) dtn = fmin(dtn, ph.t_stop - tn);
  st->t = tn;
  st->dt = dtn;
  st->dtz_last = dtmin;
  st->cycle += 1;
  st->dtz_acc = (unsigned long long)__double_as_longlong(INFINITY);
  unsigned err = st->err;
  if (!(isfinite(dtn) && dtn > 0.0) && !stop) err |= ERR_NONFINITE;
  // reading R23: dt collapse (the zone dt minimum of this cycle fell below the floor)
  if (!stop && dtmin < st->dt_floor) err |= ERR_DTMIN;
  st->halted = err;
  st->done = stop ? 1u : 0u;
}

// Folded finalize: the last CTA of a kernel to finish runs finalize_cycle (every other CTA has
// read st->dt before finishing).  Call from all threads at the very end of the kernel; ticket is
// one word of shared scratch.
__device__ __forceinline__ void finalize_if_last_block(DevState *st, const Phys &ph,
                                                       unsigned int *ticket) {
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    *ticket = atomicAdd(&st->blocks_done, 1u);
  }
  __syncthreads();
  const unsigned total = gridDim.x * gridDim.y * gridDim.z;
  if (threadIdx.x == 0 && *ticket == total - 1) {
    __threadfence();
    finalize_cycle(st, ph);
    st->blocks_done = 0;
  }
}

}  // namespace hydro
