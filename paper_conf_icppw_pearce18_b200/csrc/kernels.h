// kernels.h -- host-side launchers for the CUDA kernels (all enqueue on `s`, never synchronise).
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>

#include "device.cuh"

#define FUSED_BOX_X 36  // TMA node box width (TX + 3 = 35 rounded up to a 16-byte row)
#define ZONE_BOX_X 36   // zone-stage node box width (33 + 1 alignment shift, 16-byte rows)

namespace hydro {

// Programmatic dependent launch (PDL): the per-cycle kernels are launched with
// cudaLaunchAttributeProgrammaticStreamSerialization, start `griddepcontrol.wait` (pdl_wait in
// device.cuh) before touching global memory, and trigger their dependents right after, so the
// next kernel's CTAs are launched and set up while this one drains (CUDA graphs keep the
// programmatic edges).  HYDRO_NO_PDL=1 launches them plainly (A/B measurement).
bool pdl_enabled();
template <typename... KArgs, typename... Args>
cudaError_t launch_pdl(void (*k)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s,
                       Args... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = pdl_enabled() ? 1 : 0;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, k, static_cast<KArgs>(args)...);
}

struct HaloCopy {  // one chunk of an intra-GPU ghost slab copy (global boxes, half-open)
  int32_t dst, src;  // local domain slots
  int64_t nlo[3], nhi[3], zlo[3], zhi[3];
  int32_t kind;         // 0: the node slab (x,y,z,u,v,w), 1: the zone slab (e), 2: the zone
                        // slab of the current cycle's P (ring zones the zone stage skips)
  int32_t start, count; // elements [start, start+count) of that slab, x fastest
};
constexpr int HALO_CHUNK = 2048;  // elements per chunk (one CTA of 256 threads)

// One ghost slab a domain stores into a neighbour from the node/energy-stage epilogue (fused
// halo): the neighbour's ghost nodes / zones that this (source) domain owns, as
// boxes in SOURCE-local indices, and where they go.  Destination index of the source-local node
// (i, j, k) = nbase + k nsxy + j nsx + i (zones: zbase, zsxy, zsx); dst = the destination's
// next-parity x,y,z,u,v,w,e arrays (device pointers on this GPU, or CUDA-IPC mapped peer memory).
struct PushSlab {
  int32_t nlo[3], nhi[3];  // node box, half-open
  int32_t zlo[3], zhi[3];  // zone box, half-open
  int64_t nbase, zbase;
  int32_t nsx, nsxy, zsx, zsxy;
  double *dst[7];
  int32_t remote;          // destination in another process (system-scope fence after the stores)
  int32_t pad_;
};

// Zone-stage work of one domain (kernel_zone.cu): zone box [zlo, zhi) in local indices (the ghost
// ring where a neighbour exists), tcols x-tiles, `units` = columns x planes, u0 = first unit in
// the concatenation over the GPU's domains (grouped launch).
struct ZoneTask {
  int32_t slot, tcols;
  int32_t zlo[3], zhi[3];
  int64_t u0, units;
  int32_t zblk;  // planes per z-block of the unit order (kernel_zone.cu; = planes: column-major)
  int32_t pad_;
};

// Initialisation.
void launch_init_nodes(const DomView &d, const double origin[3], const double extent[3],
                       cudaStream_t s);
// kind: 0 Sedov (rho0, e0, E), 1 USER (rho in d.P scratch, e already in place),
// 2 USER_MASS (m already in place, e already in place).
void launch_init_zones(const DomView &d, int kind, double rho0, double e0, double E,
                       cudaStream_t s);
// d.mi = 1/m of every zone in storage (0 where m = 0) and
// d.mn8 = 8 / sum of the zone masses around each node (nodes 0..n per axis; masses are fixed
// after init, so once per run).
void launch_nodal_mass(const DomView &d, cudaStream_t s);
// dt^0 (S2-S6 at x^0 with no predictor) over owned zones -> st->dtz_acc, error flags.
// M: monotone-q lookup (reading R24; only read when ph.q_kind == 1).
void launch_dt0(const DomView &d, const Phys &ph, DevState *st, const MonoMap &M,
                cudaStream_t s);
// Reading R24: d.eps <- strain rates of the owned zones at x + dt/2 u (at_x: at x).
void launch_strain(const DomView &d, const DevState *st, int at_x, cudaStream_t s);
void launch_finalize_init(DevState *st, double dt_first, double dt_init, double dt_max,
                          double t_stop, double t0, double dt_floor, cudaStream_t s);

// Split 3-kernel pipeline (naive, obviously-correct path; HYDRO_FLAG_SPLIT).
void launch_zone_split(const DomView &d, const Phys &ph, DevState *st, const MonoMap &M,
                       cudaStream_t s);
void launch_node_split(const DomView &d, const Phys &ph, DevState *st, cudaStream_t s);
void launch_energy_split(const DomView &d, const Phys &ph, DevState *st, cudaStream_t s);

// STRICT path (HYDRO_FLAG_STRICT; strict/kernel_strict.cu, compiled with -fmad=false): the
// split pipeline in the canonical operation order of SURVEY §8c, bitwise equal to the oracle.
void launch_strict_init_zones(const DomView &d, int kind, double rho0, double e0, double E,
                              cudaStream_t s);
void launch_strict_dt0(const DomView &d, const Phys &ph, DevState *st, const MonoMap &M,
                       cudaStream_t s);
void launch_strict_strain(const DomView &d, const DevState *st, int at_x, cudaStream_t s);
void launch_strict_zone(const DomView &d, const Phys &ph, DevState *st, const MonoMap &M,
                        cudaStream_t s);
void launch_strict_node(const DomView &d, const Phys &ph, DevState *st, cudaStream_t s);
void launch_strict_energy(const DomView &d, const Phys &ph, DevState *st, cudaStream_t s);
void launch_strict_derive(const DomView &d, const Phys &ph, const MonoMap &M, cudaStream_t s);

// TMA descriptors of one domain and parity: the six node-state arrays (x,y,z,u,v,w), the
// constant nodal 8/mass array and the
// zone arrays m, e, P (box = the kernel's zone tile).
struct alignas(64) NodeMaps {
  CUtensorMap m[7];  // x, y, z, u, v, w, 8/nodal mass
  CUtensorMap z[4];  // m, e, P, 1/m
};

// Fused single-kernel cycle (default path).
// fold_finalize != 0: the kernel's last CTA also performs S9 (k_finalize is then not launched;
// only valid when this is the cycle's last kernel: one domain, one rank).
void launch_cycle_fused(const DomView &d, const NodeMaps &maps, const Phys &ph, DevState *st,
                        int fold_finalize, cudaStream_t s);
size_t fused_smem_bytes();
int fused_box_y();
int fused_tile_ty();  // tile height of the one-kernel variant

// Two-kernel cycle (default path): zone stage (P, dt) then node/energy stage.
// Node/energy-stage work of one domain in a grouped launch (kernel_cycle.cu): x-tiles, columns,
// z-chunk length and the first CTA of the domain in the concatenated grid.
struct NodeTask {
  int32_t slot, tcols, ncols, kz, cta0;
  int32_t push0, npush;  // this domain's PushSlab range (fused halo; npush 0 = none)
};
// Fills out[n] (chunk length shared by all domains); returns the total CTA count.
int node_group_tasks(const DomView *views_host, int n, NodeTask *out);
void launch_node_energy_group(const NodeTask *tasks_dev, int ntasks, int nctas,
                              const DomView *views_dev, const NodeMaps *maps_dev, const Phys &ph,
                              DevState *st, const PushSlab *push, cudaStream_t s);

// Grouped zone stage over all local domains (one persistent launch): tasks from
// zone_group_tasks (host), copied to the device by the caller; views_dev / maps_dev indexed by
// ZoneTask::slot.
// rings[i]: bit 2a+h = compute the ghost-zone ring of domain i on side h (0 low, 1 high) of
// axis a (where a neighbour exists); clear = its P comes from the owning local domain by a
// kind-2 halo copy after the zone stage (runtime.cu)
void zone_group_tasks(const DomView *views_host, const uint8_t *rings, int n, ZoneTask *out,
                      int64_t *Wtot);
void launch_zone_stage_group(const DomView *views_dev, const NodeMaps *maps_dev,
                             const ZoneTask *tasks_dev, int64_t Wtot, const Phys &ph,
                             DevState *st, cudaStream_t s);
void launch_zone_stage(const DomView &d, const NodeMaps &maps, uint8_t ring, const Phys &ph,
                       DevState *st, cudaStream_t s);
// push/npush: this domain's fused-halo slabs (nullptr/0: none; the caller then exchanges the
// ghost layer with launch_halo_copy / the transports).
// ty: node-stage tile height (node_tile_ty; the TMA maps must be built with its boxes).
void launch_node_energy(const DomView &d, const NodeMaps &maps, const Phys &ph, DevState *st,
                        int fold_finalize, const PushSlab *push, int npush, int ty,
                        cudaStream_t s);
// Node-stage tile height for a domain of n0 x n1 x n2 zones (11 or 12; HYDRO_NODE_TY forces).
int node_tile_ty(int n0, int n1, int n2);
int zone_box_y();
int node_box_y(int ty);  // node-field TMA box height of the node stage with tile height ty
int cycle_zone_box_x();  // zone-field TMA box of the cycle kernels
int cycle_zone_box_y(int ty);

// End of cycle: S9 dt / time update and error latch.
void launch_finalize(DevState *st, const Phys &ph, cudaStream_t s);

// Intra-GPU ghost exchange of the next-parity state over a table of slab copies.
void launch_halo_copy(const DomView *views_dev, const HaloCopy *chunks_dev, int nchunks,
                      cudaStream_t s);

// hydro_run_batch: t, dt, cycle 0, errors cleared (one thread).
void launch_reset_clock(DevState *st, double t, double dt, unsigned done, cudaStream_t s);

// Strided 3-D box copy (src/dst pre-offset to the box origin; pitches in elements).
void launch_copy3d(const double *src, int64_t ssx, int64_t ssxy, double *dst, int64_t dsx,
                   int64_t dsxy, int ex, int ey, int ez, cudaStream_t s);

// get_fields: derived zone fields (rho, p, q, c, vol) at (x, u) with no predictor into d.aux.
void launch_derive(const DomView &d, const Phys &ph, const MonoMap &M, cudaStream_t s);

}  // namespace hydro
