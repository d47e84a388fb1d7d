// runtime.cu -- the C ABI of include/hydro.h: context, per-domain device allocation, CUDA-graph
// capture of a cycle, host<->device field transfer.  One process drives one GPU; all domains
// assigned to this rank live in its HBM (each rank owns its domains).
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <nvtx3/nvToolsExt.h>  // header-only; ranges show up in nsys / ncu --nvtx

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <limits>
#include <string>
#include <vector>

#include "../../include/hydro.h"
#include "comm.h"
#include "kernels.h"
#include "layout.h"
#include "peer.h"

using namespace hydro;

namespace {

thread_local std::string g_err;

struct LocalDom {
  int32_t dom;  // global domain index
  DomainBox box;
  void *mem = nullptr;
  size_t bytes = 0;
  DomView view[2];  // parity p reads view[p].x and writes view[p].xn
  NodeMaps maps[2];  // TMA descriptors of view[p]'s current node arrays, fused/node box
  NodeMaps zmaps[2]; // same arrays, zone-stage box
  int node_ty = 12;  // node-stage tile height (kernel_cycle.cu node_tile_ty), sets maps' boxes
};

}  // namespace

struct hydro_ctx {
  hydro_config cfg;
  Layout L;
  Phys ph;
  int device = 0;
  cudaStream_t stream = nullptr;
  std::vector<LocalDom> doms;
  std::vector<int32_t> slot_of_dom;  // global domain -> local slot or -1
  DevState *st = nullptr;
  DomView *views_dev[2] = {nullptr, nullptr};
  HaloCopy *local_pairs_dev = nullptr;
  // grouped zone stage over all local domains (kernel_zone.cu launch_zone_stage_group)
  NodeMaps *zmaps_dev[2] = {nullptr, nullptr};
  ZoneTask *ztasks_dev = nullptr;
  int64_t zunits = 0;
  bool group = false;
  NodeMaps *nmaps_dev[2] = {nullptr, nullptr};  // grouped node/energy stage
  NodeTask *ntasks_dev = nullptr;
  std::vector<NodeTask> ntasks_host;
  int nctas = 0;
  int n_local_pairs = 0;
  // zone-stage ghost rings: ring[slot] bit 2a+h = compute the ring on that side;
  // ring zones owned by another domain of this rank get their P by a copy after the zone stage
  std::vector<uint8_t> ring;
  HaloCopy *pcopy_dev = nullptr;
  int n_pcopy = 0;
  // halo copy overlapped with the other domains' node stages: chunks sorted by source slot, each
  // domain's outgoing slabs copied on its own stream right after its node/energy stage
  // (HYDRO_HALO_OVERLAP=0 for the single copy after the join, A/B)
  // 1: per domain on its node-stage stream; 2: per domain on a dedicated halo stream; 3: per
  // node-stage stream after its last domain (the default with <= 2 domains per stream)
  int halo_overlap = 0;
  cudaStream_t halo_stream = nullptr;
  std::vector<cudaEvent_t> node_done;  // per local slot (mode 2)
  cudaEvent_t halo_join = nullptr;
  std::vector<int32_t> halo_first, halo_count;  // per local slot, into local_pairs_dev
  // fused halo (default two-kernel path): the node/energy stage stores the ghost slabs itself
  bool fused_halo = false;
  std::vector<PushTarget> push_targets;     // local and (after peer import) remote slabs
  PushSlab *push_dev[2] = {nullptr, nullptr};
  std::vector<int32_t> push_first, push_count;  // per local slot
  // several domains on this GPU: node/energy stages spread over nstreams streams (fork/join by
  // events, parallel branches in the captured graph), HYDRO_NODE_STREAMS
  int nstreams = 1;
  // launch order of the local domains' node stages and the stream of each (HYDRO_NODE_LPT=1,
  // default: largest first, each onto the least-loaded stream; 0: index order, round-robin)
  std::vector<int32_t> node_order, node_stream;
  std::vector<size_t> stream_last;  // position in node_order of each stream's last domain
  cudaStream_t side[4] = {nullptr, nullptr, nullptr, nullptr};
  cudaEvent_t fork_ev = nullptr, join_ev[4] = {nullptr, nullptr, nullptr, nullptr};
  cudaGraphExec_t graph[2] = {nullptr, nullptr};
  // graph_k cycles in one graph (per starting parity): the programmatic edges then also link one
  // cycle's finalize to the next cycle's zone stage (no graph-launch boundary between them)
  cudaGraphExec_t graphk[2] = {nullptr, nullptr};
  int graph_k = 1;
  int parity = 0;
  bool split = false;
  bool strict = false;  // HYDRO_FLAG_STRICT: the split pipeline in the oracle's operation order
  // monotone q (reading R24): strain-rate planes per domain and the owner lookup tables
  MonoMap mono = {};
  std::vector<void *> mono_mem;
  bool one_kernel = false;
  bool use_graph = true;
  int failed = 0;
  Comm *comm = nullptr;
  Peer *peer = nullptr;      // HYDRO_FLAG_PEER transport (nranks > 1)
  // hydro_run_batch: two device staging slots each for the dense global inputs and outputs
  // (x,y,z,u,v,w on nodes, e on zones), two copy streams and their slot events (lazy)
  double *bin[2] = {nullptr, nullptr}, *bout[2] = {nullptr, nullptr};
  cudaStream_t cp_in = nullptr, cp_out = nullptr;
  cudaEvent_t in_ready[2] = {}, in_free[2] = {}, out_ready[2] = {}, out_free[2] = {};
  DevState *bst = nullptr;  // per-batch final DevState
  int32_t bst_cap = 0;
  // hydro_step early stop (single rank): a ring of pinned mirrors of (halted, done)
  static constexpr int NFLAG = 8;
  unsigned int *flag_host = nullptr;
  cudaEvent_t flag_ev[NFLAG] = {};
  double *stage = nullptr;  // contiguous device staging for host transfers (lazy)
  size_t stage_cap = 0;
  std::string err;
};

namespace {

int set_err(hydro_ctx *h, int code, const std::string &msg) {
  g_err = msg;
  if (h) h->err = msg;
  return code;
}

#define CK(call)                                                                       \
  do {                                                                                 \
    cudaError_t e_ = (call);                                                           \
    if (e_ != cudaSuccess)                                                             \
      return set_err(h, HYDRO_ECUDA, std::string(#call ": ") + cudaGetErrorString(e_)); \
  } while (0)

size_t align_up(size_t v, size_t a) { return (v + a - 1) / a * a; }

// NVTX range for the duration of a C-ABI call (tracing)
struct NvtxRange {
  explicit NvtxRange(const char *name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
};

}  // namespace

namespace hydro {

// Storage of one domain inside its single allocation (also used to reconstruct the arrays of a
// remote domain from its IPC-mapped base: every rank computes the same offsets).
size_t domain_bytes(const DomainBox &b, bool split) {
  const int64_t nsx = (b.n[0] + 3 + 3) / 4 * 4, nnode = nsx * (b.n[1] + 3) * (b.n[2] + 3);
  const int64_t zsx = (b.n[0] + 2 + 3) / 4 * 4, nzone = zsx * (b.n[1] + 2) * (b.n[2] + 2);
  const size_t nb = align_up(nnode * sizeof(double), 256), zb = align_up(nzone * sizeof(double), 256);
  return 13 * nb + 10 * zb + (split ? 24 * zb : 0);  // 12 node arrays, mn8, e x2, m, mi, P, aux x5, [B x24]
}

void carve_views(void *base, const DomainBox &b, const int64_t N[3], int32_t dom, bool split,
                 DomView view[2]) {
  const int64_t n0 = b.n[0], n1 = b.n[1], n2 = b.n[2];
  // row pitches padded to 4 doubles (32 B): TMA needs 16-byte strides
  const int64_t nsx = (n0 + 3 + 3) / 4 * 4, nsxy = nsx * (n1 + 3), nnode = nsxy * (n2 + 3);
  const int64_t zsx = (n0 + 2 + 3) / 4 * 4, zsxy = zsx * (n1 + 2), nzone = zsxy * (n2 + 2);
  const size_t nb = align_up(nnode * sizeof(double), 256), zb = align_up(nzone * sizeof(double), 256);
  char *p = (char *)base;
  double *nodes[12];
  for (int a = 0; a < 12; ++a, p += nb) nodes[a] = (double *)p;
  double *mn8 = (double *)p; p += nb;
  double *e0 = (double *)p; p += zb;
  double *e1 = (double *)p; p += zb;
  double *m = (double *)p; p += zb;
  double *mi = (double *)p; p += zb;
  double *P = (double *)p; p += zb;
  double *aux = (double *)p; p += 5 * zb;
  double *B = split ? (double *)p : nullptr;
  for (int par = 0; par < 2; ++par) {
    DomView &v = view[par];
    std::memset(&v, 0, sizeof(v));
    for (int a = 0; a < 3; ++a) {
      v.lo[a] = b.lo[a];
      v.n[a] = (int32_t)b.n[a];
      v.N[a] = (int32_t)N[a];
    }
    v.nsx = nsx; v.nsxy = nsxy; v.zsx = zsx; v.zsxy = zsxy;
    v.nnode = nnode; v.nzone = zb / sizeof(double);  // zone array stride (aux/B planes)
    double **cur = nodes + 6 * par, **nxt = nodes + 6 * (1 - par);
    v.x = cur[0]; v.y = cur[1]; v.z = cur[2]; v.u = cur[3]; v.v = cur[4]; v.w = cur[5];
    v.xn = nxt[0]; v.yn = nxt[1]; v.zn = nxt[2]; v.un = nxt[3]; v.vn = nxt[4]; v.wn = nxt[5];
    v.e = par ? e1 : e0;
    v.en = par ? e0 : e1;
    v.m = m; v.P = P; v.B = B; v.aux = aux; v.mn8 = mn8; v.mi = mi;
    v.dom = dom;
  }
}

}  // namespace hydro

namespace {

bool group_node();

int alloc_domain(hydro_ctx *h, LocalDom &D, bool split) {
  const int64_t n0 = D.box.n[0], n1 = D.box.n[1], n2 = D.box.n[2];
  // node-stage tile height: chosen per domain, except for the grouped node launch and the
  // one-kernel variant, which are compiled for the default height only
  const bool fixed_ty = h->doms.size() > 1 && group_node();
  D.node_ty = h->one_kernel ? fused_tile_ty()
                            : (fixed_ty ? 12 : node_tile_ty((int)n0, (int)n1, (int)n2));
  const int64_t nsx = (n0 + 3 + 3) / 4 * 4, nsxy = nsx * (n1 + 3), nnode = nsxy * (n2 + 3);
  const int64_t zsx = (n0 + 2 + 3) / 4 * 4, zsxy = zsx * (n1 + 2);
  if (nnode >= (int64_t(1) << 31))  // the cycle kernels index a domain's storage with int32
    return set_err(h, HYDRO_EINVAL, "domain too large: split it into more domains (< 2^31 nodes)");
  const size_t bytes = domain_bytes(D.box, split);
  CK(cudaMalloc(&D.mem, bytes));
  CK(cudaMemsetAsync(D.mem, 0, bytes, h->stream));
  D.bytes = bytes;
  carve_views(D.mem, D.box, h->L.N, D.dom, split, D.view);
  // TMA descriptors (3-D tiled, fp64, box FUSED_BOX_X x (TY+3) x 1; out-of-bounds zero fill)
  static PFN_cuTensorMapEncodeTiled_v12000 encode = nullptr;
  if (!encode) {
    cudaDriverEntryPointQueryResult q;
    void *fn = nullptr;
    CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q));
    if (!fn || q != cudaDriverEntryPointSuccess)
      return set_err(h, HYDRO_ECUDA, "cuTensorMapEncodeTiled unavailable");
    encode = (PFN_cuTensorMapEncodeTiled_v12000)fn;
  }
  for (int par = 0; par < 2; ++par) {
    const double *arr[7] = {D.view[par].x, D.view[par].y, D.view[par].z,
                            D.view[par].u, D.view[par].v, D.view[par].w, D.view[par].mn8};
    const double *zarr[4] = {D.view[par].m, D.view[par].e, D.view[par].P, D.view[par].mi};
    for (int kind = 0; kind < 2; ++kind) {
      NodeMaps &M = kind ? D.zmaps[par] : D.maps[par];
      for (int f = 0; f < 11; ++f) {
        const bool zf = f >= 6 && f < 10;
        const int64_t sx = zf ? zsx : nsx, sy = zf ? (n1 + 2) : (n1 + 3);
        const int64_t sz = zf ? (n2 + 2) : (n2 + 3), sxy = zf ? zsxy : nsxy;
        cuuint64_t dims[3] = {(cuuint64_t)sx, (cuuint64_t)sy, (cuuint64_t)sz};
        cuuint64_t strides[2] = {(cuuint64_t)(sx * sizeof(double)),
                                 (cuuint64_t)(sxy * sizeof(double))};
        cuuint32_t box[3];
        if (zf) {
          box[0] = (cuuint32_t)cycle_zone_box_x();
          box[1] = (cuuint32_t)cycle_zone_box_y(D.node_ty);
        } else {
          box[0] = kind ? (cuuint32_t)ZONE_BOX_X : (cuuint32_t)FUSED_BOX_X;
          box[1] = kind ? (cuuint32_t)zone_box_y() : (cuuint32_t)node_box_y(D.node_ty);
        }
        box[2] = 1;
        cuuint32_t es[3] = {1, 1, 1};
        CUtensorMap *dst = zf ? &M.z[f - 6] : &M.m[f == 10 ? 6 : f];
        // L2 promotion: the node-stage maps keep 256 B (adjacent CTAs at the same z read the
        // neighbouring bytes of a promoted line; 128/64/none measured 1-2 % slower); the
        // persistent zone stage's CTAs sit at different z, so a promoted line's other half is
        // rarely reused: 64 B cuts its DRAM reads at 512^3 from 121 to 94 B/zone (ncu) and its
        // time by 1 % (HYDRO_ZPROMO / HYDRO_NPROMO: 0 none, 1 64 B, 2 128 B, 3 256 B)
        static const int zpromo = getenv("HYDRO_ZPROMO") ? atoi(getenv("HYDRO_ZPROMO")) : 1;
        static const int npromo = getenv("HYDRO_NPROMO") ? atoi(getenv("HYDRO_NPROMO")) : 3;
        const CUtensorMapL2promotion promos[4] = {
            CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_64B,
            CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B};
        const int pi = std::max(0, std::min(3, (kind && !zf) ? zpromo : npromo));
        CUresult r = encode(dst, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 3,
                            const_cast<double *>(zf ? zarr[f - 6] : arr[f == 10 ? 6 : f]), dims, strides, box,
                            es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                            promos[pi], CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        if (r != CUDA_SUCCESS) return set_err(h, HYDRO_ECUDA, "cuTensorMapEncodeTiled failed");
      }
    }
  }
  return HYDRO_OK;
}

// Copy a global box between a dense host array (dims gdims, x fastest) and a domain's local
// array (local index of global g is g - lo + 1 along each axis).
int copy_box(hydro_ctx *h, bool to_device, double *host, const int64_t gdims[3],
             const int64_t glo[3], const int64_t ext[3], double *dev, int64_t dsx, int64_t dsy,
             const int64_t dlo_local[3], cudaStream_t s) {
  if (ext[0] <= 0 || ext[1] <= 0 || ext[2] <= 0) return HYDRO_OK;
  double *dbox = dev + (dlo_local[2] * dsy + dlo_local[1]) * dsx + dlo_local[0];
  if (ext[0] == gdims[0] && ext[1] == gdims[1]) {
    // the host box is contiguous (whole planes): one full-bandwidth DMA through a device staging
    // buffer and a strided copy kernel on the device
    const size_t n = (size_t)ext[0] * ext[1] * ext[2];
    if (n > h->stage_cap) {
      if (h->stage) CK(cudaFreeAsync(h->stage, s));
      CK(cudaMallocAsync(&h->stage, n * sizeof(double), s));
      h->stage_cap = n;
    }
    double *hbox = host + (glo[2] * gdims[1] + glo[1]) * gdims[0] + glo[0];
    if (to_device) {
      CK(cudaMemcpyAsync(h->stage, hbox, n * sizeof(double), cudaMemcpyHostToDevice, s));
      launch_copy3d(h->stage, ext[0], ext[0] * ext[1], dbox, dsx, dsx * dsy, (int)ext[0],
                    (int)ext[1], (int)ext[2], s);
    } else {
      launch_copy3d(dbox, dsx, dsx * dsy, h->stage, ext[0], ext[0] * ext[1], (int)ext[0],
                    (int)ext[1], (int)ext[2], s);
      CK(cudaMemcpyAsync(hbox, h->stage, n * sizeof(double), cudaMemcpyDeviceToHost, s));
    }
    CK(cudaGetLastError());
    return HYDRO_OK;
  }
  cudaMemcpy3DParms p;
  std::memset(&p, 0, sizeof(p));
  cudaPitchedPtr hp = make_cudaPitchedPtr(host, gdims[0] * sizeof(double), gdims[0], gdims[1]);
  cudaPitchedPtr dp = make_cudaPitchedPtr(dev, dsx * sizeof(double), dsx, dsy);
  cudaPos hpos = make_cudaPos(glo[0] * sizeof(double), glo[1], glo[2]);
  cudaPos dpos = make_cudaPos(dlo_local[0] * sizeof(double), dlo_local[1], dlo_local[2]);
  p.extent = make_cudaExtent(ext[0] * sizeof(double), ext[1], ext[2]);
  if (to_device) {
    p.srcPtr = hp; p.srcPos = hpos; p.dstPtr = dp; p.dstPos = dpos;
    p.kind = cudaMemcpyHostToDevice;
  } else {
    p.srcPtr = dp; p.srcPos = dpos; p.dstPtr = hp; p.dstPos = hpos;
    p.kind = cudaMemcpyDeviceToHost;
  }
  CK(cudaMemcpy3DAsync(&p, s));
  return HYDRO_OK;
}

// Upload global host arrays into every local domain's parity-p arrays (existing owned+ghost
// entries).  nodes6 may be NULL; zone arrays: e -> e, z6 (rho or mass) -> P scratch or m.
int upload_state(hydro_ctx *h, int par, const double *const *nodes6, const double *e,
                 const double *zone_extra, bool extra_is_mass) {
  const int64_t gn[3] = {h->L.N[0] + 1, h->L.N[1] + 1, h->L.N[2] + 1};
  const int64_t gz[3] = {h->L.N[0], h->L.N[1], h->L.N[2]};
  for (LocalDom &D : h->doms) {
    DomView &v = D.view[par];
    int64_t nlo[3], next[3], nloc[3], zlo[3], zext[3], zloc[3];
    for (int a = 0; a < 3; ++a) {
      const int64_t lo = std::max<int64_t>(D.box.lo[a] - 1, 0);
      const int64_t hi = std::min<int64_t>(D.box.lo[a] + D.box.n[a] + 1, h->L.N[a]);  // nodes
      nlo[a] = lo; next[a] = hi - lo + 1; nloc[a] = lo - D.box.lo[a] + 1;
      const int64_t zl = std::max<int64_t>(D.box.lo[a] - 1, 0);
      const int64_t zh = std::min<int64_t>(D.box.lo[a] + D.box.n[a] + 1, h->L.N[a]);  // excl
      zlo[a] = zl; zext[a] = zh - zl; zloc[a] = zl - D.box.lo[a] + 1;
    }
    if (nodes6) {
      double *dst[6] = {const_cast<double *>(v.x), const_cast<double *>(v.y),
                        const_cast<double *>(v.z), const_cast<double *>(v.u),
                        const_cast<double *>(v.v), const_cast<double *>(v.w)};
      for (int f = 0; f < 6; ++f) {
        int rc = copy_box(h, true, const_cast<double *>(nodes6[f]), gn, nlo, next, dst[f], v.nsx,
                          v.nsxy / v.nsx, nloc, h->stream);
        if (rc) return rc;
      }
    }
    if (e) {
      int rc = copy_box(h, true, const_cast<double *>(e), gz, zlo, zext,
                        const_cast<double *>(v.e), v.zsx, v.zsxy / v.zsx, zloc, h->stream);
      if (rc) return rc;
    }
    if (zone_extra) {
      double *dst = extra_is_mass ? const_cast<double *>(v.m) : v.P;
      int rc = copy_box(h, true, const_cast<double *>(zone_extra), gz, zlo, zext, dst, v.zsx,
                        v.zsxy / v.zsx, zloc, h->stream);
      if (rc) return rc;
    }
  }
  return HYDRO_OK;
}

// S9 can run inside the cycle's last kernel when that kernel is the only one of the cycle (one
// domain, one rank, not the plain split path).  Measured on B200 at 128^3 it is slower (the
// per-CTA __threadfence before the ticket delays every CTA's exit: node stage 106 -> 110 us,
// while a separate k_finalize costs ~2.6 us; re-measured with the current node stage
// (tools/gp_fold.sh): 140.4 vs 139.1 us per cycle), so it is off unless built with -DHYDRO_FOLD.
int fold_finalize(const hydro_ctx *h) {
#ifndef HYDRO_FOLD
  (void)h;
  return 0;
#endif
  return (!h->split && h->doms.size() == 1 && !h->comm && !h->peer && h->n_local_pairs == 0) ? 1
                                                                                           : 0;
}

void launch_node_stage(hydro_ctx *h, LocalDom &D, int par, int slot, cudaStream_t s) {
  const bool p = h->fused_halo && h->push_dev[par] && h->push_count[slot] > 0;
  launch_node_energy(D.view[par], D.maps[par], h->ph, h->st, fold_finalize(h),
                     p ? h->push_dev[par] + h->push_first[slot] : nullptr,
                     p ? h->push_count[slot] : 0, D.node_ty, s);
}

void launch_zone_stages(hydro_ctx *h, int par, cudaStream_t s) {
  if (h->group)
    launch_zone_stage_group(h->views_dev[par], h->zmaps_dev[par], h->ztasks_dev, h->zunits,
                            h->ph, h->st, s);
  else
    for (size_t i = 0; i < h->doms.size(); ++i)
      launch_zone_stage(h->doms[i].view[par], h->doms[i].zmaps[par], h->ring[i], h->ph, h->st,
                        s);
  // P of the ring zones the zone stages skipped, from their owners on this GPU
  if (h->n_pcopy) launch_halo_copy(h->views_dev[par], h->pcopy_dev, h->n_pcopy, s);
}

// The grouped node/energy launch is measured slower on large domains (512^3 in 8 domains: 695
// vs 614 us per domain; uneven 448^3: equal), so per-domain launches stay the default;
// HYDRO_GROUP_NODE=1 selects it (A/B).
bool group_node() {
  static const int on = getenv("HYDRO_GROUP_NODE") ? atoi(getenv("HYDRO_GROUP_NODE")) : 0;
  return on != 0;
}

void launch_node_stages(hydro_ctx *h, int par, cudaStream_t s, bool with_halo = false) {
  if (h->group && group_node()) {
    launch_node_energy_group(h->ntasks_dev, (int)h->doms.size(), h->nctas, h->views_dev[par],
                             h->nmaps_dev[par], h->ph, h->st,
                             h->fused_halo ? h->push_dev[par] : nullptr, s);
  } else if (h->nstreams > 1 && h->doms.size() > 1) {  // independent domains: parallel branches
    cudaEventRecord(h->fork_ev, s);
    for (int k = 1; k < h->nstreams; ++k) cudaStreamWaitEvent(h->side[k], h->fork_ev, 0);
    for (size_t oi = 0; oi < h->node_order.size(); ++oi) {
      const size_t i = (size_t)h->node_order[oi];
      const int k = h->node_stream[i];
      launch_node_stage(h, h->doms[i], par, (int)i, k ? h->side[k] : s);
      // this domain's outgoing ghost slabs, while the other streams' node stages run: a source
      // element is owned (never a ghost), and the destinations are next-parity ghosts that no
      // node/energy stage writes or reads this cycle
      if (with_halo && h->halo_overlap == 3 && h->stream_last[k] == oi) {
        // the last domain of this stream: copy the slabs of all of the stream's domains (one
        // contiguous range: the chunks are sorted by (stream, source))
        int32_t first = -1, count = 0;
        for (size_t j = 0; j < h->doms.size(); ++j)
          if (h->node_stream[j] == k && h->halo_count[j] > 0) {
            if (first < 0 || h->halo_first[j] < first) first = h->halo_first[j];
            count += h->halo_count[j];
          }
        if (count > 0)
          launch_halo_copy(h->views_dev[par], h->local_pairs_dev + first, count,
                           k ? h->side[k] : s);
      } else if (with_halo && h->halo_overlap <= 2 && h->halo_count[i] > 0) {
        cudaStream_t cs = k ? h->side[k] : s;
        if (h->halo_overlap == 2) {  // the node-stage stream goes on to its next domain
          cudaEventRecord(h->node_done[i], cs);
          cudaStreamWaitEvent(h->halo_stream, h->node_done[i], 0);
          cs = h->halo_stream;
        }
        launch_halo_copy(h->views_dev[par], h->local_pairs_dev + h->halo_first[i],
                         h->halo_count[i], cs);
      }
    }
    if (with_halo && h->halo_overlap == 2) {
      cudaEventRecord(h->halo_join, h->halo_stream);
      cudaStreamWaitEvent(s, h->halo_join, 0);
    }
    for (int k = 1; k < h->nstreams; ++k) {
      cudaEventRecord(h->join_ev[k], h->side[k]);
      cudaStreamWaitEvent(s, h->join_ev[k], 0);
    }
  } else {
    for (size_t i = 0; i < h->doms.size(); ++i) launch_node_stage(h, h->doms[i], par, (int)i, s);
  }
}

// Fused-halo tables: per parity, the PushSlabs of every local source domain,
// grouped by source slot (push_first / push_count), in source-local boxes.
int build_push_tables(hydro_ctx *h) {
  const int ns = (int)h->doms.size();
  h->push_first.assign(ns, 0);
  h->push_count.assign(ns, 0);
  std::vector<PushSlab> tab[2];
  for (int slot = 0; slot < ns; ++slot) {
    h->push_first[slot] = (int)tab[0].size();
    for (const PushTarget &T : h->push_targets) {
      if (T.src_slot != slot) continue;
      for (int par = 0; par < 2; ++par) {
        const DomView &S = h->doms[slot].view[par];
        const DomView &D = T.dst[par];
        PushSlab p = {};
        int o[3];
        for (int a = 0; a < 3; ++a) {
          p.nlo[a] = (int32_t)(T.nlo[a] - S.lo[a]);
          p.nhi[a] = (int32_t)(T.nhi[a] - S.lo[a]);
          p.zlo[a] = (int32_t)(T.zlo[a] - S.lo[a]);
          p.zhi[a] = (int32_t)(T.zhi[a] - S.lo[a]);
          o[a] = (int)(S.lo[a] - D.lo[a]);  // source-local -> destination-local offset
        }
        p.nbase = D.nid(o[0], o[1], o[2]);
        p.zbase = D.zid(o[0], o[1], o[2]);
        p.nsx = (int32_t)D.nsx;
        p.nsxy = (int32_t)D.nsxy;
        p.zsx = (int32_t)D.zsx;
        p.zsxy = (int32_t)D.zsxy;
        double *dst[7] = {D.xn, D.yn, D.zn, D.un, D.vn, D.wn, D.en};
        for (int f = 0; f < 7; ++f) p.dst[f] = dst[f];
        p.remote = T.remote;
        tab[par].push_back(p);
      }
    }
    h->push_count[slot] = (int)tab[0].size() - h->push_first[slot];
    if (h->push_count[slot] > 32)  // one warp lane per slab (kernel_cycle.cu push_halo)
      return set_err(h, HYDRO_EINVAL, "fused halo: more than 32 ghost slabs from one domain");
  }
  for (int par = 0; par < 2; ++par) {
    if (h->push_dev[par]) CK(cudaFree(h->push_dev[par]));
    h->push_dev[par] = nullptr;
    if (tab[par].empty()) continue;
    CK(cudaMalloc(&h->push_dev[par], sizeof(PushSlab) * tab[par].size()));
    CK(cudaMemcpy(h->push_dev[par], tab[par].data(), sizeof(PushSlab) * tab[par].size(),
                  cudaMemcpyHostToDevice));
  }
  if (h->group && h->ntasks_dev) {
    for (int i = 0; i < ns; ++i) {
      h->ntasks_host[i].push0 = h->push_first[i];
      h->ntasks_host[i].npush = h->push_count[i];
    }
    CK(cudaMemcpy(h->ntasks_dev, h->ntasks_host.data(), sizeof(NodeTask) * ns,
                  cudaMemcpyHostToDevice));
  }
  return HYDRO_OK;
}

// Reading R24: strain rates of every local domain's owned zones (at x_p, or at x with at_x),
// before any kernel reads a limiter (limiters read their neighbours' owners).
void launch_strains(hydro_ctx *h, int par, int at_x, cudaStream_t s) {
  if (h->ph.q_kind != 1) return;
  for (LocalDom &D : h->doms) {
    if (h->strict) launch_strict_strain(D.view[par], h->st, at_x, s);
    else launch_strain(D.view[par], h->st, at_x, s);
  }
}

// Split pipeline (plain or STRICT): zone kernels of every domain, the dt / error reduction,
// then node and energy kernels.
int enqueue_split(hydro_ctx *h, int par, cudaStream_t s) {
  launch_strains(h, par, 0, s);
  for (LocalDom &D : h->doms) {
    if (h->strict) launch_strict_zone(D.view[par], h->ph, h->st, h->mono, s);
    else launch_zone_split(D.view[par], h->ph, h->st, h->mono, s);
  }
  if (h->comm) {
    int rc = comm_dt_min(h->comm, h->st, s);
    if (rc) return set_err(h, rc, "dt allreduce failed");
  }
  for (LocalDom &D : h->doms) {
    if (h->strict) launch_strict_node(D.view[par], h->ph, h->st, s);
    else launch_node_split(D.view[par], h->ph, h->st, s);
  }
  for (LocalDom &D : h->doms) {
    if (h->strict) launch_strict_energy(D.view[par], h->ph, h->st, s);
    else launch_energy_split(D.view[par], h->ph, h->st, s);
  }
  return HYDRO_OK;
}

// Enqueue one cycle on stream s reading parity `par`.
int enqueue_cycle(hydro_ctx *h, int par, cudaStream_t s) {
  if (h->split) {
    int rc = enqueue_split(h, par, s);
    if (rc) return rc;
  } else if (h->one_kernel) {
    for (LocalDom &D : h->doms) launch_cycle_fused(D.view[par], D.maps[par], h->ph, h->st, fold_finalize(h), s);
    if (h->comm) {
      int rc = comm_dt_min(h->comm, h->st, s);
      if (rc) return set_err(h, rc, "dt allreduce failed");
    }
  } else {
    launch_zone_stages(h, par, s);
    if (h->comm) {  // dt_{n+1} is first read by S9: the reduction overlaps the node stages
      int rc = comm_dt_min_async(h->comm, h->st, s);
      if (rc) return set_err(h, rc, "dt allreduce failed");
    }
    launch_node_stages(h, par, s, h->halo_overlap);
  }
  if (!h->fused_halo && !(h->halo_overlap && !h->split && !h->one_kernel))
    launch_halo_copy(h->views_dev[par], h->local_pairs_dev, h->n_local_pairs, s);
  if (h->comm) {
    int rc = comm_halo(h->comm, par, s);
    if (rc) return set_err(h, rc, "halo exchange failed");
  }
  if (h->peer) {  // halo push into the peers (unless fused) + dt / error reduction
    int rc = peer_exchange(h->peer, h->views_dev[par], par, !h->fused_halo, h->st, s);
    if (rc) return set_err(h, rc, "peer exchange failed");
  }
  if (h->comm && !h->split && !h->one_kernel) {
    int rc = comm_dt_join(h->comm, s);
    if (rc) return set_err(h, rc, "dt allreduce join failed");
  }
  if (!fold_finalize(h)) launch_finalize(h->st, h->ph, s);
  CK(cudaGetLastError());
  return HYDRO_OK;
}

int capture_cycles(hydro_ctx *h, int par, int k, cudaGraphExec_t *out) {
  cudaGraph_t g;
  CK(cudaStreamBeginCapture(h->stream, cudaStreamCaptureModeThreadLocal));
  int rc = HYDRO_OK;
  for (int c = 0; c < k && rc == HYDRO_OK; ++c) rc = enqueue_cycle(h, par ^ (c & 1), h->stream);
  cudaError_t e = cudaStreamEndCapture(h->stream, &g);
  if (rc) return rc;
  if (e != cudaSuccess) return set_err(h, HYDRO_ECUDA, cudaGetErrorString(e));
  CK(cudaGraphInstantiate(out, g, 0));
  CK(cudaGraphDestroy(g));
  return HYDRO_OK;
}

// One-cycle graphs per parity, plus graph_k-cycle graphs (HYDRO_GRAPH_CYCLES, default 8;
// measured at 128^3: K = 1 / 2 / 4 / 8 -> 142.7 / 141.3 / 140.6 / 140.3 us per cycle).
int build_graphs(hydro_ctx *h) {
  const char *env = getenv("HYDRO_GRAPH_CYCLES");
  h->graph_k = env ? std::max(1, atoi(env)) : 8;
  for (int par = 0; par < 2; ++par) {
    int rc = capture_cycles(h, par, 1, &h->graph[par]);
    if (rc) return rc;
    if (h->graph_k > 1 && (rc = capture_cycles(h, par, h->graph_k, &h->graphk[par])) != HYDRO_OK)
      return rc;
  }
  return HYDRO_OK;
}

// Device state -> info.  The status is already identical on every rank (the error bits are
// OR-reduced with dt every cycle by both transports), so this is not a collective.
int read_info(hydro_ctx *h, hydro_info *info, cudaStream_t s) {
  DevState st;
  CK(cudaMemcpyAsync(&st, h->st, sizeof(st), cudaMemcpyDeviceToHost, s));
  if (h->comm) {  // poll NCCL while the cycles drain (HYDRO_NCCL_TIMEOUT_S, default 600 s)
    static const double tmo =
        getenv("HYDRO_NCCL_TIMEOUT_S") ? atof(getenv("HYDRO_NCCL_TIMEOUT_S")) : 600.0;
    int rc = comm_wait(h->comm, s, tmo, &h->err);
    if (rc) return set_err(h, rc, h->err);
  }
  CK(cudaStreamSynchronize(s));
  int status = HYDRO_OK;
  if (st.halted & ERR_TANGLED) status = HYDRO_ETANGLED;
  else if (st.halted & ERR_NONFINITE) status = HYDRO_ENONFINITE;
  else if (st.halted & ERR_DTMIN) status = HYDRO_EDTMIN;
  if (info) {
    info->t = st.t;
    info->dt = st.dt;
    info->cycle = (int64_t)st.cycle;
    info->dt_min_zone = st.dtz_last;
    info->status = status;
    info->bad_zone = (st.bad_zone == ~0ull) ? -1 : (int64_t)st.bad_zone;
  }
  return status;
}

bool valid_phys(const hydro_config *c) {
  return c->gamma > 1.0 && c->q_lin >= 0.0 && c->q_quad >= 0.0 && c->cfl > 0.0 &&
         c->c_vol > 0.0 && c->dt_growth > 0.0 && c->dt_max > 0.0 && !std::isnan(c->dt_floor) &&
         std::isfinite(c->origin[0]) && c->extent[0] > 0.0 && c->extent[1] > 0.0 &&
         c->extent[2] > 0.0 && c->hg_coef >= 0.0 && std::isfinite(c->hg_coef);
}

}  // namespace

extern "C" {

int hydro_abi_version(void) { return HYDRO_ABI_VERSION; }

void hydro_config_default(hydro_config *c) {
  std::memset(c, 0, sizeof(*c));
  c->abi_version = HYDRO_ABI_VERSION;
  for (int a = 0; a < 3; ++a) {
    c->n[a] = 32;
    c->origin[a] = 0.0;
    c->extent[a] = 1.2;
    c->ndom[a] = 1;
  }
  c->gamma = 1.4;
  c->q_lin = 0.5;
  c->q_quad = 2.0;
  c->cfl = 0.3;
  c->c_vol = 0.1;
  c->dt_growth = 1.1;
  c->dt_max = INFINITY;
  c->dt_init = INFINITY;
  c->reflect_mask = 0x3f;
  c->init_kind = HYDRO_INIT_SEDOV;
  c->rho0 = 1.0;
  c->sedov_energy = 0.851072 / 8.0;
  c->nranks = 1;
}

const char *hydro_strerror(int s) {
  switch (s) {
    case HYDRO_OK: return "ok";
    case HYDRO_EINVAL: return "invalid argument";
    case HYDRO_ENOMEM: return "out of memory";
    case HYDRO_ECUDA: return "CUDA error";
    case HYDRO_ENCCL: return "communicator error";
    case HYDRO_ETANGLED: return "tangled mesh (zone volume <= 0)";
    case HYDRO_ENONFINITE: return "non-finite pressure or dt";
    case HYDRO_EDTMIN: return "dt below floor";
    case HYDRO_ESTATE: return "context in failed state";
    default: return "unknown status";
  }
}

const char *hydro_last_error(const hydro_ctx *h) { return h ? h->err.c_str() : g_err.c_str(); }

int hydro_comm_unique_id(void *out128) { return comm_unique_id(out128); }

int hydro_create(const hydro_config *cfg, hydro_ctx **out) {
  NvtxRange nvtx_("hydro_create");
  hydro_ctx *h = nullptr;
  if (!cfg || !out) return set_err(nullptr, HYDRO_EINVAL, "NULL argument");
  *out = nullptr;
  if (cfg->abi_version != HYDRO_ABI_VERSION)
    return set_err(nullptr, HYDRO_EINVAL, "abi_version mismatch");
  if (!valid_phys(cfg)) return set_err(nullptr, HYDRO_EINVAL, "invalid physics parameters");
  if (cfg->init_kind < 0 || cfg->init_kind > 2)
    return set_err(nullptr, HYDRO_EINVAL, "invalid init_kind");
  if (cfg->q_kind < 0 || cfg->q_kind > 1) return set_err(nullptr, HYDRO_EINVAL, "invalid q_kind");
  if (cfg->q_kind == 1 && cfg->nranks > 1)  // limiters read zones two layers out (R24)
    return set_err(nullptr, HYDRO_EINVAL, "monotone q needs a single rank");
  if (cfg->init_kind != HYDRO_INIT_SEDOV)
    for (int f = 0; f < 8; ++f)
      if (!cfg->user[f]) return set_err(nullptr, HYDRO_EINVAL, "USER init needs 8 arrays");
  h = new hydro_ctx();
  h->cfg = *cfg;
  std::memset(h->cfg.user, 0, sizeof(h->cfg.user));
  for (int a = 0; a < 3; ++a) h->cfg.cuts[a] = nullptr;
  h->cfg.dom_to_rank = nullptr;
  h->cfg.rank_weight = nullptr;
  h->cfg.comm_id = nullptr;
  std::string err;
  int rc = layout_build(cfg, &h->L, &err);
  if (rc) {
    delete h;
    return set_err(nullptr, rc, err);
  }
  h->ph.gamma = cfg->gamma;
  h->ph.gm1 = cfg->gamma - 1.0;
  h->ph.ggm1 = cfg->gamma * (cfg->gamma - 1.0);
  h->ph.q_lin = cfg->q_lin;
  h->ph.q_quad = cfg->q_quad;
  h->ph.cfl = cfg->cfl;
  h->ph.c_vol = cfg->c_vol;
  h->ph.dt_growth = cfg->dt_growth;
  h->ph.dt_max = cfg->dt_max;
  h->ph.t_stop = cfg->t_stop;
  h->ph.reflect_mask = cfg->reflect_mask;
  h->ph.hg = cfg->hg_coef;
  h->ph.q_kind = cfg->q_kind;
  // hourglass control (f1) needs per-corner forces, which only the split kernels carry
  h->strict = (cfg->flags & HYDRO_FLAG_STRICT) != 0;
  // hourglass control (f1, R17) and the monotone q (f1, R24) run on the split kernels
  h->split = (cfg->flags & HYDRO_FLAG_SPLIT) != 0 || cfg->hg_coef > 0.0 || h->strict ||
             cfg->q_kind == 1;
  h->one_kernel = !h->split && (cfg->flags & HYDRO_FLAG_ONE_KERNEL) != 0;
  h->use_graph = (cfg->flags & HYDRO_FLAG_NO_GRAPH) == 0;
  h->device = cfg->device;
  *out = nullptr;
  auto fail = [&](int code) {
    if (!h->err.empty()) g_err = h->err;  // hydro_last_error(NULL) after a failed create
    hydro_destroy(h);
    return code;
  };
  {
    int ndev = 0;
    cudaError_t e = cudaGetDeviceCount(&ndev);
    if (e != cudaSuccess || ndev == 0) {
      set_err(h, HYDRO_ECUDA, "no CUDA device available (the library has no CPU path)");
      return fail(HYDRO_ECUDA);
    }
  }
  if (cudaSetDevice(h->device) != cudaSuccess) {
    set_err(h, HYDRO_ECUDA, "cudaSetDevice failed");
    return fail(HYDRO_ECUDA);
  }
  if ((rc = [&]() -> int {
         CK(cudaStreamCreateWithFlags(&h->stream, cudaStreamNonBlocking));
         // measured (uneven 448^3, 64 domains): 1 / 2 / 4 streams -> 12.10 / 12.71 / 12.74 G;
         // neutral on the 4- and 8-domain configs
         h->nstreams = 4;
         if (const char *ns = getenv("HYDRO_NODE_STREAMS"))
           h->nstreams = std::max(1, std::min(4, atoi(ns)));
         if (h->nstreams > 1) {
           CK(cudaEventCreateWithFlags(&h->fork_ev, cudaEventDisableTiming));
           for (int k = 1; k < h->nstreams; ++k) {
             CK(cudaStreamCreateWithFlags(&h->side[k], cudaStreamNonBlocking));
             CK(cudaEventCreateWithFlags(&h->join_ev[k], cudaEventDisableTiming));
           }
         }
         CK(cudaMalloc(&h->st, sizeof(DevState)));
         DevState s0;
         std::memset(&s0, 0, sizeof(s0));
         s0.dtz_acc = (unsigned long long)0x7ff0000000000000ull;  // +inf
         s0.bad_zone = ~0ull;
         CK(cudaMemcpyAsync(h->st, &s0, sizeof(s0), cudaMemcpyHostToDevice, h->stream));
         h->slot_of_dom.assign(h->L.dom.size(), -1);
         for (size_t d = 0; d < h->L.dom.size(); ++d) {
           if (h->L.dom[d].rank != cfg->rank) continue;
           LocalDom D;
           D.dom = (int32_t)d;
           D.box = h->L.dom[d];
           h->slot_of_dom[d] = (int32_t)h->doms.size();
           h->doms.push_back(D);
         }
         for (LocalDom &D : h->doms) {
           int r = alloc_domain(h, D, h->split);
           if (r) return r;
         }
         if (h->ph.q_kind == 1) {  // R24: strain planes and owner tables (all domains local)
           for (LocalDom &D : h->doms) {
             void *p = nullptr;
             CK(cudaMalloc(&p, 3 * D.view[0].nzone * sizeof(double)));
             CK(cudaMemsetAsync(p, 0, 3 * D.view[0].nzone * sizeof(double), h->stream));
             h->mono_mem.push_back(p);
             D.view[0].eps = D.view[1].eps = (double *)p;
           }
           for (int a = 0; a < 3; ++a) {
             std::vector<int32_t> own(h->L.N[a]);
             for (int64_t g = 0; g < h->L.N[a]; ++g) {
               int d = 0;
               while (!(h->L.cuts[a][d] <= g && g < h->L.cuts[a][d + 1])) ++d;
               own[g] = d;
             }
             void *p = nullptr;
             CK(cudaMalloc(&p, own.size() * sizeof(int32_t)));
             CK(cudaMemcpy(p, own.data(), own.size() * sizeof(int32_t), cudaMemcpyHostToDevice));
             h->mono_mem.push_back(p);
             h->mono.zown[a] = (const int32_t *)p;
           }
           void *p = nullptr;
           CK(cudaMalloc(&p, h->slot_of_dom.size() * sizeof(int32_t)));
           CK(cudaMemcpy(p, h->slot_of_dom.data(), h->slot_of_dom.size() * sizeof(int32_t),
                         cudaMemcpyHostToDevice));
           h->mono_mem.push_back(p);
           h->mono.slot = (const int32_t *)p;
           h->mono.ndx = h->L.nd[0];
           h->mono.ndy = h->L.nd[1];
         }
         // device views and intra-GPU halo pairs
         for (int par = 0; par < 2; ++par) {
           CK(cudaMalloc(&h->views_dev[par], sizeof(DomView) * std::max<size_t>(1, h->doms.size())));
           std::vector<DomView> vv;
           for (LocalDom &D : h->doms) vv.push_back(D.view[par]);
           if (!vv.empty())
             CK(cudaMemcpyAsync(h->views_dev[par], vv.data(), sizeof(DomView) * vv.size(),
                                cudaMemcpyHostToDevice, h->stream));
         }
         // zone-stage rings: only on sides where a ghost zone is owned by another rank (the
         // rest is copied from the local owner after the zone stage; HYDRO_PRING=0: always
         // compute the ring, A/B)
         {
           const char *pr = getenv("HYDRO_PRING");
           const bool skip = !(pr && atoi(pr) == 0) && !h->split && !h->one_kernel;
           h->ring.assign(h->doms.size(), skip ? 0 : 0x3f);
           for (const HaloPair &P : h->L.pairs) {
             const int32_t ds = h->slot_of_dom[P.dst];
             if (!skip || ds < 0 || h->slot_of_dom[P.src] >= 0) continue;
             const DomainBox &b = h->doms[ds].box;
             bool empty = false;
             for (int a = 0; a < 3; ++a) empty |= P.zhi[a] <= P.zlo[a];
             if (empty) continue;
             for (int a = 0; a < 3; ++a) {
               if (P.zhi[a] <= b.lo[a]) h->ring[ds] |= (uint8_t)(1u << (2 * a));
               if (P.zlo[a] >= b.lo[a] + b.n[a]) h->ring[ds] |= (uint8_t)(1u << (2 * a + 1));
             }
           }
         }
         h->mono.views = h->views_dev[0];  // parity-free fields only (lo, strides, eps)
         // several domains on this GPU: one grouped zone-stage launch covers them all
         // (HYDRO_NO_GROUP=1: one launch per domain, for A/B)
         h->group = h->doms.size() > 1 && !h->split && !h->one_kernel &&
                    !(getenv("HYDRO_NO_GROUP") && atoi(getenv("HYDRO_NO_GROUP")));
         if (h->group) {
           std::vector<DomView> vv;
           for (LocalDom &D : h->doms) vv.push_back(D.view[0]);
           std::vector<ZoneTask> tasks(vv.size());
           zone_group_tasks(vv.data(), h->ring.data(), (int)vv.size(), tasks.data(), &h->zunits);
           CK(cudaMalloc(&h->ztasks_dev, sizeof(ZoneTask) * tasks.size()));
           CK(cudaMemcpy(h->ztasks_dev, tasks.data(), sizeof(ZoneTask) * tasks.size(),
                         cudaMemcpyHostToDevice));
           for (int par = 0; par < 2; ++par) {
             std::vector<NodeMaps> mm, nm;
             for (LocalDom &D : h->doms) {
               mm.push_back(D.zmaps[par]);
               nm.push_back(D.maps[par]);
             }
             CK(cudaMalloc(&h->zmaps_dev[par], sizeof(NodeMaps) * mm.size()));
             CK(cudaMemcpy(h->zmaps_dev[par], mm.data(), sizeof(NodeMaps) * mm.size(),
                           cudaMemcpyHostToDevice));
             CK(cudaMalloc(&h->nmaps_dev[par], sizeof(NodeMaps) * nm.size()));
             CK(cudaMemcpy(h->nmaps_dev[par], nm.data(), sizeof(NodeMaps) * nm.size(),
                           cudaMemcpyHostToDevice));
           }
           std::vector<NodeTask> &nt = h->ntasks_host;
           nt.resize(vv.size());
           h->nctas = node_group_tasks(vv.data(), (int)vv.size(), nt.data());
           CK(cudaMalloc(&h->ntasks_dev, sizeof(NodeTask) * nt.size()));
           CK(cudaMemcpy(h->ntasks_dev, nt.data(), sizeof(NodeTask) * nt.size(),
                         cudaMemcpyHostToDevice));
         }
         std::vector<HaloCopy> lp, pc;
         std::vector<HaloPair> remote;
         // HYDRO_FLAG_COMM_SELF: the same-rank ghost slabs go through NCCL self send/recv
         // (comm_plan self_all) instead of the intra-GPU copy; only their P copies stay
         const bool self_halo = (cfg->flags & HYDRO_FLAG_COMM_SELF) != 0;
         for (const HaloPair &P : h->L.pairs) {
           const bool dst_local = h->slot_of_dom[P.dst] >= 0;
           const bool src_local = h->slot_of_dom[P.src] >= 0;
           if (dst_local && src_local) {
             PushTarget pt;
             pt.src_slot = h->slot_of_dom[P.src];
             pt.remote = 0;
             for (int a = 0; a < 3; ++a) {
               pt.nlo[a] = P.nlo[a]; pt.nhi[a] = P.nhi[a];
               pt.zlo[a] = P.zlo[a]; pt.zhi[a] = P.zhi[a];
             }
             pt.dst[0] = h->doms[h->slot_of_dom[P.dst]].view[0];
             pt.dst[1] = h->doms[h->slot_of_dom[P.dst]].view[1];
             h->push_targets.push_back(pt);
             HaloCopy c;
             c.dst = h->slot_of_dom[P.dst];
             c.src = h->slot_of_dom[P.src];
             int64_t nn = 1, nz = 1;
             for (int a = 0; a < 3; ++a) {
               c.nlo[a] = P.nlo[a]; c.nhi[a] = P.nhi[a]; c.zlo[a] = P.zlo[a]; c.zhi[a] = P.zhi[a];
               nn *= P.nhi[a] - P.nlo[a];
               nz *= P.zhi[a] - P.zlo[a];
             }
             // chunks of HALO_CHUNK elements: the node slab, then the zone slab; the zone slab
             // once more for P when the destination's zone stage skips its ring there
             for (int kind = 0; kind < 3; ++kind) {
               if (kind == 2 && h->ring[c.dst] == 0x3f) continue;
               if (kind < 2 && self_halo) continue;
               const int64_t total = kind ? nz : nn;
               for (int64_t st = 0; st < total; st += HALO_CHUNK) {
                 c.kind = kind;
                 c.start = (int32_t)st;
                 c.count = (int32_t)std::min<int64_t>(HALO_CHUNK, total - st);
                 (kind == 2 ? pc : lp).push_back(c);
               }
             }
           } else if (dst_local || src_local) {
             remote.push_back(P);
           }
         }
         // chunks grouped by source slot (any order is correct: each chunk is independent)
         // node-stage streams: LPT on the domain sizes (largest first onto the least-loaded
         // stream), launched largest first, so small domains fill the other streams' tails
         {
           const size_t nd = h->doms.size();
           const int ns = std::max(1, h->nstreams);
           const char *lpt_env = getenv("HYDRO_NODE_LPT");
           const bool lpt = !lpt_env || atoi(lpt_env) != 0;
           h->node_order.resize(nd);
           h->node_stream.assign(nd, 0);
           for (size_t i = 0; i < nd; ++i) h->node_order[i] = (int32_t)i;
           auto zones = [&](int32_t i) {
             const DomainBox &b = h->doms[i].box;
             return (int64_t)b.n[0] * b.n[1] * b.n[2];
           };
           if (lpt) {
             std::stable_sort(h->node_order.begin(), h->node_order.end(),
                              [&](int32_t a, int32_t b) { return zones(a) > zones(b); });
             std::vector<int64_t> load(ns, 0);
             for (int32_t i : h->node_order) {
               const int k = (int)(std::min_element(load.begin(), load.end()) - load.begin());
               h->node_stream[i] = k;
               load[k] += zones(i);
             }
           } else {
             for (size_t i = 0; i < nd; ++i) h->node_stream[i] = (int32_t)(i % ns);
           }
           h->stream_last.assign(ns, (size_t)-1);
           for (size_t oi = 0; oi < nd; ++oi) h->stream_last[h->node_stream[h->node_order[oi]]] = oi;
           // halo chunks sorted by (stream of the source's node stage, source): per-domain and
           // per-stream ranges
           std::stable_sort(lp.begin(), lp.end(), [h](const HaloCopy &a, const HaloCopy &b) {
             const int sa = h->node_stream[a.src], sb = h->node_stream[b.src];
             return sa != sb ? sa < sb : a.src < b.src;
           });
         }
         h->halo_first.assign(h->doms.size(), 0);
         h->halo_count.assign(h->doms.size(), 0);
         for (size_t c = 0; c < lp.size(); ++c) {
           if (h->halo_count[lp[c].src] == 0) h->halo_first[lp[c].src] = (int32_t)c;
           ++h->halo_count[lp[c].src];
         }
         h->n_local_pairs = (int)lp.size();  // chunk entries
         h->fused_halo = !h->split && !h->one_kernel && (cfg->flags & HYDRO_FLAG_HALO_FUSED);
         {
           const char *ov = getenv("HYDRO_HALO_OVERLAP");
           // measured: per-stream copies (3) gain 0.3-0.7 % with 4 and 8 large
           // domains; with 64 uneven domains every overlapped mode loses (a copy CTA occupies an
           // SM's register file, so node-stage CTAs wait behind the slow sector-bound copies),
           // and the single copy after the join stays
           const int mode = ov ? atoi(ov) : (h->doms.size() <= 2 * (size_t)h->nstreams ? 3 : 0);
           if (!h->fused_halo && !h->split && !h->one_kernel && !group_node() &&
               h->nstreams > 1 && h->doms.size() > 1 && !lp.empty() && mode > 0)
             h->halo_overlap = std::min(mode, 3);
           if (h->halo_overlap == 2) {
             CK(cudaStreamCreateWithFlags(&h->halo_stream, cudaStreamNonBlocking));
             CK(cudaEventCreateWithFlags(&h->halo_join, cudaEventDisableTiming));
             h->node_done.assign(h->doms.size(), nullptr);
             for (cudaEvent_t &e : h->node_done)
               CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
           }
         }
         if (h->fused_halo) {
           int r = build_push_tables(h);
           if (r) return r;
         }
         if (!pc.empty()) {
           CK(cudaMalloc(&h->pcopy_dev, sizeof(HaloCopy) * pc.size()));
           CK(cudaMemcpyAsync(h->pcopy_dev, pc.data(), sizeof(HaloCopy) * pc.size(),
                              cudaMemcpyHostToDevice, h->stream));
           h->n_pcopy = (int)pc.size();
         }
         if (!lp.empty()) {
           CK(cudaMalloc(&h->local_pairs_dev, sizeof(HaloCopy) * lp.size()));
           CK(cudaMemcpyAsync(h->local_pairs_dev, lp.data(), sizeof(HaloCopy) * lp.size(),
                              cudaMemcpyHostToDevice, h->stream));
         }
         if (cfg->nranks > 1 && (cfg->flags & HYDRO_FLAG_PEER)) {
           int r = peer_create(&h->peer, cfg, &h->err);
           if (r) return r;
         } else if (cfg->nranks > 1 || (cfg->flags & HYDRO_FLAG_COMM_SELF)) {
           int r = comm_create(&h->comm, cfg, h->L, remote, h->slot_of_dom, h->doms.empty() ? nullptr : nullptr,
                               h->stream, &h->err);
           if (r) return r;
           std::vector<const DomView *> v0, v1;
           for (LocalDom &D : h->doms) {
             v0.push_back(&D.view[0]);
             v1.push_back(&D.view[1]);
           }
           r = comm_bind_views(h->comm, v0.data(), v1.data(), (int)h->doms.size(), &h->err);
           if (r) return r;
         }
         // initial state
         for (LocalDom &D : h->doms) launch_init_nodes(D.view[0], cfg->origin, cfg->extent, h->stream);
         if (cfg->init_kind != HYDRO_INIT_SEDOV) {
           int r = upload_state(h, 0, cfg->user, cfg->user[7], cfg->user[6],
                                cfg->init_kind == HYDRO_INIT_USER_MASS);
           if (r) return r;
         }
         for (LocalDom &D : h->doms) {
           if (h->strict)
             launch_strict_init_zones(D.view[0], cfg->init_kind, cfg->rho0, cfg->e0,
                                      cfg->sedov_energy, h->stream);
           else
             launch_init_zones(D.view[0], cfg->init_kind, cfg->rho0, cfg->e0, cfg->sedov_energy,
                               h->stream);
         }
         for (LocalDom &D : h->doms) launch_nodal_mass(D.view[0], h->stream);
         launch_strains(h, 0, 1, h->stream);
         for (LocalDom &D : h->doms) {
           if (h->strict) {  // dt^0, then the other parity := this one (node kernel, dt = 0)
             launch_strict_dt0(D.view[0], h->ph, h->st, h->mono, h->stream);
             launch_strict_node(D.view[0], h->ph, h->st, h->stream);
           } else {
             launch_dt0(D.view[0], h->ph, h->st, h->mono, h->stream);
           }
         }
         if (h->comm) {
           int r = comm_dt_min(h->comm, h->st, h->stream);
           if (r) return set_err(h, r, "dt allreduce failed");
         }
         if (!h->peer)  // peer transport: dt^0 is reduced over the ranks at hydro_peer_import
           launch_finalize_init(h->st, cfg->dt_first, cfg->dt_init, cfg->dt_max, cfg->t_stop,
                                cfg->t0, cfg->dt_floor, h->stream);
         CK(cudaGetLastError());
         CK(cudaStreamSynchronize(h->stream));
         return HYDRO_OK;
       }()) != HYDRO_OK)
    return fail(rc);
  hydro_info info;
  int st = read_info(h, &info, h->stream);
  if (st == HYDRO_ETANGLED) {
    set_err(h, st, "initial mesh has a zone with volume <= 0");
    return fail(st);
  }
  if (!h->peer && h->use_graph && (rc = build_graphs(h)) != HYDRO_OK) return fail(rc);
  *out = h;
  return HYDRO_OK;
}

int hydro_peer_export(hydro_ctx *h, void *buf, size_t *len) {
  if (!h || !len) return set_err(h, HYDRO_EINVAL, "NULL argument");
  if (!h->peer) return set_err(h, HYDRO_EINVAL, "context not created with HYDRO_FLAG_PEER");
  CK(cudaSetDevice(h->device));
  std::vector<int32_t> doms;
  std::vector<void *> bases;
  for (LocalDom &D : h->doms) {
    doms.push_back(D.dom);
    bases.push_back(D.mem);
  }
  return peer_export(h->peer, doms, bases, buf, len, &h->err);
}

int hydro_peer_import(hydro_ctx *h, const void *all, size_t len_per_rank) {
  if (!h || !all) return set_err(h, HYDRO_EINVAL, "NULL argument");
  if (!h->peer) return set_err(h, HYDRO_EINVAL, "context not created with HYDRO_FLAG_PEER");
  CK(cudaSetDevice(h->device));
  int rc = peer_import(h->peer, h->L, h->slot_of_dom, h->split, all, len_per_rank, &h->err);
  if (rc) return rc;
  if (h->fused_halo) {  // the inter-rank slabs join the node/energy stage's epilogue stores
    peer_push_targets(h->peer, &h->push_targets);
    if ((rc = build_push_tables(h)) != HYDRO_OK) return rc;
  }
  // dt^0 over all ranks (no halo: every rank initialised its ghosts from the global definition)
  rc = peer_exchange(h->peer, h->views_dev[0], 0, false, h->st, h->stream);
  if (rc) return set_err(h, rc, "peer dt^0 exchange failed");
  launch_finalize_init(h->st, h->cfg.dt_first, h->cfg.dt_init, h->cfg.dt_max, h->cfg.t_stop,
                       h->cfg.t0, h->cfg.dt_floor, h->stream);
  CK(cudaGetLastError());
  CK(cudaStreamSynchronize(h->stream));
  if (h->use_graph && (rc = build_graphs(h)) != HYDRO_OK) return rc;
  return HYDRO_OK;
}

int hydro_step(hydro_ctx *h, int32_t ncycles, void *cuda_stream, hydro_info *info) {
  NvtxRange nvtx_("hydro_step");
  if (!h || ncycles < 0) return set_err(h, HYDRO_EINVAL, "bad argument");
  if (h->failed) return set_err(h, HYDRO_ESTATE, "context failed earlier");
  if (h->peer && !peer_ready(h->peer))
    return set_err(h, HYDRO_ESTATE, "peer transport: hydro_peer_import not called yet");
  CK(cudaSetDevice(h->device));
  cudaStream_t s = cuda_stream ? (cudaStream_t)cuda_stream : h->stream;
  // Early stop (one rank only: every rank must launch the same cycles, whose collectives pair
  // up): once the run halted or reached t_stop, the remaining cycles are no-ops on the device
  // (that still copy the state between parities), so stop launching them.  Every 64 cycles the
  // (halted, done) words are copied to a ring of pinned host slots behind events; completed
  // slots are polled without blocking, and the host is never more than NFLAG x 64 cycles ahead
  // of the last confirmed check (it waits on the oldest slot when the ring is full), so at
  // most ~NFLAG x 64 no-op cycles run past the end.
  const bool early = h->cfg.nranks <= 1;
  constexpr int NF = hydro_ctx::NFLAG;
  if (early && !h->flag_host) {
    CK(cudaHostAlloc(&h->flag_host, 2 * NF * sizeof(unsigned int), cudaHostAllocDefault));
    for (int k = 0; k < NF; ++k)
      CK(cudaEventCreateWithFlags(&h->flag_ev[k], cudaEventDisableTiming));
  }
  int oldest = 0, npend = 0;
  int32_t next_check = 64;
  bool stop = false;
  auto pop_done = [&](bool block) -> cudaError_t {  // true in `stop` when a slot shows the end
    while (npend > 0) {
      cudaError_t q = block ? cudaEventSynchronize(h->flag_ev[oldest])
                            : cudaEventQuery(h->flag_ev[oldest]);
      if (q == cudaErrorNotReady) return cudaSuccess;
      if (q != cudaSuccess) return q;
      if ((h->flag_host[2 * oldest] | h->flag_host[2 * oldest + 1]) != 0u) stop = true;
      oldest = (oldest + 1) % NF;
      --npend;
      block = false;
      if (stop) return cudaSuccess;
    }
    return cudaSuccess;
  };
  for (int32_t c = 0; c < ncycles;) {
    if (early && c >= next_check) {
      next_check = c + 64;
      CK(pop_done(false));
      if (!stop && npend == NF) CK(pop_done(true));
      if (stop) break;
      const int slot = (oldest + npend) % NF;
      CK(cudaMemcpyAsync(&h->flag_host[2 * slot], &h->st->halted, 2 * sizeof(unsigned int),
                         cudaMemcpyDeviceToHost, s));
      CK(cudaEventRecord(h->flag_ev[slot], s));
      ++npend;
    }
    if (h->use_graph && h->graph_k > 1 && ncycles - c >= h->graph_k) {
      CK(cudaGraphLaunch(h->graphk[h->parity], s));
      h->parity ^= h->graph_k & 1;
      c += h->graph_k;
      continue;
    }
    if (h->use_graph) {
      CK(cudaGraphLaunch(h->graph[h->parity], s));
    } else {
      int rc = enqueue_cycle(h, h->parity, s);
      if (rc) return rc;
    }
    h->parity ^= 1;
    ++c;
  }
  const int status = read_info(h, info, s);
  if (status < 0 && status != HYDRO_ECUDA) h->failed = status;
  return status;
}

int hydro_get_info(hydro_ctx *h, hydro_info *info) {
  if (!h) return HYDRO_EINVAL;
  CK(cudaSetDevice(h->device));
  read_info(h, info, h->stream);
  return HYDRO_OK;
}

namespace {
// Storage sizes of a domain's migration buffer: 6 node arrays + e + m (hydro_domain_bytes).
void domain_counts(const DomainBox &b, int64_t *nnode, int64_t *nzone) {
  *nnode = (b.n[0] + 3 + 3) / 4 * 4 * (b.n[1] + 3) * (b.n[2] + 3);
  *nzone = (b.n[0] + 2 + 3) / 4 * 4 * (b.n[1] + 2) * (b.n[2] + 2);
}
}  // namespace

int hydro_domain_bytes(const hydro_ctx *h, int32_t dom, size_t *len) {
  if (!h || !len || dom < 0 || dom >= (int32_t)h->L.dom.size()) return HYDRO_EINVAL;
  int64_t nn, nz;
  domain_counts(h->L.dom[dom], &nn, &nz);
  *len = (size_t)(6 * nn + 2 * nz) * sizeof(double);
  return HYDRO_OK;
}

int hydro_domain_pack(hydro_ctx *h, int32_t dom, void *dev_buf, size_t len, void *stream) {
  NvtxRange nvtx_("hydro_domain_pack");
  size_t need = 0;
  if (hydro_domain_bytes(h, dom, &need) || !dev_buf || len < need ||
      h->slot_of_dom[dom] < 0)
    return set_err(h, HYDRO_EINVAL, "domain_pack: bad domain, buffer or length");
  CK(cudaSetDevice(h->device));
  cudaStream_t s = stream ? (cudaStream_t)stream : h->stream;
  const LocalDom &D = h->doms[h->slot_of_dom[dom]];
  const DomView &v = D.view[h->parity];
  int64_t nn, nz;
  domain_counts(D.box, &nn, &nz);
  const size_t nb = align_up(nn * sizeof(double), 256);
  char *dst = (char *)dev_buf;
  // the six current node arrays are consecutive allocations of pitch nb (carve_views)
  CK(cudaMemcpy2DAsync(dst, nn * sizeof(double), v.x, nb, nn * sizeof(double), 6,
                       cudaMemcpyDefault, s));
  dst += 6 * nn * sizeof(double);
  CK(cudaMemcpyAsync(dst, v.e, nz * sizeof(double), cudaMemcpyDefault, s));
  dst += nz * sizeof(double);
  CK(cudaMemcpyAsync(dst, v.m, nz * sizeof(double), cudaMemcpyDefault, s));
  CK(cudaStreamSynchronize(s));
  return HYDRO_OK;
}

int hydro_domain_unpack(hydro_ctx *h, int32_t dom, const void *dev_buf, size_t len,
                        void *stream) {
  NvtxRange nvtx_("hydro_domain_unpack");
  size_t need = 0;
  if (hydro_domain_bytes(h, dom, &need) || !dev_buf || len < need ||
      h->slot_of_dom[dom] < 0)
    return set_err(h, HYDRO_EINVAL, "domain_unpack: bad domain, buffer or length");
  CK(cudaSetDevice(h->device));
  cudaStream_t s = stream ? (cudaStream_t)stream : h->stream;
  const LocalDom &D = h->doms[h->slot_of_dom[dom]];
  const DomView &v = D.view[h->parity];
  int64_t nn, nz;
  domain_counts(D.box, &nn, &nz);
  const size_t nb = align_up(nn * sizeof(double), 256);
  const char *src = (const char *)dev_buf;
  CK(cudaMemcpy2DAsync(const_cast<double *>(v.x), nb, src, nn * sizeof(double), nn * sizeof(double), 6,
                       cudaMemcpyDefault, s));
  src += 6 * nn * sizeof(double);
  CK(cudaMemcpyAsync(const_cast<double *>(v.e), src, nz * sizeof(double), cudaMemcpyDefault, s));
  src += nz * sizeof(double);
  CK(cudaMemcpyAsync(const_cast<double *>(v.m), src, nz * sizeof(double), cudaMemcpyDefault, s));
  launch_nodal_mass(D.view[0], s);  // 1/m and 8 / sum m from the imported masses
  CK(cudaGetLastError());
  CK(cudaStreamSynchronize(s));
  return HYDRO_OK;
}

int hydro_set_clock(hydro_ctx *h, double t, double dt, int64_t cycle) {
  if (!h || !(dt > 0.0) || !std::isfinite(t) || cycle < 0)
    return set_err(h, HYDRO_EINVAL, "set_clock: bad argument");
  CK(cudaSetDevice(h->device));
  DevState s0;
  CK(cudaMemcpyAsync(&s0, h->st, sizeof(s0), cudaMemcpyDeviceToHost, h->stream));
  CK(cudaStreamSynchronize(h->stream));
  s0.t = t;
  s0.dt = dt;
  s0.cycle = (unsigned long long)cycle;
  s0.err = 0;
  s0.halted = 0;
  s0.done = (h->ph.t_stop > 0.0 && t >= h->ph.t_stop) ? 1u : 0u;
  s0.bad_zone = ~0ull;
  CK(cudaMemcpyAsync(h->st, &s0, sizeof(s0), cudaMemcpyHostToDevice, h->stream));
  CK(cudaStreamSynchronize(h->stream));
  h->failed = 0;
  return HYDRO_OK;
}

int hydro_get_box(hydro_ctx *h, const int64_t lo[3], const int64_t hi[3], uint32_t mask,
                  double *const *out) {
  NvtxRange nvtx_("hydro_get_box");
  if (!h || !lo || !hi || !out) return set_err(h, HYDRO_EINVAL, "NULL argument");
  for (int a = 0; a < 3; ++a)
    if (lo[a] < 0 || hi[a] > h->L.N[a] || hi[a] <= lo[a])
      return set_err(h, HYDRO_EINVAL, "box out of range");
  for (int f = 0; f < HYDRO_NFIELDS; ++f)
    if ((mask >> f & 1u) && !out[f]) return set_err(h, HYDRO_EINVAL, "missing output array");
  CK(cudaSetDevice(h->device));
  const int par = h->parity;
  const bool derived = (mask & (HYDRO_F_RHO | HYDRO_F_P | HYDRO_F_Q | HYDRO_F_C | HYDRO_F_VOL)) != 0;
  if (derived)
    launch_strains(h, par, 1, h->stream);
    for (LocalDom &D : h->doms) {
      if (h->strict) launch_strict_derive(D.view[par], h->ph, h->mono, h->stream);
      else launch_derive(D.view[par], h->ph, h->mono, h->stream);
    }
  const int64_t bn[3] = {hi[0] - lo[0] + 1, hi[1] - lo[1] + 1, hi[2] - lo[2] + 1};
  const int64_t bz[3] = {hi[0] - lo[0], hi[1] - lo[1], hi[2] - lo[2]};
  for (LocalDom &D : h->doms) {
    const DomView &v = D.view[par];
    // nodes written by this domain: lowest-index owner rule per axis
    int64_t nlo[3], next[3], zlo[3], zext[3];
    bool any_n = true, any_z = true;
    for (int a = 0; a < 3; ++a) {
      const int64_t own_lo = D.box.lo[a] + (D.box.idx[a] > 0 ? 1 : 0);
      const int64_t own_hi = D.box.lo[a] + D.box.n[a];  // inclusive
      nlo[a] = std::max(own_lo, lo[a]);
      next[a] = std::min(own_hi, hi[a]) - nlo[a] + 1;
      if (next[a] <= 0) any_n = false;
      zlo[a] = std::max(D.box.lo[a], lo[a]);
      zext[a] = std::min(D.box.lo[a] + D.box.n[a], hi[a]) - zlo[a];
      if (zext[a] <= 0) any_z = false;
    }
    if (any_n) {
      const double *src[6] = {v.x, v.y, v.z, v.u, v.v, v.w};
      int64_t hl[3], dl[3];
      for (int a = 0; a < 3; ++a) {
        hl[a] = nlo[a] - lo[a];
        dl[a] = nlo[a] - D.box.lo[a] + 1;
      }
      for (int f = 0; f < 6; ++f) {
        if (!(mask >> f & 1u)) continue;
        int rc = copy_box(h, false, out[f], bn, hl, next, const_cast<double *>(src[f]), v.nsx,
                          v.nsxy / v.nsx, dl, h->stream);
        if (rc) return rc;
      }
    }
    if (any_z) {
      int64_t hl[3], dl[3];
      for (int a = 0; a < 3; ++a) {
        hl[a] = zlo[a] - lo[a];
        dl[a] = zlo[a] - D.box.lo[a] + 1;
      }
      const double *src[HYDRO_NFIELDS] = {};
      src[6] = v.aux + 0 * v.nzone;
      src[7] = v.e;
      src[8] = v.aux + 1 * v.nzone;
      src[9] = v.aux + 2 * v.nzone;
      src[10] = v.aux + 3 * v.nzone;
      src[11] = v.aux + 4 * v.nzone;
      src[12] = v.m;
      for (int f = 6; f < HYDRO_NFIELDS; ++f) {
        if (!(mask >> f & 1u)) continue;
        int rc = copy_box(h, false, out[f], bz, hl, zext, const_cast<double *>(src[f]), v.zsx,
                          v.zsxy / v.zsx, dl, h->stream);
        if (rc) return rc;
      }
    }
  }
  CK(cudaStreamSynchronize(h->stream));
  return HYDRO_OK;
}

int hydro_get_fields(hydro_ctx *h, uint32_t mask, double *const *out) {
  NvtxRange nvtx_("hydro_get_fields");
  if (!h) return set_err(h, HYDRO_EINVAL, "NULL context");
  const int64_t lo[3] = {0, 0, 0};
  const int64_t hi[3] = {h->L.N[0], h->L.N[1], h->L.N[2]};
  return hydro_get_box(h, lo, hi, mask, out);
}

int hydro_set_state(hydro_ctx *h, const double *const *nodes6, const double *e, double t,
                    double dt) {
  NvtxRange nvtx_("hydro_set_state");
  if (!h || !nodes6 || !e || !(dt > 0.0)) return set_err(h, HYDRO_EINVAL, "bad argument");
  for (int f = 0; f < 6; ++f)
    if (!nodes6[f]) return set_err(h, HYDRO_EINVAL, "missing node array");
  CK(cudaSetDevice(h->device));
  int rc = upload_state(h, h->parity, nodes6, e, nullptr, false);
  if (rc) return rc;
  DevState s0;
  CK(cudaMemcpyAsync(&s0, h->st, sizeof(s0), cudaMemcpyDeviceToHost, h->stream));
  CK(cudaStreamSynchronize(h->stream));
  s0.t = t;
  // the t_stop clamp of S9 (as at creation): a run started before t_stop ends on it exactly
  s0.dt = (h->ph.t_stop > 0.0 && t < h->ph.t_stop) ? std::min(dt, h->ph.t_stop - t) : dt;
  s0.err = 0;
  s0.halted = 0;
  s0.done = (h->ph.t_stop > 0.0 && t >= h->ph.t_stop) ? 1u : 0u;
  s0.bad_zone = ~0ull;
  s0.dtz_acc = (unsigned long long)0x7ff0000000000000ull;
  CK(cudaMemcpyAsync(h->st, &s0, sizeof(s0), cudaMemcpyHostToDevice, h->stream));
  CK(cudaStreamSynchronize(h->stream));
  h->failed = 0;
  return HYDRO_OK;
}

namespace {
// Dense global staging <-> the local domains of parity par, on stream s (hydro_run_batch).
// Scatter: owned + ghost entries, as upload_state; gather: the lowest-index owner of each node
// and every owned zone, as hydro_get_box.  Field f of the dense block: nodes f*NnG, e at 6*NnG.
void batch_scatter(hydro_ctx *h, const double *dense, int par, cudaStream_t s) {
  const int64_t gn[3] = {h->L.N[0] + 1, h->L.N[1] + 1, h->L.N[2] + 1};
  const int64_t gz[3] = {h->L.N[0], h->L.N[1], h->L.N[2]};
  const int64_t NnG = gn[0] * gn[1] * gn[2];
  for (LocalDom &D : h->doms) {
    const DomView &v = D.view[par];
    int64_t nlo[3], next[3], nloc[3], zlo[3], zext[3], zloc[3];
    for (int a = 0; a < 3; ++a) {
      const int64_t lo = std::max<int64_t>(D.box.lo[a] - 1, 0);
      const int64_t hi = std::min<int64_t>(D.box.lo[a] + D.box.n[a] + 1, h->L.N[a]);
      nlo[a] = lo; next[a] = hi - lo + 1; nloc[a] = lo - D.box.lo[a] + 1;
      zlo[a] = lo; zext[a] = hi - lo; zloc[a] = nloc[a];
    }
    double *dst[7] = {const_cast<double *>(v.x), const_cast<double *>(v.y),
                      const_cast<double *>(v.z), const_cast<double *>(v.u),
                      const_cast<double *>(v.v), const_cast<double *>(v.w),
                      const_cast<double *>(v.e)};
    for (int f = 0; f < 7; ++f) {
      const bool z = f == 6;
      const int64_t *g = z ? gz : gn, *lo = z ? zlo : nlo, *ex = z ? zext : next,
                    *lc = z ? zloc : nloc;
      const int64_t dsx = z ? v.zsx : v.nsx, dsxy = z ? v.zsxy : v.nsxy;
      const double *src = dense + f * NnG + (lo[2] * g[1] + lo[1]) * g[0] + lo[0];
      launch_copy3d(src, g[0], g[0] * g[1], dst[f] + (lc[2] * (dsxy / dsx) + lc[1]) * dsx + lc[0],
                    dsx, dsxy, (int)ex[0], (int)ex[1], (int)ex[2], s);
    }
  }
}
void batch_gather(hydro_ctx *h, double *dense, int par, cudaStream_t s) {
  const int64_t gn[3] = {h->L.N[0] + 1, h->L.N[1] + 1, h->L.N[2] + 1};
  const int64_t gz[3] = {h->L.N[0], h->L.N[1], h->L.N[2]};
  const int64_t NnG = gn[0] * gn[1] * gn[2];
  for (LocalDom &D : h->doms) {
    const DomView &v = D.view[par];
    int64_t nlo[3], next[3], zlo[3], zext[3];
    for (int a = 0; a < 3; ++a) {
      nlo[a] = D.box.lo[a] + (D.box.idx[a] > 0 ? 1 : 0);
      next[a] = D.box.lo[a] + D.box.n[a] - nlo[a] + 1;
      zlo[a] = D.box.lo[a];
      zext[a] = D.box.n[a];
    }
    const double *src[7] = {v.x, v.y, v.z, v.u, v.v, v.w, v.e};
    for (int f = 0; f < 7; ++f) {
      const bool z = f == 6;
      const int64_t *g = z ? gz : gn, *lo = z ? zlo : nlo, *ex = z ? zext : next;
      const int64_t dsx = z ? v.zsx : v.nsx, dsxy = z ? v.zsxy : v.nsxy;
      int64_t lc[3];
      for (int a = 0; a < 3; ++a) lc[a] = lo[a] - D.box.lo[a] + 1;
      launch_copy3d(src[f] + (lc[2] * (dsxy / dsx) + lc[1]) * dsx + lc[0], dsx, dsxy,
                    dense + f * NnG + (lo[2] * g[1] + lo[1]) * g[0] + lo[0], g[0], g[0] * g[1],
                    (int)ex[0], (int)ex[1], (int)ex[2], s);
    }
  }
}
}  // namespace

int hydro_run_batch(hydro_ctx *h, int32_t nbatch, int32_t ncycles, const double *const *in,
                    double *const *out, const double *t0, const double *dt0, hydro_info *info) {
  NvtxRange nvtx_("hydro_run_batch");
  if (!h || nbatch < 0 || ncycles < 0 || (nbatch > 0 && (!in || !out || !t0 || !dt0)))
    return set_err(h, HYDRO_EINVAL, "run_batch: bad argument");
  if (h->cfg.nranks > 1 || h->peer || h->comm)
    return set_err(h, HYDRO_EINVAL, "run_batch: single-rank contexts only");
  for (int32_t b = 0; b < nbatch; ++b) {
    if (!(dt0[b] > 0.0) || !std::isfinite(t0[b]))
      return set_err(h, HYDRO_EINVAL, "run_batch: bad t0/dt0");
    for (int f = 0; f < 7; ++f)
      if (!in[7 * b + f] || !out[7 * b + f])
        return set_err(h, HYDRO_EINVAL, "run_batch: missing array");
  }
  if (nbatch == 0) return HYDRO_OK;
  CK(cudaSetDevice(h->device));
  const int64_t NnG = (h->L.N[0] + 1) * (h->L.N[1] + 1) * (h->L.N[2] + 1);
  const int64_t NzG = h->L.N[0] * h->L.N[1] * h->L.N[2];
  const size_t nbytes = (size_t)NnG * sizeof(double), zbytes = (size_t)NzG * sizeof(double);
  if (!h->cp_in) {
    CK(cudaStreamCreateWithFlags(&h->cp_in, cudaStreamNonBlocking));
    CK(cudaStreamCreateWithFlags(&h->cp_out, cudaStreamNonBlocking));
    for (int i = 0; i < 2; ++i) {
      CK(cudaMalloc(&h->bin[i], 6 * nbytes + zbytes));
      CK(cudaMalloc(&h->bout[i], 6 * nbytes + zbytes));
      for (cudaEvent_t *e : {&h->in_ready[i], &h->in_free[i], &h->out_ready[i], &h->out_free[i]})
        CK(cudaEventCreateWithFlags(e, cudaEventDisableTiming));
    }
  }
  if (nbatch > h->bst_cap) {
    if (h->bst) CK(cudaFree(h->bst));
    CK(cudaMalloc(&h->bst, sizeof(DevState) * nbatch));
    h->bst_cap = nbatch;
  }
  cudaStream_t s = h->stream;
  // the copy streams start after everything already enqueued on the compute stream
  CK(cudaEventRecord(h->in_free[0], s));
  CK(cudaStreamWaitEvent(h->cp_in, h->in_free[0], 0));
  CK(cudaStreamWaitEvent(h->cp_out, h->in_free[0], 0));
  CK(cudaEventRecord(h->in_free[0], h->cp_in));
  CK(cudaEventRecord(h->in_free[1], h->cp_in));
  CK(cudaEventRecord(h->out_free[0], h->cp_out));
  CK(cudaEventRecord(h->out_free[1], h->cp_out));
  auto h2d = [&](int32_t b) -> int {  // batch b's inputs into staging slot b & 1 (copy-in stream)
    const int k = b & 1;
    CK(cudaStreamWaitEvent(h->cp_in, h->in_free[k], 0));
    for (int f = 0; f < 7; ++f)
      CK(cudaMemcpyAsync(h->bin[k] + f * NnG, in[7 * b + f], f < 6 ? nbytes : zbytes,
                         cudaMemcpyHostToDevice, h->cp_in));
    CK(cudaEventRecord(h->in_ready[k], h->cp_in));
    return HYDRO_OK;
  };
  int rc = h2d(0);
  if (rc) return rc;
  for (int32_t b = 0; b < nbatch; ++b) {
    const int k = b & 1;
    // the copy-in of batch b+1 overlaps batch b's cycles
    if (b + 1 < nbatch && (rc = h2d(b + 1))) return rc;
    CK(cudaStreamWaitEvent(s, h->in_ready[k], 0));
    batch_scatter(h, h->bin[k], h->parity, s);
    CK(cudaEventRecord(h->in_free[k], s));
    const unsigned done = (h->ph.t_stop > 0.0 && t0[b] >= h->ph.t_stop) ? 1u : 0u;
    const double dtb = (h->ph.t_stop > 0.0 && t0[b] < h->ph.t_stop)
                           ? std::min(dt0[b], h->ph.t_stop - t0[b]) : dt0[b];  // as set_state
    launch_reset_clock(h->st, t0[b], dtb, done, s);
    for (int32_t c = 0; c < ncycles;) {
      if (h->use_graph && h->graph_k > 1 && ncycles - c >= h->graph_k) {
        CK(cudaGraphLaunch(h->graphk[h->parity], s));
        h->parity ^= h->graph_k & 1;
        c += h->graph_k;
        continue;
      }
      if (h->use_graph) {
        CK(cudaGraphLaunch(h->graph[h->parity], s));
      } else if ((rc = enqueue_cycle(h, h->parity, s))) {
        return rc;
      }
      h->parity ^= 1;
      ++c;
    }
    CK(cudaMemcpyAsync(h->bst + b, h->st, sizeof(DevState), cudaMemcpyDeviceToDevice, s));
    // results into staging slot k once its previous copy-out is done; the copy-out of batch b
    // overlaps batch b+1's cycles
    CK(cudaStreamWaitEvent(s, h->out_free[k], 0));
    batch_gather(h, h->bout[k], h->parity, s);
    CK(cudaEventRecord(h->out_ready[k], s));
    CK(cudaStreamWaitEvent(h->cp_out, h->out_ready[k], 0));
    for (int f = 0; f < 7; ++f)
      CK(cudaMemcpyAsync(out[7 * b + f], h->bout[k] + f * NnG, f < 6 ? nbytes : zbytes,
                         cudaMemcpyDeviceToHost, h->cp_out));
    CK(cudaEventRecord(h->out_free[k], h->cp_out));
  }
  CK(cudaStreamSynchronize(h->cp_out));
  CK(cudaStreamSynchronize(s));
  std::vector<DevState> fin(nbatch);
  CK(cudaMemcpy(fin.data(), h->bst, sizeof(DevState) * nbatch, cudaMemcpyDeviceToHost));
  int status = HYDRO_OK;
  for (int32_t b = 0; b < nbatch; ++b) {
    int sb = HYDRO_OK;
    if (fin[b].halted & ERR_TANGLED) sb = HYDRO_ETANGLED;
    else if (fin[b].halted & ERR_NONFINITE) sb = HYDRO_ENONFINITE;
    if (info) {
      info[b].t = fin[b].t;
      info[b].dt = fin[b].dt;
      info[b].cycle = (int64_t)fin[b].cycle;
      info[b].dt_min_zone = fin[b].dtz_last;
      info[b].status = sb;
      info[b].bad_zone = (fin[b].bad_zone == ~0ull) ? -1 : (int64_t)fin[b].bad_zone;
    }
    if (status == HYDRO_OK) status = sb;
  }
  // the context continues from the last batch's state (its clock is on the device already)
  h->failed = 0;
  return status;
}

int hydro_kernels_per_cycle(const hydro_ctx *h) {
  if (!h) return HYDRO_EINVAL;
  const int nd = (int)h->doms.size();
  int k = h->group ? 1 + (group_node() ? 1 : nd)
                   : (h->split ? 3 : (h->one_kernel ? 1 : 2)) * nd;  // cycle kernels
  if (h->halo_overlap == 3) {  // one copy per node-stage stream
    for (int s = 0; s < h->nstreams; ++s) {
      bool any = false;
      for (size_t j = 0; j < h->halo_count.size(); ++j)
        any |= h->node_stream[j] == s && h->halo_count[j] > 0;
      k += any;
    }
  } else if (h->halo_overlap) {  // one copy per source domain
    for (int32_t c : h->halo_count) k += c > 0;
  } else if (h->n_local_pairs > 0 && !h->fused_halo) {
    k += 1;  // intra-GPU halo copy
  }
  if (h->n_pcopy) k += 1;           // P of skipped zone-stage rings
  if (!fold_finalize(h)) k += 1;     // finalize
  if (h->comm) k += comm_kernels_per_cycle(h->comm);
  if (h->peer) k += peer_kernels_per_cycle(h->peer, !h->fused_halo);
  return k;
}

int hydro_time_kernels(hydro_ctx *h, int32_t ncycles, double out_ms[6]) {
  NvtxRange nvtx_("hydro_time_kernels");
  if (!h || ncycles <= 0 || !out_ms) return set_err(h, HYDRO_EINVAL, "bad argument");
  if (h->failed) return set_err(h, HYDRO_ESTATE, "context failed earlier");
  if (h->peer && !peer_ready(h->peer))
    return set_err(h, HYDRO_ESTATE, "peer transport: hydro_peer_import not called yet");
  CK(cudaSetDevice(h->device));
  cudaStream_t s = h->stream;
  cudaEvent_t ev[5];
  for (int i = 0; i < 5; ++i) CK(cudaEventCreate(&ev[i]));
  double acc[6] = {0, 0, 0, 0, 0, 0};
  for (int32_t c = 0; c < ncycles; ++c) {
    const int par = h->parity;
    CK(cudaEventRecord(ev[0], s));
    CK(cudaEventRecord(ev[4], s));
    if (h->split) {
      int rc = enqueue_split(h, par, s);
      if (rc) return rc;
    } else if (h->one_kernel) {
      for (LocalDom &D : h->doms) launch_cycle_fused(D.view[par], D.maps[par], h->ph, h->st, fold_finalize(h), s);
      if (h->comm && comm_dt_min(h->comm, h->st, s)) return HYDRO_ENCCL;
    } else {
      launch_zone_stages(h, par, s);
      if (h->comm && comm_dt_min(h->comm, h->st, s)) return HYDRO_ENCCL;
      CK(cudaEventRecord(ev[4], s));
      launch_node_stages(h, par, s);
    }
    CK(cudaEventRecord(ev[1], s));
    if (!h->fused_halo)
      launch_halo_copy(h->views_dev[par], h->local_pairs_dev, h->n_local_pairs, s);
    if (h->comm && comm_halo(h->comm, par, s)) return HYDRO_ENCCL;
    if (h->peer && peer_exchange(h->peer, h->views_dev[par], par, !h->fused_halo, h->st, s))
      return HYDRO_ECUDA;
    CK(cudaEventRecord(ev[2], s));
    if (!fold_finalize(h)) launch_finalize(h->st, h->ph, s);
    CK(cudaEventRecord(ev[3], s));
    CK(cudaEventSynchronize(ev[3]));
    float a, b, cc, d;
    CK(cudaEventElapsedTime(&a, ev[0], ev[1]));
    CK(cudaEventElapsedTime(&b, ev[1], ev[2]));
    CK(cudaEventElapsedTime(&cc, ev[2], ev[3]));
    CK(cudaEventElapsedTime(&d, ev[0], ev[3]));
    acc[0] += a; acc[1] += b; acc[2] += cc; acc[3] += d;
    if (!h->split && !h->one_kernel) {
      float z, n;
      CK(cudaEventElapsedTime(&z, ev[0], ev[4]));
      CK(cudaEventElapsedTime(&n, ev[4], ev[1]));
      acc[4] += z;
      acc[5] += n;
    }
    h->parity ^= 1;
  }
  for (int i = 0; i < 5; ++i) cudaEventDestroy(ev[i]);
  const double nd = h->doms.empty() ? 1.0 : (double)h->doms.size();
  out_ms[0] = acc[0] / ncycles / nd;
  out_ms[1] = acc[1] / ncycles;
  out_ms[2] = acc[2] / ncycles;
  out_ms[3] = acc[3] / ncycles;
  out_ms[4] = acc[4] / ncycles / nd;
  out_ms[5] = acc[5] / ncycles / nd;
  hydro_info info;
  const int status = read_info(h, &info, s);
  if (status < 0 && status != HYDRO_ECUDA) h->failed = status;
  return status;
}

int hydro_peer_detach(hydro_ctx *h) {
  if (!h) return HYDRO_OK;
  if (!h->peer) return HYDRO_OK;
  CK(cudaSetDevice(h->device));
  CK(cudaStreamSynchronize(h->stream));
  CK(cudaDeviceSynchronize());  // no cycle of this rank still stores into a peer
  peer_detach(h->peer);
  return HYDRO_OK;
}

int hydro_destroy(hydro_ctx *h) {
  if (!h) return HYDRO_OK;
  cudaSetDevice(h->device);
  if (h->stream) cudaStreamSynchronize(h->stream);
  for (int k = 0; k < hydro_ctx::NFLAG; ++k)
    if (h->flag_ev[k]) cudaEventDestroy(h->flag_ev[k]);
  if (h->flag_host) cudaFreeHost(h->flag_host);
  if (h->pcopy_dev) cudaFree(h->pcopy_dev);
  for (void *p : h->mono_mem) cudaFree(p);
  for (int p = 0; p < 2; ++p) {
    if (h->graph[p]) cudaGraphExecDestroy(h->graph[p]);
    if (h->graphk[p]) cudaGraphExecDestroy(h->graphk[p]);
    if (h->views_dev[p]) cudaFree(h->views_dev[p]);
    if (h->zmaps_dev[p]) cudaFree(h->zmaps_dev[p]);
    if (h->nmaps_dev[p]) cudaFree(h->nmaps_dev[p]);
    if (p == 0 && h->ntasks_dev) cudaFree(h->ntasks_dev);
    if (p == 0 && h->ztasks_dev) cudaFree(h->ztasks_dev);
  }
  if (h->comm) comm_destroy(h->comm);
  if (h->peer) peer_destroy(h->peer);
  for (LocalDom &D : h->doms)
    if (D.mem) cudaFree(D.mem);
  if (h->local_pairs_dev) cudaFree(h->local_pairs_dev);
  for (int p = 0; p < 2; ++p)
    if (h->push_dev[p]) cudaFree(h->push_dev[p]);
  if (h->stage) cudaFree(h->stage);
  if (h->st) cudaFree(h->st);
  for (cudaEvent_t e : h->node_done)
    if (e) cudaEventDestroy(e);
  if (h->halo_join) cudaEventDestroy(h->halo_join);
  if (h->halo_stream) cudaStreamDestroy(h->halo_stream);
  for (int i = 0; i < 2; ++i) {
    if (h->bin[i]) cudaFree(h->bin[i]);
    if (h->bout[i]) cudaFree(h->bout[i]);
    for (cudaEvent_t e : {h->in_ready[i], h->in_free[i], h->out_ready[i], h->out_free[i]})
      if (e) cudaEventDestroy(e);
  }
  if (h->bst) cudaFree(h->bst);
  if (h->cp_in) cudaStreamDestroy(h->cp_in);
  if (h->cp_out) cudaStreamDestroy(h->cp_out);
  if (h->stream) cudaStreamDestroy(h->stream);
  for (int k = 1; k < 4; ++k) {
    if (h->side[k]) cudaStreamDestroy(h->side[k]);
    if (h->join_ev[k]) cudaEventDestroy(h->join_ev[k]);
  }
  if (h->fork_ev) cudaEventDestroy(h->fork_ev);
  delete h;
  return HYDRO_OK;
}

}  // extern "C"
