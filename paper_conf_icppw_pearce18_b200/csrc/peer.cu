// peer.cu -- inter-rank halo exchange and dt reduction over peer memory (CUDA IPC), no NCCL.
//
// The paper exchanged halos through the host and named GPU-direct as future work (PAPER.md
// L513-520).  Here every rank maps its neighbours' domain allocations (cudaIpcOpenMemHandle; over
// NVLink/NVSwitch on a multi-GPU node, or the same device when several ranks share one GPU) and
// one kernel stores its boundary layer straight into the neighbours' ghost arrays: the pack, send,
// receive and unpack of a message-passing exchange collapse into peer stores issued right after
// the node/energy stage.  A one-block sync kernel then publishes this rank's dt_z minimum and
// error bits into every peer's mailbox, raises its flag for the exchange epoch, spins until every
// peer's flag for the epoch arrived, and reduces dt (min) and the error bits (or) locally -- the
// 8-byte allreduce-min of S9 without a collective library.  All of it is captured in the CUDA
// graph of a cycle.
#include "peer.h"

#include <cstring>

namespace hydro {

namespace {

struct PeerSlab {   // one inter-rank ghost slab pushed by this rank
  int32_t src_slot; // local source domain slot
  int32_t dst_view; // index into the remote-view table
  int64_t nlo[3], nhi[3], zlo[3], zhi[3];
};

// Mailbox layout (uint64 words): [0, R) epoch flags written by rank r; then per epoch parity
// (e & 1) R dt-bit slots and R error-bit slots.  Two parities are needed: a fast peer that has
// seen this rank's flag for epoch e may already publish its epoch e+1 values before this rank
// read epoch e's, but it cannot reach e+2 before this rank raised its own flag for e+1.
__global__ void k_peer_push(const DomView *local, const DomView *remote, const PeerSlab *slabs) {
  const PeerSlab p = slabs[blockIdx.y];
  const DomView &S = local[p.src_slot];
  const DomView &D = remote[p.dst_view];
  const int64_t nx = p.nhi[0] - p.nlo[0], ny = p.nhi[1] - p.nlo[1], nz = p.nhi[2] - p.nlo[2];
  const int64_t nn = nx * ny * nz;
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < nn;
       t += (int64_t)gridDim.x * blockDim.x) {
    const int64_t a = t % nx, b = (t / nx) % ny, c = t / (nx * ny);
    const int64_t gx = p.nlo[0] + a, gy = p.nlo[1] + b, gz = p.nlo[2] + c;
    const int64_t si = S.nid((int)(gx - S.lo[0]), (int)(gy - S.lo[1]), (int)(gz - S.lo[2]));
    const int64_t di = D.nid((int)(gx - D.lo[0]), (int)(gy - D.lo[1]), (int)(gz - D.lo[2]));
    // all six loads before the stores (sources are never written here: read-only path)
    const double v0 = __ldg(S.xn + si), v1 = __ldg(S.yn + si), v2 = __ldg(S.zn + si);
    const double v3 = __ldg(S.un + si), v4 = __ldg(S.vn + si), v5 = __ldg(S.wn + si);
    D.xn[di] = v0; D.yn[di] = v1; D.zn[di] = v2;
    D.un[di] = v3; D.vn[di] = v4; D.wn[di] = v5;
  }
  const int64_t zx = p.zhi[0] - p.zlo[0], zy = p.zhi[1] - p.zlo[1], zz = p.zhi[2] - p.zlo[2];
  const int64_t nzn = zx * zy * zz;
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < nzn;
       t += (int64_t)gridDim.x * blockDim.x) {
    const int64_t a = t % zx, b = (t / zx) % zy, c = t / (zx * zy);
    const int64_t gx = p.zlo[0] + a, gy = p.zlo[1] + b, gz = p.zlo[2] + c;
    D.en[D.zid((int)(gx - D.lo[0]), (int)(gy - D.lo[1]), (int)(gz - D.lo[2]))] =
        S.en[S.zid((int)(gx - S.lo[0]), (int)(gy - S.lo[1]), (int)(gz - S.lo[2]))];
  }
  __threadfence_system();  // peer stores visible before the sync kernel raises the flag
}

__device__ __forceinline__ unsigned long long ld_acquire_sys(const unsigned long long *p) {
  unsigned long long v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_sys(unsigned long long *p, unsigned long long v) {
  asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// One block of 32 threads, thread r serves rank r.
__global__ void k_peer_sync(DevState *st, unsigned long long *const *mbox, int rank, int nranks) {
  const int r = threadIdx.x;
  const unsigned long long epoch = st->xchg + 1;
  const unsigned long long mydt = st->dtz_acc, myerr = st->err;
  const int base = nranks + (int)(epoch & 1) * 2 * nranks;  // this epoch's dt / err slots
  __syncthreads();
  if (r < nranks) {
    unsigned long long *mb = mbox[r];  // rank r's mailbox (mapped)
    st_release_sys(mb + base + rank, mydt);
    st_release_sys(mb + base + nranks + rank, myerr);
    __threadfence_system();
    st_release_sys(mb + rank, epoch);
  }
  __syncthreads();
  unsigned long long *own = mbox[rank];
  if (r < nranks)
    while (ld_acquire_sys(own + r) < epoch) {
    }
  __syncthreads();
  if (r == 0) {
    unsigned long long dt = ld_acquire_sys(own + base), err = ld_acquire_sys(own + base + nranks);
    for (int q = 1; q < nranks; ++q) {
      const unsigned long long v = ld_acquire_sys(own + base + q);
      dt = v < dt ? v : dt;  // non-negative doubles order like their bit patterns
      err |= ld_acquire_sys(own + base + nranks + q);
    }
    st->dtz_acc = dt;
    st->err = (unsigned int)err;
    st->xchg = epoch;
  }
}

}  // namespace

struct Peer {
  int rank = 0, nranks = 1;
  unsigned long long *mailbox = nullptr;           // this rank's mailbox (device)
  unsigned long long **mbox_dev = nullptr;         // [nranks] mapped mailbox pointers (device)
  std::vector<void *> opened;                      // IPC-mapped bases to close
  DomView *remote_dev[2] = {nullptr, nullptr};     // remote destination views per parity
  PeerSlab *slabs_dev = nullptr;
  std::vector<PushTarget> targets;  // host copy of the slabs (fused halo tables)
  int nslabs = 0;
  int blocks = 1;
  bool ready = false;
};

int peer_create(Peer **out, const hydro_config *cfg, std::string *err) {
  Peer *p = new Peer();
  *out = p;
  p->rank = cfg->rank;
  p->nranks = cfg->nranks;
  if (p->nranks > 32) {
    *err = "peer transport supports up to 32 ranks";
    return HYDRO_EINVAL;
  }
  if (cudaMalloc(&p->mailbox, 5 * p->nranks * sizeof(unsigned long long)) != cudaSuccess ||
      cudaMemset(p->mailbox, 0, 5 * p->nranks * sizeof(unsigned long long)) != cudaSuccess) {
    *err = "peer mailbox allocation failed";
    return HYDRO_ENOMEM;
  }
  return HYDRO_OK;
}

size_t peer_export_size(int nlocal) { return sizeof(cudaIpcMemHandle_t) * (1 + nlocal) + 8 * (1 + nlocal); }

int peer_export(Peer *p, const std::vector<int32_t> &local_doms, const std::vector<void *> &bases,
                void *buf, size_t *len, std::string *err) {
  const size_t need = peer_export_size((int)local_doms.size());
  const size_t cap = *len;
  *len = need;
  if (!buf) return HYDRO_OK;
  if (cap < need) {
    *err = "peer export buffer too small";
    return HYDRO_EINVAL;
  }
  char *w = (char *)buf;
  const int64_t count = (int64_t)local_doms.size();
  std::memcpy(w, &count, 8);
  w += 8;
  cudaIpcMemHandle_t hm;
  if (cudaIpcGetMemHandle(&hm, p->mailbox) != cudaSuccess) {
    *err = "cudaIpcGetMemHandle(mailbox) failed";
    return HYDRO_ECUDA;
  }
  std::memcpy(w, &hm, sizeof(hm));
  w += sizeof(hm);
  for (size_t i = 0; i < local_doms.size(); ++i) {
    const int64_t dom = local_doms[i];
    std::memcpy(w, &dom, 8);
    w += 8;
    if (cudaIpcGetMemHandle(&hm, bases[i]) != cudaSuccess) {
      *err = "cudaIpcGetMemHandle(domain) failed";
      return HYDRO_ECUDA;
    }
    std::memcpy(w, &hm, sizeof(hm));
    w += sizeof(hm);
  }
  return HYDRO_OK;
}

int peer_import(Peer *p, const Layout &L, const std::vector<int32_t> &slot_of_dom, bool split,
                const void *all, size_t len_per_rank, std::string *err) {
  std::vector<unsigned long long *> mboxes(p->nranks, nullptr);
  std::vector<void *> dom_base(L.dom.size(), nullptr);
  for (int r = 0; r < p->nranks; ++r) {
    const char *w = (const char *)all + (size_t)r * len_per_rank;
    int64_t count;
    std::memcpy(&count, w, 8);
    w += 8;
    cudaIpcMemHandle_t hm;
    std::memcpy(&hm, w, sizeof(hm));
    w += sizeof(hm);
    if (r == p->rank) {
      mboxes[r] = p->mailbox;
      continue;
    }
    void *ptr = nullptr;
    if (cudaIpcOpenMemHandle(&ptr, hm, cudaIpcMemLazyEnablePeerAccess) != cudaSuccess) {
      *err = "cudaIpcOpenMemHandle(mailbox) failed";
      return HYDRO_ECUDA;
    }
    p->opened.push_back(ptr);
    mboxes[r] = (unsigned long long *)ptr;
    for (int64_t i = 0; i < count; ++i) {
      int64_t dom;
      std::memcpy(&dom, w, 8);
      w += 8;
      std::memcpy(&hm, w, sizeof(hm));
      w += sizeof(hm);
      if (dom < 0 || dom >= (int64_t)L.dom.size() || L.dom[dom].rank != r) {
        *err = "peer import: inconsistent domain ownership";
        return HYDRO_EINVAL;
      }
      // map only domains this rank pushes into
      bool needed = false;
      for (const HaloPair &P : L.pairs)
        if (P.dst == dom && slot_of_dom[P.src] >= 0) needed = true;
      if (!needed) continue;
      if (cudaIpcOpenMemHandle(&ptr, hm, cudaIpcMemLazyEnablePeerAccess) != cudaSuccess) {
        *err = "cudaIpcOpenMemHandle(domain) failed";
        return HYDRO_ECUDA;
      }
      p->opened.push_back(ptr);
      dom_base[dom] = ptr;
    }
  }
  if (cudaMalloc(&p->mbox_dev, p->nranks * sizeof(void *)) != cudaSuccess ||
      cudaMemcpy(p->mbox_dev, mboxes.data(), p->nranks * sizeof(void *),
                 cudaMemcpyHostToDevice) != cudaSuccess) {
    *err = "peer mailbox table";
    return HYDRO_ECUDA;
  }
  // slabs this rank pushes (it owns the source, a peer owns the destination) in plan order
  std::vector<PlanEntry> snd, rcv;
  comm_plan(L, p->rank, &snd, &rcv);
  std::vector<PeerSlab> slabs;
  std::vector<DomView> rv[2];
  std::vector<int> view_of_dom(L.dom.size(), -1);
  int64_t biggest = 0;
  for (const PlanEntry &e : snd) {
    const HaloPair &P = L.pairs[e.pair];
    if (view_of_dom[P.dst] < 0) {
      if (!dom_base[P.dst]) {
        *err = "peer import: destination domain not mapped";
        return HYDRO_EINVAL;
      }
      DomView v[2];
      carve_views(dom_base[P.dst], L.dom[P.dst], L.N, P.dst, split, v);
      view_of_dom[P.dst] = (int)rv[0].size();
      rv[0].push_back(v[0]);
      rv[1].push_back(v[1]);
    }
    PeerSlab s;
    s.src_slot = slot_of_dom[P.src];
    s.dst_view = view_of_dom[P.dst];
    int64_t nn = 1;
    for (int a = 0; a < 3; ++a) {
      s.nlo[a] = P.nlo[a]; s.nhi[a] = P.nhi[a]; s.zlo[a] = P.zlo[a]; s.zhi[a] = P.zhi[a];
      nn *= P.nhi[a] - P.nlo[a];
    }
    biggest = std::max(biggest, nn);
    slabs.push_back(s);
    PushTarget pt;
    pt.src_slot = s.src_slot;
    pt.remote = 1;
    for (int a = 0; a < 3; ++a) {
      pt.nlo[a] = P.nlo[a]; pt.nhi[a] = P.nhi[a]; pt.zlo[a] = P.zlo[a]; pt.zhi[a] = P.zhi[a];
    }
    pt.dst[0] = rv[0][s.dst_view];
    pt.dst[1] = rv[1][s.dst_view];
    p->targets.push_back(pt);
  }
  p->nslabs = (int)slabs.size();
  p->blocks = (int)std::max<int64_t>(1, std::min<int64_t>(1024, biggest / 1024));
  if (p->nslabs) {
    for (int par = 0; par < 2; ++par) {
      if (cudaMalloc(&p->remote_dev[par], rv[par].size() * sizeof(DomView)) != cudaSuccess ||
          cudaMemcpy(p->remote_dev[par], rv[par].data(), rv[par].size() * sizeof(DomView),
                     cudaMemcpyHostToDevice) != cudaSuccess) {
        *err = "peer view table";
        return HYDRO_ECUDA;
      }
    }
    if (cudaMalloc(&p->slabs_dev, slabs.size() * sizeof(PeerSlab)) != cudaSuccess ||
        cudaMemcpy(p->slabs_dev, slabs.data(), slabs.size() * sizeof(PeerSlab),
                   cudaMemcpyHostToDevice) != cudaSuccess) {
      *err = "peer slab table";
      return HYDRO_ECUDA;
    }
  }
  p->ready = true;
  return HYDRO_OK;
}

bool peer_ready(const Peer *p) { return p && p->ready; }

int peer_exchange(Peer *p, const DomView *local_views_dev, int par, bool halo, DevState *st,
                  cudaStream_t s) {
  if (halo && p->nslabs)
    k_peer_push<<<dim3(p->blocks, p->nslabs), 256, 0, s>>>(local_views_dev, p->remote_dev[par],
                                                           p->slabs_dev);
  k_peer_sync<<<1, 32, 0, s>>>(st, p->mbox_dev, p->rank, p->nranks);
  return cudaGetLastError() == cudaSuccess ? HYDRO_OK : HYDRO_ECUDA;
}

int peer_kernels_per_cycle(const Peer *p, bool halo) { return (halo && p->nslabs ? 1 : 0) + 1; }

void peer_push_targets(const Peer *p, std::vector<PushTarget> *out) {
  out->insert(out->end(), p->targets.begin(), p->targets.end());
}

void peer_detach(Peer *p) {
  if (!p) return;
  for (void *ptr : p->opened) cudaIpcCloseMemHandle(ptr);
  p->opened.clear();
  p->ready = false;  // the remote slabs are gone: no more cycles
}

void peer_destroy(Peer *p) {
  if (!p) return;
  peer_detach(p);
  cudaFree(p->mailbox);
  cudaFree(p->mbox_dev);
  cudaFree(p->remote_dev[0]);
  cudaFree(p->remote_dev[1]);
  cudaFree(p->slabs_dev);
  delete p;
}

}  // namespace hydro
