// comm.cu -- see comm.h.  NCCL transport for ranks > 1.
#include <nccl.h>

#include <chrono>
#include <cstdlib>
#include <cstring>
#include <thread>

#include "comm.h"

namespace hydro {

namespace {

struct SlabDesc {   // one remote slab: which local domain, which global boxes, buffer offset
  int32_t slot;     // local domain slot (source when packing, destination when unpacking)
  int32_t peer;     // remote rank
  int64_t nlo[3], nhi[3], zlo[3], zhi[3];
  int64_t offset;   // in doubles, into the send or receive buffer
  int64_t count;    // doubles: 6 * nodes + zones
};

__global__ void k_pack(const DomView *views, const SlabDesc *descs, double *buf, int unpack) {
  const SlabDesc p = descs[blockIdx.y];
  const DomView &D = views[p.slot];
  double *b = buf + p.offset;
  const int64_t nx = p.nhi[0] - p.nlo[0], ny = p.nhi[1] - p.nlo[1], nz = p.nhi[2] - p.nlo[2];
  const int64_t nn = nx * ny * nz;
  double *arr[6] = {D.xn, D.yn, D.zn, D.un, D.vn, D.wn};
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < nn;
       t += (int64_t)gridDim.x * blockDim.x) {
    const int64_t a = t % nx, bb = (t / nx) % ny, c = t / (nx * ny);
    const int64_t id = D.nid((int)(p.nlo[0] + a - D.lo[0]), (int)(p.nlo[1] + bb - D.lo[1]),
                             (int)(p.nlo[2] + c - D.lo[2]));
#pragma unroll
    for (int f = 0; f < 6; ++f) {
      if (unpack) arr[f][id] = b[f * nn + t];
      else b[f * nn + t] = arr[f][id];
    }
  }
  const int64_t zx = p.zhi[0] - p.zlo[0], zy = p.zhi[1] - p.zlo[1], zz = p.zhi[2] - p.zlo[2];
  const int64_t nzn = zx * zy * zz;
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < nzn;
       t += (int64_t)gridDim.x * blockDim.x) {
    const int64_t a = t % zx, bb = (t / zx) % zy, c = t / (zx * zy);
    const int64_t id = D.zid((int)(p.zlo[0] + a - D.lo[0]), (int)(p.zlo[1] + bb - D.lo[1]),
                             (int)(p.zlo[2] + c - D.lo[2]));
    if (unpack) D.en[id] = b[6 * nn + t];
    else b[6 * nn + t] = D.en[id];
  }
}

// dt / error words for the allreduce (see comm.h): red[0] = ~dt bits, red[1 + b] = error bit b
__global__ void k_red_pack(const DevState *st, unsigned long long *red) {
  red[0] = ~st->dtz_acc;
#pragma unroll
  for (int b = 0; b < 3; ++b) red[1 + b] = (st->err >> b) & 1u;
}
__global__ void k_red_unpack(DevState *st, const unsigned long long *red) {
  st->dtz_acc = ~red[0];
  unsigned e = 0;
#pragma unroll
  for (int b = 0; b < 3; ++b) e |= red[1 + b] ? (1u << b) : 0u;
  st->err = e;
}

}  // namespace

struct Comm {
  ncclComm_t nccl = nullptr;
  int rank = 0, nranks = 1;
  std::vector<SlabDesc> sends, recvs;  // in global pair order
  SlabDesc *sends_dev = nullptr, *recvs_dev = nullptr;
  double *sendbuf = nullptr, *recvbuf = nullptr;
  int64_t send_total = 0, recv_total = 0;
  DomView *views_dev[2] = {nullptr, nullptr};
  unsigned long long *red_dev = nullptr;  // [4]: the S9 allreduce words
  // overlapped dt reduction (HYDRO_DT_OVERLAP, default on): own communicator and stream
  ncclComm_t dtcomm = nullptr;
  cudaStream_t cs = nullptr;
  cudaEvent_t fork = nullptr, join = nullptr;
};

int comm_unique_id(void *out128) {
  static_assert(sizeof(ncclUniqueId) == 128, "NCCL unique id size");
  ncclUniqueId id;
  if (ncclGetUniqueId(&id) != ncclSuccess) return HYDRO_ENCCL;
  std::memcpy(out128, &id, sizeof(id));
  return HYDRO_OK;
}

int comm_create(Comm **out, const hydro_config *cfg, const Layout &L,
                const std::vector<HaloPair> &remote, const std::vector<int32_t> &slot_of_dom,
                void *, cudaStream_t s, std::string *err) {
  if (!cfg->comm_id) {
    *err = "nranks > 1 needs comm_id";
    return HYDRO_EINVAL;
  }
  Comm *c = new Comm();
  *out = c;
  c->rank = cfg->rank;
  c->nranks = cfg->nranks;
  ncclUniqueId id;
  std::memcpy(&id, cfg->comm_id, sizeof(id));
  if (ncclCommInitRank(&c->nccl, cfg->nranks, id, cfg->rank) != ncclSuccess) {
    *err = "ncclCommInitRank failed";
    return HYDRO_ENCCL;
  }
  std::vector<PlanEntry> snd, rcv;
  comm_plan(L, cfg->rank, &snd, &rcv, (cfg->flags & HYDRO_FLAG_COMM_SELF) != 0);
  (void)remote;
  for (int dir = 0; dir < 2; ++dir) {
    for (const PlanEntry &e : dir ? rcv : snd) {
      const HaloPair &P = L.pairs[e.pair];
      SlabDesc d;
      for (int a = 0; a < 3; ++a) {
        d.nlo[a] = P.nlo[a]; d.nhi[a] = P.nhi[a]; d.zlo[a] = P.zlo[a]; d.zhi[a] = P.zhi[a];
      }
      d.count = e.count;
      d.peer = e.peer;
      if (dir == 0) {  // we own the source: send
        d.slot = slot_of_dom[P.src];
        d.offset = c->send_total;
        c->send_total += d.count;
        c->sends.push_back(d);
      } else {         // we own the destination: receive
        d.slot = slot_of_dom[P.dst];
        d.offset = c->recv_total;
        c->recv_total += d.count;
        c->recvs.push_back(d);
      }
    }
  }
  auto ck = [&](cudaError_t e) {
    if (e != cudaSuccess) *err = cudaGetErrorString(e);
    return e == cudaSuccess;
  };
  {
    const char *ov = getenv("HYDRO_DT_OVERLAP");
    if (!(ov && atoi(ov) == 0)) {
      if (ncclCommSplit(c->nccl, 0, cfg->rank, &c->dtcomm, nullptr) != ncclSuccess) {
        *err = "ncclCommSplit failed";
        return HYDRO_ENCCL;
      }
      int lo = 0, hi = 0;
      cudaDeviceGetStreamPriorityRange(&lo, &hi);
      if (!ck(cudaStreamCreateWithPriority(&c->cs, cudaStreamNonBlocking, hi))) return HYDRO_ECUDA;
      if (!ck(cudaEventCreateWithFlags(&c->fork, cudaEventDisableTiming))) return HYDRO_ECUDA;
      if (!ck(cudaEventCreateWithFlags(&c->join, cudaEventDisableTiming))) return HYDRO_ECUDA;
    }
  }
  if (!ck(cudaMalloc(&c->red_dev, 4 * sizeof(unsigned long long)))) return HYDRO_ECUDA;
  if (c->send_total) {
    if (!ck(cudaMalloc(&c->sendbuf, c->send_total * sizeof(double)))) return HYDRO_ENOMEM;
    if (!ck(cudaMalloc(&c->sends_dev, c->sends.size() * sizeof(SlabDesc)))) return HYDRO_ENOMEM;
    if (!ck(cudaMemcpyAsync(c->sends_dev, c->sends.data(), c->sends.size() * sizeof(SlabDesc),
                            cudaMemcpyHostToDevice, s)))
      return HYDRO_ECUDA;
  }
  if (c->recv_total) {
    if (!ck(cudaMalloc(&c->recvbuf, c->recv_total * sizeof(double)))) return HYDRO_ENOMEM;
    if (!ck(cudaMalloc(&c->recvs_dev, c->recvs.size() * sizeof(SlabDesc)))) return HYDRO_ENOMEM;
    if (!ck(cudaMemcpyAsync(c->recvs_dev, c->recvs.data(), c->recvs.size() * sizeof(SlabDesc),
                            cudaMemcpyHostToDevice, s)))
      return HYDRO_ECUDA;
  }
  return HYDRO_OK;
}

int comm_bind_views(Comm *c, const DomView *const *v0, const DomView *const *v1, int n,
                    std::string *err) {
  for (int p = 0; p < 2; ++p) {
    std::vector<DomView> vv;
    for (int i = 0; i < n; ++i) vv.push_back(*(p ? v1[i] : v0[i]));
    if (cudaMalloc(&c->views_dev[p], sizeof(DomView) * (n ? n : 1)) != cudaSuccess) {
      *err = "cudaMalloc views";
      return HYDRO_ENOMEM;
    }
    if (n && cudaMemcpy(c->views_dev[p], vv.data(), sizeof(DomView) * n,
                        cudaMemcpyHostToDevice) != cudaSuccess) {
      *err = "cudaMemcpy views";
      return HYDRO_ECUDA;
    }
  }
  return HYDRO_OK;
}

int comm_dt_min(Comm *c, DevState *st, cudaStream_t s) {
  k_red_pack<<<1, 1, 0, s>>>(st, c->red_dev);
  if (ncclAllReduce(c->red_dev, c->red_dev, 4, ncclUint64, ncclMax, c->nccl, s) != ncclSuccess)
    return HYDRO_ENCCL;
  k_red_unpack<<<1, 1, 0, s>>>(st, c->red_dev);
  return cudaGetLastError() == cudaSuccess ? HYDRO_OK : HYDRO_ECUDA;
}

bool comm_dt_overlap(const Comm *c) { return c && c->dtcomm; }

int comm_dt_min_async(Comm *c, DevState *st, cudaStream_t s) {
  if (!c->dtcomm) return comm_dt_min(c, st, s);
  if (cudaEventRecord(c->fork, s) != cudaSuccess) return HYDRO_ECUDA;
  if (cudaStreamWaitEvent(c->cs, c->fork, 0) != cudaSuccess) return HYDRO_ECUDA;
  k_red_pack<<<1, 1, 0, c->cs>>>(st, c->red_dev);
  if (ncclAllReduce(c->red_dev, c->red_dev, 4, ncclUint64, ncclMax, c->dtcomm, c->cs) !=
      ncclSuccess)
    return HYDRO_ENCCL;
  k_red_unpack<<<1, 1, 0, c->cs>>>(st, c->red_dev);
  if (cudaEventRecord(c->join, c->cs) != cudaSuccess) return HYDRO_ECUDA;
  return cudaGetLastError() == cudaSuccess ? HYDRO_OK : HYDRO_ECUDA;
}

int comm_dt_join(Comm *c, cudaStream_t s) {
  if (!c->dtcomm) return HYDRO_OK;
  return cudaStreamWaitEvent(s, c->join, 0) == cudaSuccess ? HYDRO_OK : HYDRO_ECUDA;
}

int comm_halo(Comm *c, int par, cudaStream_t s) {
  if (!c->sends.empty())
    k_pack<<<dim3(8, (unsigned)c->sends.size()), 256, 0, s>>>(c->views_dev[par], c->sends_dev,
                                                              c->sendbuf, 0);
  if (ncclGroupStart() != ncclSuccess) return HYDRO_ENCCL;
  // Every rank walks the global pair list in the same order, so sends and receives between a
  // pair of ranks match one to one.
  for (const SlabDesc &d : c->sends)
    if (ncclSend(c->sendbuf + d.offset, d.count, ncclFloat64, d.peer, c->nccl, s) != ncclSuccess)
      return HYDRO_ENCCL;
  for (const SlabDesc &d : c->recvs)
    if (ncclRecv(c->recvbuf + d.offset, d.count, ncclFloat64, d.peer, c->nccl, s) != ncclSuccess)
      return HYDRO_ENCCL;
  if (ncclGroupEnd() != ncclSuccess) return HYDRO_ENCCL;
  if (!c->recvs.empty())
    k_pack<<<dim3(8, (unsigned)c->recvs.size()), 256, 0, s>>>(c->views_dev[par], c->recvs_dev,
                                                              c->recvbuf, 1);
  return cudaGetLastError() == cudaSuccess ? HYDRO_OK : HYDRO_ECUDA;
}

int comm_wait(Comm *c, cudaStream_t s, double timeout_s, std::string *err) {
  if (!c->nccl) return HYDRO_OK;  // aborted earlier: the caller's stream sync reports the rest
  const auto t0 = std::chrono::steady_clock::now();
  for (int spin = 0;; ++spin) {
    const cudaError_t q = cudaStreamQuery(s);
    if (q == cudaSuccess) return HYDRO_OK;
    if (q != cudaErrorNotReady) {
      *err = std::string("stream: ") + cudaGetErrorString(q);
      return HYDRO_ECUDA;
    }
    // asynchronous error of either communicator (a failing query counts as an error too)
    auto async_error = [](ncclComm_t comm) {
      ncclResult_t r = ncclSuccess;
      if (ncclCommGetAsyncError(comm, &r) != ncclSuccess) return ncclInternalError;
      return r;
    };
    ncclResult_t ae = async_error(c->nccl);
    if (ae == ncclSuccess && c->dtcomm) ae = async_error(c->dtcomm);
    if (ae != ncclSuccess) {
      *err = std::string("NCCL asynchronous error: ") + ncclGetErrorString(ae);
      if (c->dtcomm) ncclCommAbort(c->dtcomm);
      ncclCommAbort(c->nccl);
      c->nccl = nullptr;
      c->dtcomm = nullptr;
      return HYDRO_ENCCL;
    }
    const double el =
        std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
    if (timeout_s > 0.0 && el > timeout_s) {
      *err = "NCCL wait timed out (a peer rank stalled or died)";
      if (c->dtcomm) ncclCommAbort(c->dtcomm);
      ncclCommAbort(c->nccl);
      c->nccl = nullptr;
      c->dtcomm = nullptr;
      return HYDRO_ENCCL;
    }
    if (spin > 64) std::this_thread::sleep_for(std::chrono::microseconds(50));
  }
}

int comm_kernels_per_cycle(const Comm *c) {
  return (c->sends.empty() ? 0 : 1) + (c->recvs.empty() ? 0 : 1) + 2;  // + dt pack/unpack
}

void comm_destroy(Comm *c) {
  if (!c) return;
  if (c->dtcomm) ncclCommDestroy(c->dtcomm);
  if (c->nccl) ncclCommDestroy(c->nccl);
  if (c->cs) cudaStreamDestroy(c->cs);
  if (c->fork) cudaEventDestroy(c->fork);
  if (c->join) cudaEventDestroy(c->join);
  cudaFree(c->sendbuf);
  cudaFree(c->recvbuf);
  cudaFree(c->sends_dev);
  cudaFree(c->recvs_dev);
  cudaFree(c->views_dev[0]);
  cudaFree(c->views_dev[1]);
  cudaFree(c->red_dev);
  delete c;
}

}  // namespace hydro
