// peer.h -- inter-rank transport over peer memory (CUDA IPC): see peer.cu.
#pragma once
#include <cuda_runtime.h>

#include <string>
#include <vector>

#include "device.cuh"
#include "layout.h"

namespace hydro {

struct Peer;

// A ghost slab that a local source domain stores into a neighbour (fused halo):
// global node / zone boxes (half-open) and the destination's views per parity.
struct PushTarget {
  int32_t src_slot;
  int32_t remote;  // destination owned by another process (peer memory)
  int64_t nlo[3], nhi[3], zlo[3], zhi[3];
  DomView dst[2];
};

// Storage helpers shared with the runtime (runtime.cu): a remote domain's arrays are rebuilt
// from its IPC-mapped base with the same offsets its owner used.
size_t domain_bytes(const DomainBox &b, bool split);
void carve_views(void *base, const DomainBox &b, const int64_t N[3], int32_t dom, bool split,
                 DomView view[2]);

int peer_create(Peer **out, const hydro_config *cfg, std::string *err);
size_t peer_export_size(int nlocal);
// Serialise this rank's IPC handles: [count, mailbox handle, (domain, handle) x count].
int peer_export(Peer *p, const std::vector<int32_t> &local_doms, const std::vector<void *> &bases,
                void *buf, size_t *len, std::string *err);
// all = nranks consecutive records of len_per_rank bytes (every rank's export, rank order).
int peer_import(Peer *p, const Layout &L, const std::vector<int32_t> &slot_of_dom, bool split,
                const void *all, size_t len_per_rank, std::string *err);
bool peer_ready(const Peer *p);
// Push the next-parity ghost slabs of parity-`par` views into the peers (if halo) and reduce dt
// and the error bits over all ranks through the mailboxes.
int peer_exchange(Peer *p, const DomView *local_views_dev, int par, bool halo, DevState *st,
                  cudaStream_t s);
int peer_kernels_per_cycle(const Peer *p, bool halo);
// The inter-rank slabs this rank pushes (after peer_import), for the fused-halo tables.
void peer_push_targets(const Peer *p, std::vector<PushTarget> *out);
// Close every imported IPC mapping (idempotent).  Teardown order across ranks: every rank
// detaches, the caller barriers, then every rank frees (CUDA: freeing an allocation another
// process still has open is undefined).
void peer_detach(Peer *p);
void peer_destroy(Peer *p);

}  // namespace hydro
