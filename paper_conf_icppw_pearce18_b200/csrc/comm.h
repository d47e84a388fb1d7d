// comm.h -- inter-rank communication of the cycle (one process per GPU): the ghost-layer halo
// exchange with neighbouring domains on other ranks ("halo exchange" between
// neighbouring domains; L513-520: the paper routed it through the host, GPU-direct was future
// work) and the global dt min-reduction (S9).  Transport: NCCL 2.28 over NVLink/NVSwitch,
// grouped ncclSend/ncclRecv for the halo, and one ncclAllReduce(max, uint64) per cycle over
// [~dt bits, one word per error bit]: the complemented bit pattern of the non-negative dt gives
// the min (bit order == numeric order for non-negative doubles), the error words give the OR,
// so every rank latches the same status (a tangled zone on one rank halts all of them).
#pragma once
#include <cuda_runtime.h>

#include <string>
#include <vector>

#include "device.cuh"
#include "layout.h"

namespace hydro {

struct Comm;

int comm_unique_id(void *out128);
// remote: halo pairs with exactly one local end (dst or src on this rank).
int comm_create(Comm **out, const hydro_config *cfg, const Layout &L,
                const std::vector<HaloPair> &remote, const std::vector<int32_t> &slot_of_dom,
                void *unused, cudaStream_t s, std::string *err);
// views_p[slot] = &DomView of parity p for every local domain slot (kept by pointer).
int comm_bind_views(Comm *c, const DomView *const *views0, const DomView *const *views1, int n,
                    std::string *err);
// Global S9 inputs: st->dtz_acc <- min over ranks, st->err <- OR over ranks (in place, on s).
int comm_dt_min(Comm *c, DevState *st, cudaStream_t s);
// The same reduction off the critical path (two-kernel path): forked from s after the zone
// stage onto the communicator's own stream and a second communicator (ncclCommSplit), so it
// overlaps the node stages (dt_{n+1} is first read by S9); comm_dt_join makes s wait for it.
int comm_dt_min_async(Comm *c, DevState *st, cudaStream_t s);
int comm_dt_join(Comm *c, cudaStream_t s);
bool comm_dt_overlap(const Comm *c);
// Exchange the next-parity ghost slabs of parity-`par` views with remote neighbours.
int comm_halo(Comm *c, int par, cudaStream_t s);
// Wait for stream s while polling the communicator: returns HYDRO_OK once s is
// idle, HYDRO_ENCCL (after ncclCommAbort) on an asynchronous NCCL error or when the wait exceeds
// timeout_s seconds (a peer that died or a mismatched plan would otherwise hang the caller).
int comm_wait(Comm *c, cudaStream_t s, double timeout_s, std::string *err);
int comm_kernels_per_cycle(const Comm *c);
void comm_destroy(Comm *c);

}  // namespace hydro
