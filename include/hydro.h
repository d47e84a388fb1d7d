/*
 * hydro.h -- C ABI of the B200-native explicit Lagrangian hydro library (libhydro_b200.so).
 *
 * What the library computes.  One explicit staggered-grid Lagrangian hydrodynamics cycle per
 * hydro_step() cycle, over a structured 3-D mesh decomposed into domains that are owned by ranks
 * (one process per GPU) and exchange a one-layer halo: the problem statement of PAPER.md
 * L307-310 ("2D and 3D block-structured ... meshes", "each MPI rank owns its domain"),
 * L525-557 (§6.1 domain decomposition, halo exchange between neighbouring domains) and
 * L559-572 (hierarchical decomposition).  The workload is the 3-D Sedov blast wave of
 * L637-642.  The paper does not state the hydro equations; the cycle is SURVEY.md §8c
 * (readings R1-R18): per cycle S1 half-step positions, S2 zone geometry,
 * S3 EOS p and c with an energy predictor, S4 artificial viscosity, S5 corner forces,
 * S6 zone dt, S7 nodal force gather / acceleration / velocity and position update,
 * S8 compatible internal-energy update, S9 global dt min-reduction.
 *
 * Conventions (all calls).
 *   - Global zones (i,j,k), 0 <= i < n[0], x fastest (x is the innermost
 *     dimension).  Global nodes 0 <= i <= n[0].  Host field arrays are dense, x fastest:
 *     (n0+1)(n1+1)(n2+1) doubles for node fields, n0*n1*n2 doubles for zone fields.
 *   - All arithmetic is IEEE fp64 on the GPU (sm_100a).  No CPU fallback exists: every call that
 *     computes returns HYDRO_ECUDA if no CUDA device is usable.
 *   - Return codes: HYDRO_OK (0) or a negative HYDRO_E* code; no exception or abort crosses the
 *     ABI.  hydro_last_error() gives a message for the last failure on a context.
 *   - Ownership: every pointer in hydro_config is borrowed for the duration of hydro_create only.
 *     The context owns all device memory, streams, events, CUDA graphs and communicators.
 *     Output buffers are caller-allocated host memory (pageable or pinned).
 *   - Threading: one host thread per context at a time.
 */
#ifndef HYDRO_B200_H
#define HYDRO_B200_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define HYDRO_ABI_VERSION 4

typedef struct hydro_ctx hydro_ctx; /* opaque; owned by the library */

enum {
  HYDRO_OK = 0,
  HYDRO_EINVAL = -1,     /* invalid argument or configuration */
  HYDRO_ENOMEM = -2,     /* device or host allocation failed */
  HYDRO_ECUDA = -3,      /* CUDA runtime error (or no device) */
  HYDRO_ENCCL = -4,      /* communicator error */
  HYDRO_ETANGLED = -5,   /* a zone volume became <= 0 */
  HYDRO_ENONFINITE = -6, /* a non-finite pressure or dt appeared */
  HYDRO_EDTMIN = -7,     /* the zone dt minimum of a cycle fell below hydro_config.dt_floor
                            (dt collapse, reading R23; bad_zone = -1: a global condition) */
  HYDRO_ESTATE = -8      /* the context failed earlier; only get_fields/destroy still work */
};

enum { HYDRO_INIT_SEDOV = 0, HYDRO_INIT_USER = 1, HYDRO_INIT_USER_MASS = 2 };

/* Field selectors for hydro_get_fields / hydro_get_box (bit f selects out[f]). */
enum {
  HYDRO_F_X = 1 << 0, HYDRO_F_Y = 1 << 1, HYDRO_F_Z = 1 << 2,    /* node positions */
  HYDRO_F_U = 1 << 3, HYDRO_F_V = 1 << 4, HYDRO_F_W = 1 << 5,    /* node velocities */
  HYDRO_F_RHO = 1 << 6, HYDRO_F_E = 1 << 7, HYDRO_F_P = 1 << 8, /* zone density, energy, p */
  HYDRO_F_Q = 1 << 9, HYDRO_F_C = 1 << 10,                       /* zone viscosity, sound speed */
  HYDRO_F_VOL = 1 << 11, HYDRO_F_MASS = 1 << 12                  /* zone volume, mass */
};
#define HYDRO_NFIELDS 13

/* hydro_config.flags */
#define HYDRO_FLAG_NO_GRAPH (1ull << 0) /* launch kernels directly instead of CUDA graphs */
#define HYDRO_FLAG_SPLIT (1ull << 1)    /* plain 3-kernel pipeline (one thread per element) */
#define HYDRO_FLAG_ONE_KERNEL (1ull << 2) /* one fused kernel per cycle (zone ring recomputed)
                                             instead of the default zone + node/energy pair */
#define HYDRO_FLAG_PEER (1ull << 3)       /* nranks > 1: exchange halos and reduce dt through peer
                                             memory (CUDA IPC; ranks may share a GPU) instead of
                                             NCCL; needs hydro_peer_export/import after create */
#define HYDRO_FLAG_HALO_FUSED (1ull << 4) /* default path: the node/energy stage stores the ghost
                                             slabs into the neighbours (intra-GPU and peer) from
                                             its own epilogue instead of the separate copy / push
                                             kernels after it (correct, measured
                                             slower on B200, so opt-in) */
#define HYDRO_FLAG_COMM_SELF (1ull << 6) /* nranks == 1: still create the NCCL communicator
                                             (a one-rank world; comm_id required) and move the
                                             ghost slabs between this rank's domains by NCCL
                                             send/recv to itself (pack, grouped send/recv,
                                             unpack) instead of the copy kernel, so the NCCL
                                             halo and dt / error allreduce, its overlap stream,
                                             the async-error polling and the teardown run on a
                                             one-GPU box (testing; results equal the
                                             communicator-free run bitwise) */
#define HYDRO_FLAG_STRICT (1ull << 5)     /* the split pipeline evaluated in the canonical
                                             operation order of SURVEY §8c (readings R12, R13),
                                             compiled without FMA contraction: BITWISE equal to
                                             the oracle (hg_coef = 0; with hg_coef > 0 to within
                                             the rounding of cbrt).  A checking path, not a
                                             fast one. */

typedef struct {
  int32_t abi_version;          /* must be HYDRO_ABI_VERSION */
  int64_t n[3];                 /* global zones per axis, >= 1 */
  double origin[3], extent[3];  /* box; initial node i at origin + (extent*i)/n (reading R1) */
  int32_t ndom[3];              /* domains per axis, >= 1 */
  const int64_t *cuts[3];       /* optional per-axis cut points, ndom[a]+1 strictly increasing
                                   values from 0 to n[a]; NULL = even split n*d/ndom */
  const int32_t *dom_to_rank;   /* optional explicit domain -> rank map (domain index
                                   (c*ndom1+b)*ndom0+a); NULL = weighted LPT rule (reading R19,
                                   PAPER.md L597-603) */
  const double *rank_weight;    /* optional per-rank speed weights for the LPT rule; NULL=equal */
  double gamma;                 /* ideal-gas gamma > 1 (reading R5) */
  double q_lin, q_quad;         /* artificial-viscosity coefficients >= 0 (reading R7) */
  double cfl, c_vol;            /* dt_z = min(cfl*L/sigma, c_vol/|D|) (reading R8) */
  double dt_growth, dt_max;     /* dt_{n+1} = min(dt_growth*dt_n, dt_max, min_z dt_z) */
  double dt_init;               /* dt^0 = min(dt_init, dt_max, min_z dt_z^0) */
  double t_stop;                /* > 0: clamp dt to hit t_stop exactly, then cycles are no-ops */
  double dt_first;              /* > 0: use exactly this as dt^0 (restart) */
  double t0;                    /* start time */
  uint32_t reflect_mask;        /* reflecting walls, bits -x,+x,-y,+y,-z,+z (reading R9) */
  int32_t init_kind;            /* HYDRO_INIT_* */
  double rho0, e0, sedov_energy;/* SEDOV: density, background energy, energy in zone (0,0,0) */
  const double *user[8];        /* USER/USER_MASS global host arrays (every rank): x,y,z,u,v,w
                                   on nodes; [6] rho (USER) or zone mass (USER_MASS); [7] e */
  int32_t rank, nranks;         /* this process and the job size (1 = single process) */
  int32_t device;               /* CUDA device ordinal for this rank */
  const void *comm_id;          /* nranks > 1: 128-byte id from hydro_comm_unique_id() on rank 0,
                                   broadcast by the caller (e.g. torch.distributed) */
  uint64_t flags;               /* HYDRO_FLAG_* */
  double hg_coef;               /* viscous hourglass coefficient kappa >= 0 (SURVEY §8f row f1,
                                   reading R17): f_l += -kappa rho c V^(2/3) sum_a gamma_al g_a
                                   (Flanagan-Belytschko).  0 = off (the default,
                                   north_star's phase list).  kappa > 0 runs the split kernels
                                   (corner-force planes in HBM), whatever the path flags say. */
  double dt_floor;              /* dt-collapse floor (reading R23): > 0 absolute;
                                   0 (the default) = 1e-6 * dt^0 (dt^0 before the t_stop clamp);
                                   < 0 = no floor.  A cycle whose min_z dt_z falls below it halts
                                   the run with HYDRO_EDTMIN (state = the one after that cycle),
                                   unless that cycle reaches t_stop. */
  int32_t q_kind;               /* artificial viscosity: 0 = scalar von
                                   Neumann-Richtmyer + Landshoff q (reading R7, the default);
                                   1 = monotone q (reading R24: per logical direction, limited by
                                   the neighbours' strain rates; single rank only, runs the split
                                   kernels like hg_coef > 0; EINVAL with nranks > 1) */
} hydro_config;

typedef struct {
  double t;            /* time after the last cycle */
  double dt;           /* dt the next cycle will use */
  int64_t cycle;       /* cycles completed since create */
  double dt_min_zone;  /* global min_z dt_z of the last cycle */
  int32_t status;      /* HYDRO_OK or the physics error that halted the run */
  int64_t bad_zone;    /* global linear index of the lowest failing zone, or -1 */
} hydro_info;

/* Fill cfg with the defaults of DESIGN.md §3 (gamma 1.4, q 0.5/2.0, cfl 0.3, c_vol 0.1,
   dt_growth 1.1, dt_max = dt_init = +inf, reflecting walls, Sedov on [0,1.2]^3 with
   sedov_energy = 0.851072/8, dt_floor 0 = 1e-6 dt^0, single rank, device 0). */
void hydro_config_default(hydro_config *cfg);

/* Create: validate cfg, build the layout (domains, halo maps, domain->rank map), allocate the
   domains owned by cfg->rank on cfg->device, initialise them (Sedov on the device, or USER
   arrays copied host->device), exchange the halo and compute dt^0.  Collective over ranks.
   Errors: HYDRO_EINVAL (bad cfg; *out = NULL), HYDRO_ENOMEM, HYDRO_ECUDA, HYDRO_ENCCL,
   HYDRO_ETANGLED (initial mesh has a zone with V <= 0). */
int hydro_create(const hydro_config *cfg, hydro_ctx **out);

/* Run ncycles >= 0 cycles.  Work is enqueued on cuda_stream (a cudaStream_t; NULL = the
   context's own stream) and the call returns after it completed (one host synchronisation per
   call, not per cycle).  info (optional) receives the state after the last cycle.  Collective.
   Returns HYDRO_OK, or the physics error of the cycle that failed (the state is the one after
   that cycle; later calls return HYDRO_ESTATE), or HYDRO_ECUDA / HYDRO_ENCCL.  Cycles after
   t_stop or after a failure are no-ops; a single-rank context stops launching them (within
   ~512 cycles of the end), a multi-rank one launches all of them (their collectives pair up
   across ranks).  HYDRO_ENCCL also covers an NCCL asynchronous error or a wait longer than
   HYDRO_NCCL_TIMEOUT_S seconds (default 600): the communicators are then aborted. */
int hydro_step(hydro_ctx *h, int32_t ncycles, void *cuda_stream, hydro_info *info);

/* Copy fields of the current state into caller-owned global host arrays.  out[f] is used for
   every bit f in mask (HYDRO_F_*); derived zone fields (rho, p, q, c, vol) are evaluated on the
   device at (x, u) with no predictor (SURVEY §8c.3 "Outputs").  With nranks > 1 each rank writes
   only the entries owned by its domains (interface nodes: lowest domain index) and leaves the
   rest untouched, so the caller combines ranks (the Python binding all-reduces).  Works on a
   failed context.  Errors: HYDRO_EINVAL, HYDRO_ECUDA. */
int hydro_get_fields(hydro_ctx *h, uint32_t mask, double *const *out);

/* Like hydro_get_fields but for the global zone box [lo, hi) (nodes [lo, hi] inclusive);
   out arrays are dense boxes of (hi-lo+1) node or (hi-lo) zone extents, x fastest. */
int hydro_get_box(hydro_ctx *h, const int64_t lo[3], const int64_t hi[3], uint32_t mask,
                  double *const *out);

/* Replace the state (x,y,z,u,v,w on nodes, e on zones; global host arrays, every rank) and set
   t and the next dt (clamped to t_stop - t when t_stop > 0, as at creation); zone masses are
   kept.  Used for restart and for the end-to-end benchmark
   (host -> device copies through the public API).  Clears a failed state.  Collective. */
int hydro_set_state(hydro_ctx *h, const double *const *nodes6, const double *e, double t,
                    double dt);

/* Streamed batches of independent runs on this context's mesh (an ensemble: many initial
   states through the same cycle).  Batch b starts from the host state in[7b .. 7b+6] = x, y, z,
   u, v, w (global node arrays) and e (global zone array), laid out as for hydro_set_state,
   with clock t0[b], dt0[b] (clamped as by hydro_set_state) and cycle 0; it runs ncycles cycles (the hot path of hydro_step)
   and writes x, y, z, u, v, w, e after them into out[7b .. 7b+6] (as hydro_get_fields).  Zone
   masses are the context's, as for hydro_set_state.  The host->device copy of batch b+1 and
   the device->host copy of batch b-1 run on two copy streams while batch b computes (two
   device staging slots each way, allocated on first use and kept until hydro_destroy), so for
   page-locked host buffers the transfers hide behind the cycles.  info (NULL or nbatch
   entries) receives each batch's final clock and status; the return value is the first
   nonzero batch status (a physics error ends only that batch's cycles, later batches still
   run), HYDRO_EINVAL for bad arguments or a multi-rank context (nranks > 1), HYDRO_ECUDA.
   Synchronous on return; the context then holds the last batch's state.  Not collective. */
int hydro_run_batch(hydro_ctx *h, int32_t nbatch, int32_t ncycles, const double *const *in,
                    double *const *out, const double *t0, const double *dt0, hydro_info *info);

/* Peer transport (HYDRO_FLAG_PEER) bootstrap, collective: after hydro_create every rank calls
   hydro_peer_export (buf NULL: *len = bytes needed), the caller all-gathers the records (padded to
   a common len_per_rank, rank order), and every rank calls hydro_peer_import with all of them;
   import maps the neighbours' domain allocations and mailboxes, reduces dt^0 over the ranks and
   captures the cycle graphs.  hydro_step returns HYDRO_ESTATE before import.
   Errors: HYDRO_EINVAL (bad records), HYDRO_ECUDA (IPC failures). */
int hydro_peer_export(hydro_ctx *h, void *buf, size_t *len);
int hydro_peer_import(hydro_ctx *h, const void *all, size_t len_per_rank);

/* Peer transport teardown, step 1 of 3 (collective order): close this rank's mappings of the
   other ranks' memory after its own work drained.  Then the caller barriers over all ranks, then
   every rank calls hydro_destroy (which frees memory the others had mapped: freeing it while
   another process still has it open is undefined in CUDA).  No-op without HYDRO_FLAG_PEER.
   After it, hydro_step returns HYDRO_ESTATE. */
int hydro_peer_detach(hydro_ctx *h);

/* Current info without stepping.  Local (not a collective): the status is already identical on
   every rank because both transports OR-reduce the error bits with dt every cycle. */
int hydro_get_info(hydro_ctx *h, hydro_info *info);

/* Domain migration: the complete state of one domain this rank owns, i.e.
   its current node arrays x,y,z,u,v,w and zone arrays e and m over the domain's storage box
   including the ghost layer (layout: 6 node arrays of (n0+3 padded to 4)(n1+3)(n2+3) doubles,
   then e and m of (n0+2 padded to 4)(n1+2)(n2+2) doubles), as a flat device buffer.  The
   storage depends only on the domain box, so a buffer packed by one context unpacks into any
   context with the same cuts, on any rank; moving it between ranks is the caller's (e.g.
   torch.distributed send/recv over NCCL).  hydro_domain_bytes: *len = bytes of dom's buffer
   (host-only arithmetic, any domain).  pack: dev_buf (device memory, or host memory: the
   copies use the unified address space, page-locked host memory runs at DMA speed; >= len
   bytes, caller-owned) <- state, on `stream` (NULL = the context's), synchronised before
   return.  unpack: state <- dev_buf (same), then 1/m and the nodal 8/sum m are recomputed for
   that domain.  With host buffers this pair is the rank-local end-to-end path (bench.py e2e at
   N > 1: each rank moves exactly its own domains).  Errors:
   HYDRO_EINVAL (dom not owned by this rank, len too small), HYDRO_ECUDA. */
int hydro_domain_bytes(const hydro_ctx *h, int32_t dom, size_t *len);
int hydro_domain_pack(hydro_ctx *h, int32_t dom, void *dev_buf, size_t len, void *stream);
int hydro_domain_unpack(hydro_ctx *h, int32_t dom, const void *dev_buf, size_t len,
                        void *stream);
/* Set the run clock (t, the dt of the next cycle, the cycle counter) and clear error state:
   continues a migrated or restarted run exactly.  dt > 0.  Errors: HYDRO_EINVAL, HYDRO_ECUDA. */
int hydro_set_clock(hydro_ctx *h, double t, double dt, int64_t cycle);

/* Destroy; NULL-safe; collective. */
int hydro_destroy(hydro_ctx *h);

/* Measurement helper (bench.py): run ncycles cycles WITHOUT CUDA graphs on the context stream,
   bracketing each kernel class with CUDA events, and report mean device milliseconds:
   out_ms[0] cycle kernels of one domain (zone + node/energy stage by default; the one fused
   kernel with HYDRO_FLAG_ONE_KERNEL; zone+node+energy with HYDRO_FLAG_SPLIT),
   out_ms[1] halo exchange per cycle, out_ms[2] dt finalize per cycle, out_ms[3] whole cycle,
   out_ms[4] zone stage and out_ms[5] node/energy stage of one domain (default path, else 0).
   Advances the state like hydro_step.  Collective. */
int hydro_time_kernels(hydro_ctx *h, int32_t ncycles, double out_ms[6]);

/* Number of kernels of this library launched per cycle on this rank (bench.py gpu_launches). */
int hydro_kernels_per_cycle(const hydro_ctx *h);

/* --- host-only helpers (no CUDA device needed) --------------------------------------------- */

/* Build the integer layout for cfg without touching the GPU and serialise it as int64 words
   into buf (capacity *len words; on return *len = words needed).  Format in DESIGN.md §5:
   header [version, ndom, nranks, npairs], per domain [lo0,lo1,lo2,n0,n1,n2,rank],
   per halo pair [dst_dom, src_dom, dir, node box (6), zone box (6)].  Used by the bitwise
   layout tests. */
int hydro_layout_export(const hydro_config *cfg, int64_t *buf, size_t *len);

/* Inter-rank halo plan of cfg->rank (host-only; what the communicator will send and receive):
   words [nsend, nrecv, then per message (sends first, each list in global pair order)
   pair, peer rank, count of doubles, dst domain, src domain, direction].  Every rank enumerates
   the messages between two ranks in the same order, which is what makes the grouped NCCL
   send/recv match.  Returns HYDRO_EINVAL if cfg is invalid or buf is too small. */
int hydro_comm_plan_export(const hydro_config *cfg, int64_t *buf, size_t *len);

/* Hierarchical decomposition (Fig. 10a,b): split n into ngpu near-cubic
   blocks (minimum total interface area; x split last, L587), then each block into dpg slabs along
   y ("a single dimension").  Writes ndom[3], cuts (cuts[a] must hold n[a]+1 entries) and
   dom_to_rank (capacity ngpu*dpg).  Returns HYDRO_EINVAL if impossible. */
int hydro_decompose_hierarchical(const int64_t n[3], int32_t ngpu, int32_t dpg, int32_t ndom[3],
                                 int64_t *const cuts[3], int32_t *dom_to_rank);

/* Weighted slab split (Fig. 10c, whole-plane granularity L657-660):
   nplanes planes over nparts parts with weights w: n_g = floor(N w_g / W), remaining planes to
   the largest remainders (ties: lowest g), every n_g >= 1.  out[nparts] receives n_g. */
int hydro_weighted_slabs(int64_t nplanes, int32_t nparts, const double *w, int64_t *out);

/* Measured-weight rebalancing between runs ("an initial
   guess of work split ... based on FLOPS.  We measured the respective contributions ... and
   adjusted the split"; L1077-1081: "static within an iteration, but the decomposition can be
   adjusted between iterations").  Host-only and deterministic, so every rank computes the same
   plan.  cfg describes the CURRENT layout (its dom_to_rank or weighted-rule map); busy[nranks]
   is each rank's measured device time per cycle under it (> 0, any unit).  Domain cost =
   owned zones + beta * ghost elements (beta >= 0, the surface term); rank speed
   w_g = load_g / busy_g (normalised to mean 1; a rank without domains gets the mean); the new
   map is the LPT rule with those weights (reading R19), kept only if the modelled makespan
   max_g load_g / w_g drops by more than min_gain (fraction), else new_map = the current map.
   Outputs: new_map[ndomains], weights[nranks] (may be NULL), predicted[2] = modelled makespan
   before / after in busy units (may be NULL).  Errors: HYDRO_EINVAL. */
int hydro_rebalance_plan(const hydro_config *cfg, const double *busy, double beta,
                         double min_gain, int32_t *new_map, double *weights, double *predicted);

/* 128-byte communicator id for nranks > 1 (call on rank 0, broadcast to all ranks). */
int hydro_comm_unique_id(void *out128);

const char *hydro_strerror(int status);
const char *hydro_last_error(const hydro_ctx *h);
int hydro_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* HYDRO_B200_H */
