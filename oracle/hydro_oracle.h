/*
 * hydro_oracle.h -- TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, single-threaded C++ fp64 reference ("oracle") of the explicit staggered-grid
 * Lagrangian hydro cycle that the B200 library computes.  Only tests/, __graft_entry__.smoke()
 * and bench.py's cpu_baseline / --impl reference legs may load this library.  It shares no code,
 * header, table or constant with the CUDA path (include/hydro.h, paper_conf_icppw_pearce18_b200/).
 *
 * What it computes: the workload is the 3-D Sedov blast wave of PAPER.md L637-642 ("The Sedov
 * problem stresses the hydrodynamics calculation"), on a block-structured mesh decomposed into
 * domains (§6.1).  The paper never writes the hydro algorithm down; the cycle
 * (steps S1-S9) and every silent point follow SURVEY.md §8c and are listed as readings R1-R18 in
 * DESIGN.md §3.
 *
 * Conventions: zones (i,j,k), 0<=i<nx, x fastest; nodes 0<=i<=nx.  Corner l = a+2b+4c of zone
 * (i,j,k) is node (i+a,j+b,k+c).  All arithmetic is IEEE fp64, compiled -O2 -ffp-contract=off.
 */
#ifndef HYDRO_ORACLE_H
#define HYDRO_ORACLE_H
#include <stdint.h>
#include <stddef.h>

#ifdef __cplusplus
extern "C" {
#endif

enum { ORC_INIT_SEDOV = 0, ORC_INIT_USER = 1, ORC_INIT_USER_MASS = 2 };

enum {
  ORC_OK = 0,
  ORC_EINVAL = -1,
  ORC_ETANGLED = -5,   /* a zone volume <= 0 */
  ORC_ENONFINITE = -6, /* non-finite P or dt */
  ORC_EDTMIN = -7,     /* min_z dt_z of a cycle fell below the dt floor (reading R23) */
  ORC_ESTATE = -8      /* context already failed */
};

typedef struct {
  int64_t n[3];                 /* global zones per axis */
  double origin[3], extent[3];  /* box; node i at origin + (extent*i)/n   (reading R1) */
  int32_t ndom[3];              /* domains per axis (>=1) */
  const int64_t *cuts[3];       /* optional: ndom[a]+1 strictly increasing cut points, 0..n */
  double gamma, q_lin, q_quad;  /* ideal-gas gamma (R5); viscosity coefficients (R7) */
  double cfl, c_vol, dt_growth, dt_max, dt_init, t_stop; /* dt rule (R8) */
  double dt_first;              /* >0: use exactly this as dt^0 (restart / window runs) */
  double t0;                    /* start time */
  uint32_t reflect_mask;        /* bits: -x,+x,-y,+y,-z,+z  (R9) */
  int32_t init_kind;            /* ORC_INIT_* */
  double rho0, e0, sedov_energy;/* SEDOV: rho0, background e0, energy put in zone (0,0,0) (R10) */
  /* USER / USER_MASS: global arrays, x fastest.  [0..5] = x,y,z,u,v,w on (n+1)^3 nodes;
     [6] = rho (USER) or zone mass (USER_MASS) on n^3 zones; [7] = e on zones. */
  const double *user[8];
  double hg_coef;               /* viscous hourglass coefficient kappa >= 0 (reading R17; 0 = off) */
  double dt_floor;              /* dt-collapse floor (reading R23): > 0 absolute; 0 = 1e-6 * dt^0;
                                   < 0 = none.  A cycle whose min_z dt_z is below it halts the run
                                   with ORC_EDTMIN (bad_zone -1), unless it ends the run at t_stop */
  int32_t q_kind;               /* 0: scalar q (reading R7); 1: monotone q (reading R24) */
} orc_config;

typedef struct {
  double t, dt;        /* time after the last cycle, and the dt the next cycle will use */
  int64_t cycle;
  double dt_min_zone;  /* min_z dt_z of the last cycle (before growth/max limits) */
  int64_t bad_zone;    /* global linear index of the first zone that failed, or -1 */
} orc_info;

/* field selectors for orc_get_fields (global arrays, x fastest) */
enum {
  ORC_F_X = 1 << 0, ORC_F_Y = 1 << 1, ORC_F_Z = 1 << 2,
  ORC_F_U = 1 << 3, ORC_F_V = 1 << 4, ORC_F_W = 1 << 5,
  ORC_F_RHO = 1 << 6, ORC_F_E = 1 << 7, ORC_F_P = 1 << 8, ORC_F_Q = 1 << 9,
  ORC_F_C = 1 << 10, ORC_F_VOL = 1 << 11, ORC_F_MASS = 1 << 12
};
#define ORC_NFIELDS 13

typedef struct orc_ctx orc_ctx;

int orc_create(const orc_config *cfg, orc_ctx **out);
int orc_step(orc_ctx *h, int32_t ncycles, orc_info *info);
/* out[f] for every bit f set in mask: caller-owned array of (n+1)^3 (nodes) or n^3 (zones). */
int orc_get_fields(const orc_ctx *h, uint32_t mask, double *const *out);
int orc_info_get(const orc_ctx *h, orc_info *info);
void orc_destroy(orc_ctx *h);
const char *orc_last_error(void);

/* --- single-zone kernels exposed for pins (tests/test_oracle_geometry.py) --------------- */
/* S2 geometry of one hex: X[l][d] corner positions -> corner vectors B[l][d], volume V,
   characteristic length L = V/sqrt(max face area^2) (readings R2-R4). */
void orc_zone_geometry(const double X[8][3], double B[8][3], double *V, double *L);
/* S2-S6 for one zone: positions X (already the half-step positions), velocities U, mass m,
   energy e, half step hh -> rho, e_p, p, c, q, P, dt_z (readings R5-R8). */
void orc_zone_state(const double X[8][3], const double U[8][3], double m, double e, double hh,
                    double gamma, double q_lin, double q_quad, double cfl, double c_vol,
                    double out[8] /* rho, e_p, p, c, q, P, dt_z, V */);

/* f1 (reading R24): strain rate eps_d and length L_d of one zone along each logical direction,
   and the monotonic limiter of one direction from the strain rates (em, e0, ep). */
void orc_zone_strain(const double X[8][3], const double U[8][3], double eps[3], double L[3]);
double orc_mono_limiter(double em, double e0, double ep);

/* f1 (reading R17): Flanagan-Belytschko viscous hourglass corner forces of one zone, from the
   half-step positions X, velocities U, corner vectors B, V, rho, c and kappa (hydro_oracle.cpp). */
void orc_zone_hourglass(const double X[8][3], const double U[8][3], const double B[8][3],
                        double V, double rho, double c, double kappa, double F[8][3]);

#ifdef __cplusplus
}
#endif
#endif
