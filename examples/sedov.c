/* sedov.c -- the C ABI without Python: a 3-D Sedov octant through
 * include/hydro.h only.  Build (done by __graft_entry__.build()):
 *   gcc -O2 -std=c99 -Iinclude examples/sedov.c -Lpaper_conf_icppw_pearce18_b200 -lhydro_b200 \
 *       -Wl,-rpath,<abs path of paper_conf_icppw_pearce18_b200> -lm -o build/sedov_c
 * Run on a GPU box:  build/sedov_c [n] [cycles]
 * Prints t, dt, total mass and total energy (internal + kinetic with lumped nodal masses) before
 * and after, and exits non-zero on any library error or if the energy drifts by more than 1e-10.
 */
#include <math.h>
#include <stdio.h>
#include <stdlib.h>

#include "hydro.h"

static double total_energy(int64_t n, const double *const *f) {
  /* f: u, v, w (nodes), e, mass (zones) */
  const int64_t nn = n + 1;
  double ie = 0.0, ke = 0.0;
  for (int64_t z = 0; z < n * n * n; ++z) ie += f[4][z] * f[3][z];
  for (int64_t k = 0; k < nn; ++k)
    for (int64_t j = 0; j < nn; ++j)
      for (int64_t i = 0; i < nn; ++i) {
        double mp = 0.0; /* 1/8 of the masses of the existing zones around the node */
        for (int c = -1; c <= 0; ++c)
          for (int b = -1; b <= 0; ++b)
            for (int a = -1; a <= 0; ++a) {
              const int64_t zi = i + a, zj = j + b, zk = k + c;
              if (zi < 0 || zj < 0 || zk < 0 || zi >= n || zj >= n || zk >= n) continue;
              mp += 0.125 * f[4][(zk * n + zj) * n + zi];
            }
        const int64_t id = (k * nn + j) * nn + i;
        ke += 0.5 * mp * (f[0][id] * f[0][id] + f[1][id] * f[1][id] + f[2][id] * f[2][id]);
      }
  return ie + ke;
}

static int check(int rc, hydro_ctx *h, const char *what) {
  if (rc != HYDRO_OK) {
    fprintf(stderr, "%s: %s (%s)\n", what, hydro_strerror(rc), hydro_last_error(h));
    return 1;
  }
  return 0;
}

int main(int argc, char **argv) {
  const int64_t n = argc > 1 ? atoll(argv[1]) : 32;
  const int cycles = argc > 2 ? atoi(argv[2]) : 100;
  hydro_config cfg;
  hydro_config_default(&cfg);
  cfg.n[0] = cfg.n[1] = cfg.n[2] = n;
  hydro_ctx *h = NULL;
  if (check(hydro_create(&cfg, &h), NULL, "hydro_create")) return 1;
  const size_t nn = (size_t)(n + 1) * (n + 1) * (n + 1), nz = (size_t)n * n * n;
  double *u = malloc(nn * 8), *v = malloc(nn * 8), *w = malloc(nn * 8);
  double *e = malloc(nz * 8), *m = malloc(nz * 8);
  double *out[HYDRO_NFIELDS] = {0};
  out[3] = u; out[4] = v; out[5] = w; out[7] = e; out[12] = m;
  const uint32_t mask = HYDRO_F_U | HYDRO_F_V | HYDRO_F_W | HYDRO_F_E | HYDRO_F_MASS;
  const double *f[5] = {u, v, w, e, m};
  if (check(hydro_get_fields(h, mask, out), h, "hydro_get_fields")) return 1;
  const double E0 = total_energy(n, f);
  hydro_info info;
  if (check(hydro_step(h, cycles, NULL, &info), h, "hydro_step")) return 1;
  if (check(hydro_get_fields(h, mask, out), h, "hydro_get_fields")) return 1;
  const double E1 = total_energy(n, f);
  double mass = 0.0;
  for (size_t z = 0; z < nz; ++z) mass += m[z];
  printf("n=%lld cycles=%lld t=%.9g dt=%.6g mass=%.15g E0=%.15g E=%.15g rel=%.3e\n",
         (long long)n, (long long)info.cycle, info.t, info.dt, mass, E0, E1,
         fabs(E1 - E0) / E0);
  hydro_destroy(h);
  free(u); free(v); free(w); free(e); free(m);
  return fabs(E1 - E0) / E0 <= 1e-10 ? 0 : 2;
}
