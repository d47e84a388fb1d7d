// Test infrastructure (tests/test_oracle_sanitizers.py): drives the oracle through every code
// path -- single and uneven multi-domain Sedov, user input, hourglass control, t_stop, the
// EDTMIN and tangled-mesh failures, field output -- in a binary built with AddressSanitizer and
// UndefinedBehaviorSanitizer, so out-of-bounds ghost indexing or UB in the checker
// fails the CPU suite.
#include <cmath>
#include <cstdio>
#include <cstring>
#include <vector>

#include "../../oracle/hydro_oracle.h"

static orc_config base(int64_t n0, int64_t n1, int64_t n2) {
  orc_config c;
  std::memset(&c, 0, sizeof(c));
  c.n[0] = n0; c.n[1] = n1; c.n[2] = n2;
  for (int a = 0; a < 3; ++a) { c.extent[a] = 1.2; c.ndom[a] = 1; }
  c.gamma = 1.4; c.q_lin = 0.5; c.q_quad = 2.0; c.cfl = 0.3; c.c_vol = 0.1;
  c.dt_growth = 1.1; c.dt_max = INFINITY; c.dt_init = INFINITY;
  c.reflect_mask = 0x3f; c.init_kind = ORC_INIT_SEDOV; c.rho0 = 1.0;
  c.sedov_energy = 0.851072 / 8.0;
  return c;
}

static int run(const orc_config &c, int cycles, int expect) {
  orc_ctx *h = nullptr;
  int rc = orc_create(&c, &h);
  if (rc != ORC_OK) return rc == expect ? 0 : 1;
  orc_info info;
  rc = orc_step(h, cycles, &info);
  const int64_t nn = (c.n[0] + 1) * (c.n[1] + 1) * (c.n[2] + 1), nz = c.n[0] * c.n[1] * c.n[2];
  std::vector<std::vector<double>> f(ORC_NFIELDS);
  double *out[ORC_NFIELDS];
  for (int k = 0; k < ORC_NFIELDS; ++k) {
    f[k].assign(k < 6 ? nn : nz, 0.0);
    out[k] = f[k].data();
  }
  orc_get_fields(h, (1u << ORC_NFIELDS) - 1, out);
  orc_destroy(h);
  if (rc != expect) {
    std::printf("status %d, expected %d\n", rc, expect);
    return 1;
  }
  return 0;
}

int main() {
  int bad = 0;
  orc_config c = base(12, 10, 9);
  bad += run(c, 30, ORC_OK);
  // uneven multi-domain cuts incl. 1-zone-thick domains, hourglass on
  int64_t cx[4] = {0, 1, 7, 12}, cy[3] = {0, 5, 10}, cz[3] = {0, 8, 9};
  orc_config d = c;
  d.ndom[0] = 3; d.ndom[1] = 2; d.ndom[2] = 2;
  d.cuts[0] = cx; d.cuts[1] = cy; d.cuts[2] = cz;
  d.hg_coef = 0.03;
  bad += run(d, 30, ORC_OK);
  // user input (perturbed lattice, random-ish velocities), t_stop
  const int n = 6;
  std::vector<double> X[8];
  const int64_t nn = (n + 1) * (n + 1) * (n + 1), nz = n * n * n;
  for (int k = 0; k < 6; ++k) X[k].assign(nn, 0.0);
  X[6].assign(nz, 1.0);
  X[7].assign(nz, 1.0);
  for (int k = 0; k <= n; ++k)
    for (int j = 0; j <= n; ++j)
      for (int i = 0; i <= n; ++i) {
        const int64_t id = (k * (n + 1) + j) * (n + 1) + i;
        X[0][id] = 1.2 * i / n; X[1][id] = 1.2 * j / n; X[2][id] = 1.2 * k / n;
        X[3][id] = (i > 0 && i < n) ? 0.01 * std::sin(3.0 * id) : 0.0;
      }
  orc_config u = base(n, n, n);
  u.init_kind = ORC_INIT_USER;
  for (int k = 0; k < 8; ++k) u.user[k] = X[k].data();
  u.t_stop = 0.05;
  bad += run(u, 1000, ORC_OK);
  // dt collapse floor (reading R23) and a tangled mesh
  orc_config e = base(8, 8, 8);
  e.dt_floor = 1.0;
  bad += run(e, 5, ORC_EDTMIN);
  X[3][(3 * (n + 1) + 3) * (n + 1) + 3] = 1e4;
  u.dt_first = 1e-3;
  u.t_stop = 0.0;
  bad += run(u, 5, ORC_ETANGLED);
  std::printf(bad ? "FAIL\n" : "ok\n");
  return bad;
}
