// Checkpointing configuration model (§3.5): Eq. 3 wasted time and the Eq. 5
// optimum (f*, b*), plus the best integer (FCF, B) around it. Host-only fp64 arithmetic.
#include <math.h>

#include "internal.h"

namespace {

bool valid(const lowdiff_config_model* m) {
  if (!m) return false;
  const double v[7] = {m->N, m->M, m->W, m->S, m->T, m->R_F, m->R_D};
  for (double x : v)
    if (!(x > 0.0) || !isfinite(x)) return false;
  return true;
}

// Eq. 3
double wasted(const lowdiff_config_model& m, double f, double b) {
  const double fail = m.N * m.T / m.M;
  return fail * (b / 2.0 + (m.R_F + m.R_D / 2.0 * (1.0 / (f * b) - 1.0))) + m.N * m.T * m.S * f / m.W;
}

}  // namespace

extern "C" lowdiff_status lowdiff_wasted_time(const lowdiff_config_model* m, double f, double b,
                                              double* t_wasted) {
  if (!valid(m)) return lowdiff::fail(LOWDIFF_EINVAL, "wasted_time: model parameters must be > 0 and finite");
  if (!(f > 0.0) || !(b > 0.0) || !isfinite(f) || !isfinite(b) || !t_wasted)
    return lowdiff::fail(LOWDIFF_EINVAL, "wasted_time: f, b must be > 0 and finite, t_wasted non-null");
  *t_wasted = wasted(*m, f, b);
  return LOWDIFF_OK;
}

extern "C" lowdiff_status lowdiff_optimal_config(const lowdiff_config_model* m, double* f_star,
                                                 double* b_star, uint32_t* fcf, uint32_t* batch) {
  if (!valid(m)) return lowdiff::fail(LOWDIFF_EINVAL, "optimal_config: model parameters must be > 0 and finite");
  // Eq. 5
  const double fs = cbrt(m->R_D * m->W * m->W / (4.0 * m->S * m->S * m->M * m->M));
  const double bs = cbrt(2.0 * m->S * m->R_D * m->M / m->W);
  if (f_star) *f_star = fs;
  if (b_star) *b_star = bs;
  if (fcf || batch) {
    // Integer optimum (reading #30): Eq. 3 is convex in FCF = 1/f for fixed b, and its minimum
    // over FCF is convex in b with its minimum at b*, so B is floor/ceil(b*) and, for each B,
    // FCF is floor/ceil of the b = B root of dT/df = 0 (Eq. 4), clamped to FCF >= B.
    double best = INFINITY;
    uint32_t bf = 0, bb = 0;
    const double Bc[2] = {floor(bs) < 1.0 ? 1.0 : floor(bs), ceil(bs) < 1.0 ? 1.0 : ceil(bs)};
    for (double B : Bc) {
      const double FB = sqrt(2.0 * m->S * m->M * B / (m->R_D * m->W));
      const double Fc[2] = {floor(FB) < B ? B : floor(FB), ceil(FB) < B ? B : ceil(FB)};
      for (double F : Fc) {
        if (F > 4294967295.0) continue;
        const double w = wasted(*m, 1.0 / F, B);
        const uint32_t Fu = (uint32_t)F, Bu = (uint32_t)B;
        if (w < best || (w == best && (Fu < bf || (Fu == bf && Bu < bb)))) { best = w; bf = Fu; bb = Bu; }
      }
    }
    if (!isfinite(best)) return lowdiff::fail(LOWDIFF_EINVAL, "optimal_config: no integer configuration in range");
    if (fcf) *fcf = bf;
    if (batch) *batch = bb;
  }
  return LOWDIFF_OK;
}
