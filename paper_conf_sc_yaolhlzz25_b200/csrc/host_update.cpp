// LowDiff+ CPU replica update (Alg. 2 line 12: "M^C_{t+1} <- M^C_t +
// Adam(o_t, G_t)", the in-memory checkpoint kept in host memory). The same IEEE binary32 op
// sequence as the GPU kernels (csrc/plus.cu, csrc/replay.cu): every expression below is evaluated
// left to right with each product and sum rounded once (compiled with -ffp-contract=off and
// -fno-math-errno, so sqrt/div are the correctly rounded SSE/AVX instructions and the loops
// vectorise without changing a bit). Work is split into contiguous chunks over std::threads.
#include <cmath>
#include <cstring>
#include <thread>
#include <vector>

#include "dense_step.h"

namespace lowdiff {
namespace {

inline float bf16_to_f32(uint16_t h) {
  const uint32_t u = (uint32_t)h << 16;
  float f;
  std::memcpy(&f, &u, 4);
  return f;
}

template <int KIND, bool BF16G>
void chunk(const DenseStep& d, float* __restrict__ x, float* __restrict__ m, float* __restrict__ v,
           const void* g, uint64_t a, uint64_t e) {
  const float* gf = static_cast<const float*>(g);
  const uint16_t* gh = static_cast<const uint16_t*>(g);
  for (uint64_t i = a; i < e; ++i) {
    const float gi = BF16G ? bf16_to_f32(gh[i]) : gf[i];
    if (KIND == 2) {                               // Adam (Eq. 1)
      const float mi = d.b1 * m[i] + d.omb1 * gi;
      const float vi = d.b2 * v[i] + d.omb2 * (gi * gi);
      const float den = std::sqrt(vi) * d.isb + d.eps;
      x[i] = x[i] - d.ss * (mi / den);
      m[i] = mi;
      v[i] = vi;
    } else {
      float dd = gi;
      if (d.has_wd) dd = dd + d.wd * x[i];
      if (KIND == 1) {                             // SGD-momentum (torch.optim.SGD conventions)
        const float b = d.init ? d.mu * m[i] + d.omd * dd : dd;
        m[i] = b;
        dd = d.nesterov ? dd + d.mu * b : b;
      }
      x[i] = x[i] - d.lr * dd;
    }
  }
}

template <int KIND>
void run_kind(const DenseStep& d, float* x, float* m, float* v, const void* g, int bf16, uint64_t a,
              uint64_t e) {
  if (bf16) chunk<KIND, true>(d, x, m, v, g, a, e);
  else chunk<KIND, false>(d, x, m, v, g, a, e);
}

}  // namespace

void host_update_run(const DenseStep& d, float* x, float* m, float* v, const void* g, int g_bf16,
                     uint64_t len, int threads) {
  if (threads < 1) threads = 1;
  const uint64_t per = ((len + threads - 1) / threads + 63) & ~(uint64_t)63;
  auto work = [&](uint64_t a, uint64_t e) {
    if (d.kind == 2) run_kind<2>(d, x, m, v, g, g_bf16, a, e);
    else if (d.kind == 1) run_kind<1>(d, x, m, v, g, g_bf16, a, e);
    else run_kind<0>(d, x, m, v, g, g_bf16, a, e);
  };
  std::vector<std::thread> pool;
  for (int t = 1; t < threads; ++t) {
    const uint64_t a = per * t, e = a + per < len ? a + per : len;
    if (a < e) pool.emplace_back(work, a, e);
  }
  work(0, per < len ? per : len);
  for (auto& th : pool) th.join();
}

}  // namespace lowdiff
