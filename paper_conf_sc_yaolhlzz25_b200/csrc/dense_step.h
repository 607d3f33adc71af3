// One dense optimizer step's fp32 scalars (LowDiff+, csrc/plus.cu) and the host replica update
// (csrc/host_update.cpp, plain C++: no CUDA types). Not part of the ABI.
#pragma once
#include <stdint.h>

namespace lowdiff {

struct DenseStep {
  int kind, nesterov, has_wd, init;
  float lr, ss, isb, b1, omb1, b2, omb2, eps, mu, omd, wd;
};

// M^C_{t+1} = M^C_t + Opt(G_t) over [0, len) of host arrays (Alg. 2 line 12), `threads` workers.
void host_update_run(const DenseStep& d, float* x, float* m, float* v, const void* g, int g_bf16,
                     uint64_t len, int threads);

}  // namespace lowdiff
