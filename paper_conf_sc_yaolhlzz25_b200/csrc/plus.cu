// LowDiff+ (§5, Algorithm 2): training without gradient compression. The
// dense, synchronized gradient G_t updates the GPU model (Alg. 2 line 7, M^G_{t+1} = M^G_t +
// Adam(o_t, G_t)) and, after a layer-wise snapshot to host memory, the CPU-resident replica
// (line 12, M^C_{t+1} = M^C_t + Adam(o_t, G_t)) that serves as the in-memory checkpoint.
//
// Both updates execute the SAME IEEE binary32 operation sequence as the replay (DESIGN.md
// readings #16, #18, #19; the oracle's step), so the replica equals the GPU model bit for bit:
//   SGD        d = g (+ wd*x);  momentum: buf = mu*buf + (1-dampening)*d (d on the first step),
//              d = nesterov ? d + mu*buf : buf;  x = x - lr*d
//   Adam       m = b1*m + (1-b1)*g;  v = b2*v + (1-b2)*(g*g);  x = x - ss*(m / (sqrt(v)*isb + eps))
// with ss = fp32(lr / (1 - b1^step)), isb = fp32(1 / sqrt(1 - b2^step)) from the host in double.
//
// GPU: one grid-stride pass, 4 parameters per thread (128-bit loads of x, m, v and of g, fp32 or
// bf16). 28 B of HBM traffic per parameter for Adam with fp32 g; the few IEEE instructions per
// parameter stay far below the ALU ceiling, so the kernel is HBM-bound (no paired fast path).
// Host: the same loop over [0, len) split into contiguous chunks across std::threads, compiled
// (host_update.cpp) without FMA contraction and with IEEE sqrt/div so it vectorises exactly.
#include "common.cuh"
#include "internal.h"

namespace lowdiff {
namespace {

struct DUArgs {
  int kind, nesterov, has_wd, init;
  float lr, ss, isb, b1, omb1, b2, omb2, eps, mu, omd, wd;
  uint64_t len;
};

template <bool BF16G>
__device__ __forceinline__ void load_g(const void* g, uint64_t i, float (&gv)[4]) {
  if constexpr (BF16G) {
    const uint2 u = *reinterpret_cast<const uint2*>(static_cast<const uint16_t*>(g) + i);
    gv[0] = __uint_as_float(u.x << 16); gv[1] = __uint_as_float(u.x & 0xFFFF0000u);
    gv[2] = __uint_as_float(u.y << 16); gv[3] = __uint_as_float(u.y & 0xFFFF0000u);
  } else {
    const float4 t = *reinterpret_cast<const float4*>(static_cast<const float*>(g) + i);
    gv[0] = t.x; gv[1] = t.y; gv[2] = t.z; gv[3] = t.w;
  }
}

template <bool BF16G>
__device__ __forceinline__ float load_g1(const void* g, uint64_t i) {
  if constexpr (BF16G) return __uint_as_float(((uint32_t) static_cast<const uint16_t*>(g)[i]) << 16);
  else return static_cast<const float*>(g)[i];
}

template <int KIND>
__device__ __forceinline__ void step1(const DUArgs& a, float g, float& x, float& m, float& v) {
  if (KIND == LOWDIFF_OPT_ADAM) {
    m = __fadd_rn(__fmul_rn(a.b1, m), __fmul_rn(a.omb1, g));
    v = __fadd_rn(__fmul_rn(a.b2, v), __fmul_rn(a.omb2, __fmul_rn(g, g)));
    const float den = __fadd_rn(__fmul_rn(__fsqrt_rn(v), a.isb), a.eps);
    x = __fsub_rn(x, __fmul_rn(a.ss, __fdiv_rn(m, den)));
  } else {
    float d = g;
    if (a.has_wd) d = __fadd_rn(d, __fmul_rn(a.wd, x));
    if (KIND == LOWDIFF_OPT_MOMENTUM) {
      m = a.init ? __fadd_rn(__fmul_rn(a.mu, m), __fmul_rn(a.omd, d)) : d;
      d = a.nesterov ? __fadd_rn(d, __fmul_rn(a.mu, m)) : m;
    }
    x = __fsub_rn(x, __fmul_rn(a.lr, d));
  }
}

template <int KIND, bool BF16G>
__global__ void __launch_bounds__(kThreads) dense_update_kernel(const DUArgs a, const void* __restrict__ g,
                                                                float* __restrict__ X, float* __restrict__ M,
                                                                float* __restrict__ V) {
  const uint64_t n4 = a.len / 4;
  const uint64_t stride = (uint64_t)gridDim.x * kThreads;
  for (uint64_t q = (uint64_t)blockIdx.x * kThreads + threadIdx.x; q < n4; q += stride) {
    const uint64_t i = q * 4;
    float gv[4], x[4], m[4] = {0, 0, 0, 0}, v[4] = {0, 0, 0, 0};
    load_g<BF16G>(g, i, gv);
    float4 t = *reinterpret_cast<const float4*>(X + i);
    x[0] = t.x; x[1] = t.y; x[2] = t.z; x[3] = t.w;
    if (KIND != LOWDIFF_OPT_SGD) {
      t = *reinterpret_cast<const float4*>(M + i);
      m[0] = t.x; m[1] = t.y; m[2] = t.z; m[3] = t.w;
    }
    if (KIND == LOWDIFF_OPT_ADAM) {
      t = *reinterpret_cast<const float4*>(V + i);
      v[0] = t.x; v[1] = t.y; v[2] = t.z; v[3] = t.w;
    }
#pragma unroll
    for (int p = 0; p < 4; ++p) step1<KIND>(a, gv[p], x[p], m[p], v[p]);
    *reinterpret_cast<float4*>(X + i) = make_float4(x[0], x[1], x[2], x[3]);
    if (KIND != LOWDIFF_OPT_SGD) *reinterpret_cast<float4*>(M + i) = make_float4(m[0], m[1], m[2], m[3]);
    if (KIND == LOWDIFF_OPT_ADAM) *reinterpret_cast<float4*>(V + i) = make_float4(v[0], v[1], v[2], v[3]);
  }
  // ragged tail (len % 4), one thread per element
  const uint64_t i = n4 * 4 + (uint64_t)blockIdx.x * kThreads + threadIdx.x;
  if (i < a.len) {
    float x = X[i], m = KIND != LOWDIFF_OPT_SGD ? M[i] : 0.f, v = KIND == LOWDIFF_OPT_ADAM ? V[i] : 0.f;
    step1<KIND>(a, load_g1<BF16G>(g, i), x, m, v);
    X[i] = x;
    if (KIND != LOWDIFF_OPT_SGD) M[i] = m;
    if (KIND == LOWDIFF_OPT_ADAM) V[i] = v;
  }
}

template <int KIND>
void launch_du(const DUArgs& a, const void* g, bool bf16, lowdiff_state* st, cudaStream_t s) {
  uint64_t grid = (a.len / 4 + kThreads - 1) / kThreads;
  if (grid > 8ull * kNumSMs) grid = 8ull * kNumSMs;
  if (grid == 0) grid = 1;
  if (bf16)
    LD_LAUNCH("dense_update", s, (dense_update_kernel<KIND, true>), (int)grid, kThreads, 0, a, g, st->x, st->m,
              st->v);
  else
    LD_LAUNCH("dense_update", s, (dense_update_kernel<KIND, false>), (int)grid, kThreads, 0, a, g, st->x, st->m,
              st->v);
}

}  // namespace

// Host scalars of one step (advances st->adam_step / momentum_initialized / t), shared by the
// GPU and host updates so both use the same fp32 constants.
void dense_update_scalars(lowdiff_state* st, const lowdiff_opt* o, float lr, DenseStep* d) {
  d->kind = o->kind;
  d->nesterov = o->nesterov;
  d->has_wd = o->weight_decay != 0.0;
  d->init = st->momentum_initialized;
  d->lr = lr;
  d->b1 = (float)o->beta1; d->omb1 = (float)(1.0 - o->beta1);
  d->b2 = (float)o->beta2; d->omb2 = (float)(1.0 - o->beta2);
  d->eps = (float)o->eps;
  d->mu = (float)o->momentum; d->omd = (float)(1.0 - o->dampening);
  d->wd = (float)o->weight_decay;
  d->ss = d->isb = 0.f;
  if (o->kind == LOWDIFF_OPT_ADAM) {
    st->adam_step += 1;
    const double step = (double)st->adam_step;
    d->ss = (float)((double)lr / (1.0 - pow(o->beta1, step)));
    d->isb = (float)(1.0 / sqrt(1.0 - pow(o->beta2, step)));
  }
  if (o->kind == LOWDIFF_OPT_MOMENTUM) st->momentum_initialized = 1;
  st->t += 1;
}

lowdiff_status dense_update_run(lowdiff_state* st, const lowdiff_opt* o, const void* grad, int gdt, float lr,
                                cudaStream_t s) {
  DenseStep d;
  dense_update_scalars(st, o, lr, &d);
  DUArgs a;
  a.kind = d.kind; a.nesterov = d.nesterov; a.has_wd = d.has_wd; a.init = d.init;
  a.lr = d.lr; a.ss = d.ss; a.isb = d.isb; a.b1 = d.b1; a.omb1 = d.omb1; a.b2 = d.b2; a.omb2 = d.omb2;
  a.eps = d.eps; a.mu = d.mu; a.omd = d.omd; a.wd = d.wd;
  a.len = st->hi - st->lo;
  const bool bf = gdt == LOWDIFF_BF16;
  if (o->kind == LOWDIFF_OPT_ADAM) launch_du<LOWDIFF_OPT_ADAM>(a, grad, bf, st, s);
  else if (o->kind == LOWDIFF_OPT_MOMENTUM) launch_du<LOWDIFF_OPT_MOMENTUM>(a, grad, bf, st, s);
  else launch_du<LOWDIFF_OPT_SGD>(a, grad, bf, st, s);
  return cuda_status(cudaGetLastError(), "dense_update launch");
}

}  // namespace lowdiff
