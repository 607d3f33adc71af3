// Multiway index merge engine (sm_100a) — serves two steps of the path:
//   * coalesce after the sparse all-gather: Sync(G~_{i,t}) (Alg.1 line 5)
//       P rank lists -> sorted unique union in [lo, hi), rank-ascending fp32 fold, / P
//   * batch merge of B differentials (§4.2 Step 2; "tensor addition or dictionary
//       accumulation") -> one record (SUM: iteration-ascending fold; STACK: per-index
//       iteration lists)
//
// Sort-free design: the index range [lo, hi) is cut into windows of W = 4096
// consecutive parameter indices. K2a writes, for every list, the position of each window's first
// entry (one streaming pass over the entries). K2b is a persistent, ticket-ordered kernel: one
// CTA takes one window, folds the lists' entries of that window into a dense W-slot
// shared-memory accumulator IN LIST ORDER (so the fp32 fold order is the definition's, with no
// float atomics), compacts the occupied slots in index order, and finds its global output offset
// with a decoupled look-back. The merge writes sections into the workspace; K2c packs them into
// the byte-exact record (header | lr[] | idx | val  or  off | it | val, 16-byte aligned).
#include "common.cuh"
#include "internal.h"
#include "starts.cuh"

namespace lowdiff {
namespace {

constexpr int kW = 4096;                    // parameter indices per window
constexpr int kSlotsPerThread = kW / kThreads;

struct __align__(256) MCtl {
  uint32_t ticket;
  uint32_t pad;
  uint64_t nnz;      // unique indices (written by the last window)
  uint64_t nent;     // entries (STACK) (written by the last window)
};

struct MLayout {
  uint64_t ctl, status, zero_end, starts, widx, wval, woff, wit, went, total;
  uint32_t num_w;
};

MLayout mlayout(int L, uint64_t max_entries, uint64_t lo, uint64_t hi, bool record) {
  MLayout M;
  M.num_w = (uint32_t)((hi - lo + kW - 1) / kW);
  const uint64_t cap_u = max_entries < hi - lo ? max_entries : hi - lo;
  uint64_t o = 0;
  M.ctl = o;    o += align256(sizeof(MCtl));
  M.status = o; o += align256(8ull * M.num_w);
  M.zero_end = o;
  M.starts = o; o += align256(4ull * L * (M.num_w + 1));
  M.widx = M.wval = M.woff = M.wit = M.went = 0;
  if (record) {
    M.widx = o; o += align256(4 * cap_u);
    M.wval = o; o += align256(4 * cap_u);         // SUM values, or STACK off[] (u32)
    M.woff = M.wval;
    M.wit = o;  o += align256(max_entries);
    M.went = o; o += align256(4 * max_entries);
  }
  M.total = o;
  return M;
}

template <bool BF16>
__device__ __forceinline__ float list_val(const ListSet& ls, int l, uint64_t e) {
  if constexpr (BF16)
    return __uint_as_float(((uint32_t) static_cast<const uint16_t*>(ls.list[l].val)[e]) << 16);
  else
    return static_cast<const float*>(ls.list[l].val)[e];
}

// ---- K2b: window merge --------------------------------------------------------------------------
template <int KIND, bool BF16>
__global__ void __launch_bounds__(kThreads) window_kernel(const __grid_constant__ ListSet ls, uint64_t lo,
                                                          uint64_t hi, uint32_t num_w,
                                                          const uint32_t* __restrict__ starts,
                                                          MCtl* ctl, uint64_t* status, int average,
                                                          uint32_t* __restrict__ out_idx,
                                                          float* __restrict__ out_val,
                                                          uint64_t* d_out_nnz,
                                                          uint8_t* __restrict__ out_it,
                                                          float* __restrict__ out_ent) {
  __shared__ float s_acc[kW];                 // SUM: running fold; STACK: slot entry cursor (u32)
  __shared__ uint32_t s_cnt[kW];              // entries per slot (lists present)
  __shared__ uint32_t s_beg[kMaxLists], s_end[kMaxLists];
  __shared__ uint64_t s_scan[kThreads / 32];
  __shared__ uint64_t s_base;
  __shared__ uint32_t s_ticket;
  const int tid = threadIdx.x;
  const int L = ls.L;
  const float fP = (float)L;
  for (int j = tid; j < kW; j += kThreads) s_cnt[j] = 0;
  while (true) {
    if (tid == 0) s_ticket = atomicAdd(&ctl->ticket, 1u);
    __syncthreads();
    const uint32_t w = s_ticket;
    if (w >= num_w) break;
    const uint64_t w0 = lo + (uint64_t)w * kW;
    int nonempty = 0;
    for (int l = tid; l < L; l += kThreads) {
      const uint32_t b = starts[(uint64_t)l * (num_w + 1) + w];
      const uint32_t e = starts[(uint64_t)l * (num_w + 1) + w + 1];
      s_beg[l] = b; s_end[l] = e;
      nonempty |= (e > b);
    }
    nonempty = __syncthreads_or(nonempty);
    uint64_t my_u = 0, my_e = 0, local = 0;
    if (nonempty) {
      if (KIND == kMergeStack) {
        for (int l = 0; l < L; ++l)                     // integer counts: order-free
          for (uint32_t e = s_beg[l] + tid; e < s_end[l]; e += kThreads)
            atomicAdd(&s_cnt[ls.list[l].idx[e] - w0], 1u);
      } else {
        for (int l = 0; l < L; ++l) {                   // fp32 fold in list (rank/iteration) order
          if (s_end[l] == s_beg[l]) continue;           // block-uniform
          for (uint32_t e = s_beg[l] + tid; e < s_end[l]; e += kThreads) {
            const uint32_t slot = ls.list[l].idx[e] - (uint32_t)w0;
            const float v = list_val<BF16>(ls, l, e);
            const uint32_t c = s_cnt[slot];
            s_acc[slot] = c ? s_acc[slot] + v : v;
            s_cnt[slot] = c + 1;
          }
          __syncthreads();
        }
      }
      __syncthreads();
#pragma unroll
      for (int j = 0; j < kSlotsPerThread; ++j) {
        const uint32_t c = s_cnt[tid * kSlotsPerThread + j];
        my_u += c ? 1 : 0;
        my_e += c;
      }
      uint64_t tot;
      local = block_exclusive_scan((my_u << 31) | my_e, s_scan, &tot);
      if (tid < 32) {
        const uint64_t pre = lookback_exclusive(status, w, tot);
        if (tid == 0) s_base = pre;
      }
    } else {
      if (tid < 32) {
        const uint64_t pre = lookback_exclusive(status, w, 0);
        if (tid == 0) s_base = pre;
      }
    }
    __syncthreads();
    const uint64_t base = s_base;
    if (nonempty) {
      uint64_t u = (base >> 31) + (local >> 31);
      uint64_t e = (base & 0x7FFFFFFFull) + (local & 0x7FFFFFFFull);
#pragma unroll 4
      for (int j = 0; j < kSlotsPerThread; ++j) {
        const int slot = tid * kSlotsPerThread + j;
        const uint32_t c = s_cnt[slot];
        if (!c) continue;
        out_idx[u] = (uint32_t)(w0 + slot);
        if (KIND == kMergeStack) {
          reinterpret_cast<uint32_t*>(out_val)[u] = (uint32_t)e;      // off[u]
          reinterpret_cast<uint32_t*>(s_acc)[slot] = (uint32_t)e;     // entry cursor
        } else {
          const float s = s_acc[slot];
          out_val[u] = average ? __fdiv_rn(s, fP) : s;
        }
        ++u;
        e += c;
      }
      if (KIND == kMergeStack) {
        __syncthreads();
        for (int l = 0; l < L; ++l) {                   // entries in iteration order per slot
          if (s_end[l] == s_beg[l]) continue;
          for (uint32_t x = s_beg[l] + tid; x < s_end[l]; x += kThreads) {
            const uint32_t slot = ls.list[l].idx[x] - (uint32_t)w0;
            const uint32_t pos = reinterpret_cast<uint32_t*>(s_acc)[slot];
            out_it[pos] = (uint8_t)l;
            out_ent[pos] = list_val<BF16>(ls, l, x);
            reinterpret_cast<uint32_t*>(s_acc)[slot] = pos + 1;
          }
          __syncthreads();
        }
      }
      if (tid == kThreads - 1 && w == num_w - 1) {
        ctl->nnz = u;
        ctl->nent = e;
        if (d_out_nnz) *d_out_nnz = u;
      }
#pragma unroll
      for (int j = 0; j < kSlotsPerThread; ++j) s_cnt[tid * kSlotsPerThread + j] = 0;
    } else if (tid == 0 && w == num_w - 1) {
      ctl->nnz = base >> 31;
      ctl->nent = base & 0x7FFFFFFFull;
      if (d_out_nnz) *d_out_nnz = base >> 31;
    }
    __syncthreads();
  }
}

// ---- K2c: record packer ---------------------------------------------------------------------
struct PackArgs {
  uint32_t mode, B, nranks;
  uint64_t n, lo, hi, t_first, cap;
  float lr[256];
};

__global__ void __launch_bounds__(kThreads) pack_kernel(const __grid_constant__ PackArgs a, const MCtl* ctl,
                                                        const uint32_t* __restrict__ widx,
                                                        const uint32_t* __restrict__ wval,
                                                        const uint8_t* __restrict__ wit,
                                                        const uint32_t* __restrict__ went,
                                                        uint8_t* __restrict__ rec, uint64_t* d_bytes) {
  const uint64_t nnz = ctl->nnz, nent = (a.mode == LOWDIFF_MERGE_SUM) ? ctl->nnz : ctl->nent;
  const uint64_t o_lr = 80, o_idx = o_lr + pad16(4ull * a.B), o_v = o_idx + pad16(4 * nnz);
  uint64_t o_it = 0, o_ent = 0, total;
  if (a.mode == LOWDIFF_MERGE_SUM) {
    total = o_v + pad16(4 * nnz);
  } else {
    o_it = o_v + pad16(4 * (nnz + 1));
    o_ent = o_it + pad16(nent);
    total = o_ent + pad16(4 * nent);
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) *d_bytes = total;
  if (total > a.cap) return;
  const uint64_t chunks = total / 16;
  for (uint64_t c = (uint64_t)blockIdx.x * kThreads + threadIdx.x; c < chunks;
       c += (uint64_t)gridDim.x * kThreads) {
    const uint64_t off = c * 16;
    uint32_t wd[4];
    if (off < o_lr) {                          // header
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const int word = (int)(off / 4) + q;
        uint32_t v = 0;
        switch (word) {
          case 0: v = 0x44574F4Cu; break;        // "LOWD"
          case 1: v = 0x01464649u; break;        // "IFF\x01"
          case 2: v = 1; break;
          case 3: v = a.mode; break;
          case 4: v = a.B; break;
          case 5: v = a.nranks; break;
          case 6: v = (uint32_t)a.n; break;          case 7: v = (uint32_t)(a.n >> 32); break;
          case 8: v = (uint32_t)a.lo; break;         case 9: v = (uint32_t)(a.lo >> 32); break;
          case 10: v = (uint32_t)a.hi; break;        case 11: v = (uint32_t)(a.hi >> 32); break;
          case 12: v = (uint32_t)a.t_first; break;   case 13: v = (uint32_t)(a.t_first >> 32); break;
          case 14: v = (uint32_t)nnz; break;         case 15: v = (uint32_t)(nnz >> 32); break;
          case 16: v = (uint32_t)nent; break;        case 17: v = (uint32_t)(nent >> 32); break;
          case 18: v = (uint32_t)total; break;       case 19: v = (uint32_t)(total >> 32); break;
        }
        wd[q] = v;
      }
    } else if (off < o_idx) {                  // lr[B]
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const uint64_t j = (off - o_lr) / 4 + q;
        wd[q] = j < a.B ? __float_as_uint(a.lr[j]) : 0u;
      }
    } else if (off < o_v) {                    // idx[nnz]
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const uint64_t j = (off - o_idx) / 4 + q;
        wd[q] = j < nnz ? widx[j] : 0u;
      }
    } else if (a.mode == LOWDIFF_MERGE_SUM || off < o_it) {   // SUM val[nnz] / STACK off[nnz+1]
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const uint64_t j = (off - o_v) / 4 + q;
        if (a.mode == LOWDIFF_MERGE_SUM) wd[q] = j < nnz ? wval[j] : 0u;
        else wd[q] = j < nnz ? wval[j] : (j == nnz ? (uint32_t)nent : 0u);
      }
    } else if (off < o_ent) {                  // it[nent] (u8)
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        uint32_t v = 0;
#pragma unroll
        for (int b = 0; b < 4; ++b) {
          const uint64_t j = (off - o_it) + 4 * q + b;
          v |= (j < nent ? (uint32_t)wit[j] : 0u) << (8 * b);
        }
        wd[q] = v;
      }
    } else {                                   // STACK val[nent]
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const uint64_t j = (off - o_ent) / 4 + q;
        wd[q] = j < nent ? went[j] : 0u;
      }
    }
    *reinterpret_cast<uint4*>(rec + off) = make_uint4(wd[0], wd[1], wd[2], wd[3]);
  }
}

}  // namespace

uint64_t merge_ws_bytes(int L, uint64_t max_entries, uint64_t lo, uint64_t hi) {
  return mlayout(L, max_entries, lo, hi, true).total;
}

lowdiff_status merge_run(const ListSet& ls, MergeKind kind, uint64_t lo, uint64_t hi, int average,
                         uint64_t max_entries, uint32_t* out_idx, float* out_val, uint64_t out_cap,
                         uint64_t* d_out_nnz, const float* lr, uint64_t n, uint64_t t_first,
                         uint32_t nranks, void* d_record, uint64_t record_cap,
                         uint64_t* d_record_bytes, void* ws, cudaStream_t s) {
  (void)out_cap;
  const bool record = kind != kCoalesce;
  const MLayout M = mlayout(ls.L, max_entries, lo, hi, record);
  uint8_t* w = static_cast<uint8_t*>(ws);
  MCtl* ctl = reinterpret_cast<MCtl*>(w + M.ctl);
  uint64_t* status = reinterpret_cast<uint64_t*>(w + M.status);
  uint32_t* starts = reinterpret_cast<uint32_t*>(w + M.starts);
  LD_CUDA(cudaMemsetAsync(w, 0, M.zero_end, s), "memset merge workspace");

  uint64_t per_list = max_entries / (ls.L ? ls.L : 1) + 1;
  uint64_t gx = (per_list + kThreads - 1) / kThreads;
  if (gx > 512) gx = 512;
  if (gx < 1) gx = 1;
  LD_LAUNCH("starts", s, starts_kernel<kW>, dim3((unsigned)gx, (unsigned)ls.L), kThreads, 0, ls, lo, hi,
            M.num_w, starts);

  const int grid = (int)(M.num_w < 4u * kNumSMs ? M.num_w : 4u * kNumSMs);
  uint32_t* oidx = record ? reinterpret_cast<uint32_t*>(w + M.widx) : out_idx;
  float* oval = record ? reinterpret_cast<float*>(w + M.wval) : out_val;
  uint8_t* oit = record ? w + M.wit : nullptr;
  float* oent = record ? reinterpret_cast<float*>(w + M.went) : nullptr;
  const char* cls = record ? "merge" : "coalesce";
  if (kind == kCoalesce) {
    if (ls.bf16)
      LD_LAUNCH(cls, s, (window_kernel<kCoalesce, true>), grid, kThreads, 0, ls, lo, hi, M.num_w,
                starts, ctl, status, average, oidx, oval, d_out_nnz, oit, oent);
    else
      LD_LAUNCH(cls, s, (window_kernel<kCoalesce, false>), grid, kThreads, 0, ls, lo, hi, M.num_w,
                starts, ctl, status, average, oidx, oval, d_out_nnz, oit, oent);
    return cuda_status(cudaGetLastError(), "coalesce launch");
  }
  if (kind == kMergeSum)
    LD_LAUNCH(cls, s, (window_kernel<kMergeSum, false>), grid, kThreads, 0, ls, lo, hi, M.num_w,
              starts, ctl, status, 0, oidx, oval, nullptr, oit, oent);
  else
    LD_LAUNCH(cls, s, (window_kernel<kMergeStack, false>), grid, kThreads, 0, ls, lo, hi, M.num_w,
              starts, ctl, status, 0, oidx, oval, nullptr, oit, oent);

  PackArgs pa;
  pa.mode = kind == kMergeSum ? LOWDIFF_MERGE_SUM : LOWDIFF_MERGE_STACK;
  pa.B = (uint32_t)ls.L;
  pa.nranks = nranks;
  pa.n = n; pa.lo = lo; pa.hi = hi; pa.t_first = t_first; pa.cap = record_cap;
  for (int j = 0; j < 256; ++j) pa.lr[j] = j < ls.L ? lr[j] : 0.f;
  const uint64_t est = lowdiff_record_max_bytes((lowdiff_merge_mode)pa.mode, pa.B, max_entries) / 16;
  uint64_t pg = (est + kThreads - 1) / kThreads;
  if (pg > 8ull * kNumSMs) pg = 8ull * kNumSMs;
  if (pg < 1) pg = 1;
  LD_LAUNCH("merge_pack", s, pack_kernel, (int)pg, kThreads, 0, pa, ctl,
            reinterpret_cast<const uint32_t*>(w + M.widx), reinterpret_cast<const uint32_t*>(w + M.wval),
            w + M.wit, reinterpret_cast<const uint32_t*>(w + M.went), static_cast<uint8_t*>(d_record),
            d_record_bytes);
  return cuda_status(cudaGetLastError(), "merge launch");
}

}  // namespace lowdiff
