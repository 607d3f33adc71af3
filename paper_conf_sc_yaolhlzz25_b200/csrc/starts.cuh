// Window-start index of sorted u32 lists (used by the merge engine and by replay).
#pragma once
#include "common.cuh"
#include "internal.h"

namespace lowdiff {

__device__ __forceinline__ uint64_t list_len(const ListSet& ls, int l) {
  return ls.list[l].d_len ? *ls.list[l].d_len : ls.list[l].len;
}

// starts[l*(num_w+1) + w] = first position e of list l with idx[e] >= lo + w*W (entries below
// lo are skipped); starts[l*(num_w+1) + num_w] = first position with idx >= hi (or len).
// One streaming pass over the entries: entry e writes the windows in (win(e-1), win(e)].
// ebnd (optional, from bounds_kernel): list l's entries in [lo, hi) are [ebnd[2l], ebnd[2l+1]), so
// only they are scanned — a rank coalescing its shard of P gathered (or peer-resident) lists reads
// about 1/P of each list's indices instead of all of them.
template <int W>
__global__ void __launch_bounds__(kThreads) starts_kernel(const __grid_constant__ ListSet ls, uint64_t lo,
                                                          uint64_t hi, uint32_t num_w, uint32_t* starts,
                                                          const uint32_t* __restrict__ ebnd) {
  const int l = blockIdx.y;
  const uint32_t* idx = ls.list[l].idx;
  const uint64_t len = list_len(ls, l);
  const uint64_t e_first = ebnd ? ebnd[2 * l] : 0, e_last = ebnd ? ebnd[2 * l + 1] : len;
  uint32_t* st = starts + (uint64_t)l * (num_w + 1);
  auto win = [&](uint64_t e) -> int64_t {
    if (e >= len) return (int64_t)num_w;
    const uint64_t i = idx[e];
    if (i < lo) return -1;
    if (i >= hi) return (int64_t)num_w;
    return (int64_t)((i - lo) / W);
  };
  // Short runs of windows are written by the entry's own lane; long gaps (sparse lists leave
  // thousands of empty windows between entries) are written by the whole warp, coalesced.
  const int lane = threadIdx.x & 31;
  const uint64_t stride = (uint64_t)gridDim.x * kThreads;
  for (uint64_t e0 = e_first + (uint64_t)blockIdx.x * kThreads + (threadIdx.x & ~31u); e0 <= e_last; e0 += stride) {
    const uint64_t e = e0 + lane;
    int64_t prev = 0, cur = -1;
    if (e <= e_last) {
      prev = (e == 0) ? -1 : win(e - 1);
      cur = win(e);
    }
    const bool longr = cur - prev > 8;
    if (!longr)
      for (int64_t w = prev + 1; w <= cur; ++w) st[w] = (uint32_t)e;
    uint32_t lm = __ballot_sync(0xFFFFFFFFu, longr);
    while (lm) {
      const int src = __ffs(lm) - 1;
      lm &= lm - 1;
      const int64_t from = __shfl_sync(0xFFFFFFFFu, prev, src) + 1;
      const int64_t to = __shfl_sync(0xFFFFFFFFu, cur, src);
      const uint32_t ee = (uint32_t)__shfl_sync(0xFFFFFFFFu, (unsigned long long)e, src);
      for (int64_t w = from + lane; w <= to; w += 32) st[w] = ee;
    }
  }
}

// The same starts table, 4 entries per thread per step with 16-byte loads and 2 steps in flight
// (lists whose idx base is 16-byte aligned, no ebnd): the HBM-bound form for long lists (replay
// records, batch-merge lists). Entry e writes the windows in (win(e-1), win(e)]; e = len writes
// the tail up to num_w. Long gaps are filled by the whole warp, coalesced.
template <int W>
__global__ void __launch_bounds__(kThreads) starts4_kernel(const __grid_constant__ ListSet ls, uint64_t lo,
                                                           uint64_t hi, uint32_t num_w, uint32_t* starts) {
  static_assert((W & (W - 1)) == 0, "W is a power of two");
  constexpr int kLog = __builtin_ctz(W);
  const int l = blockIdx.y;
  const uint32_t* idx = ls.list[l].idx;
  const uint32_t len = (uint32_t)list_len(ls, l);   // < 2^31
  uint32_t* st = starts + (uint64_t)l * (num_w + 1);
  const int lane = threadIdx.x & 31;
  const uint32_t lo32 = (uint32_t)lo, hi32 = (uint32_t)hi;
  auto win_of = [&](uint32_t i) -> int32_t {         // window of an index value (32-bit: n < 2^31)
    if (i < lo32) return -1;
    if (i >= hi32) return (int32_t)num_w;
    return (int32_t)((i - lo32) >> kLog);
  };
  const uint32_t nq = len / 4 + 1;                 // quads; the last (partial) quad carries e = len
  const uint32_t stride = gridDim.x * kThreads;
  for (uint32_t q0 = blockIdx.x * kThreads + (threadIdx.x & ~31u); q0 < nq; q0 += 2 * stride) {
    uint4 v[2];
    uint32_t before[2];
#pragma unroll
    for (int h = 0; h < 2; ++h) {                  // both steps' loads first
      const uint32_t q = q0 + h * stride + lane;
      const uint32_t e = 4 * q;
      v[h] = make_uint4(0u, 0u, 0u, 0u);
      if (q < nq) {
        if (e + 4 <= len) {
          v[h] = *reinterpret_cast<const uint4*>(idx + e);
        } else {
          uint32_t t[4] = {0u, 0u, 0u, 0u};
          for (uint32_t j = 0; j < 4; ++j) if (e + j < len) t[j] = idx[e + j];
          v[h] = make_uint4(t[0], t[1], t[2], t[3]);
        }
      }
      before[h] = (lane == 0 && e > 0 && q < nq) ? idx[e - 1] : 0u;
    }
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      if (q0 + h * stride >= nq) break;            // warp-uniform
      const uint32_t q = q0 + h * stride + lane;
      const uint32_t e = 4 * q;
      const uint32_t up = __shfl_up_sync(0xFFFFFFFFu, v[h].w, 1);
      const uint32_t iv[4] = {v[h].x, v[h].y, v[h].z, v[h].w};
      int32_t wv[5];                               // windows of entries e-1 .. e+3 (num_w at e+j = len)
      wv[0] = (e == 0 || q >= nq) ? -1 : win_of(lane == 0 ? before[h] : up);
#pragma unroll
      for (int j = 0; j < 4; ++j)
        wv[j + 1] = (q >= nq || e + j > len) ? wv[j] : (e + j == len ? (int32_t)num_w : win_of(iv[j]));
      bool longr = false;
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        if (wv[j + 1] - wv[j] > 8) longr = true;
        else for (int32_t w = wv[j] + 1; w <= wv[j + 1]; ++w) st[w] = e + j;
      }
      uint32_t lm = __ballot_sync(0xFFFFFFFFu, longr);
      while (lm) {                                 // long gaps (rare): the whole warp fills them
        const int src = __ffs(lm) - 1;
        lm &= lm - 1;
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          const int32_t from = __shfl_sync(0xFFFFFFFFu, wv[j], src) + 1;
          const int32_t to = __shfl_sync(0xFFFFFFFFu, wv[j + 1], src);
          if (to - from + 1 > 8) {                 // (uniform) this entry's gap
            const uint32_t ee = __shfl_sync(0xFFFFFFFFu, e, src) + j;
            for (int32_t w = from + lane; w <= to; w += 32) st[w] = ee;
          }
        }
      }
    }
  }
}

// ebnd[2l] / ebnd[2l+1] = first position of list l with idx >= lo / idx >= hi (lists strictly
// ascending). One block of 64 threads per list, one warp per bound: a 32-ary search, each round a
// single coalesced probe of 32 positions (about 5 dependent rounds for a list of 3.4 M entries).
static __global__ void __launch_bounds__(64) bounds_kernel(const __grid_constant__ ListSet ls, uint64_t lo, uint64_t hi,
                                                    uint32_t* __restrict__ ebnd) {
  const int l = blockIdx.x, w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t* idx = ls.list[l].idx;
  const uint64_t key = w ? hi : lo;
  uint64_t a = 0, b = list_len(ls, l);     // answer in [a, b]: idx[a-1] < key, idx[b] >= key
  while (a < b) {
    const uint64_t p = a + ((b - a) * (uint64_t)(lane + 1)) / 33;   // in [a, b), non-decreasing in lane
    const uint32_t m = __ballot_sync(0xFFFFFFFFu, (uint64_t)idx[p] >= key);
    const int f = m ? __ffs(m) - 1 : 32;                              // first probe >= key
    const uint64_t nb = __shfl_sync(0xFFFFFFFFu, p, f & 31), na = __shfl_sync(0xFFFFFFFFu, p, (f + 31) & 31);
    if (f < 32) b = nb;
    if (f > 0) a = na + 1;
  }
  if (lane == 0) ebnd[2 * l + w] = (uint32_t)a;
}

}  // namespace lowdiff
