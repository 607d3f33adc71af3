// lowdiff_compress — Comp(G_{i,t}) (Alg.1 line 4): exact top-k of |g + r| with
// error feedback, on sm_100a.
//
// Design: the only HBM-heavy step is one fused streaming pass
//   a = g + r;  r <- a;  if |a| >= T: append (i, a) to a candidate buffer
// which moves the algorithmic floor of 12n bytes (fp32 g) / 10n (bf16 g). The candidate threshold
// T comes from the previous call's exact k-th key K*_prev, lowered by an adaptive margin delta
// (persistent per-residual state kept in the workspace; a hint only — the result never depends on
// it): in error-feedback steady state the k-th key moves by a fraction of a percent per iteration,
// while the key density right below it piles up (every unselected element keeps accumulating
// until it crosses the threshold), so a sampled estimate with a few percent of resolution is not
// accurate enough there (305 of 1300 C3 calls fell back with the sample alone).
// One cooperative kernel then does the rest: an exact 3-digit radix select (12/10/9 bits of the
// 31-bit key) over the candidates finds K* and the number m of K*-ties to keep, and an ordered
// emission (per-tile counts, a scan over tiles, ballot prefixes inside each tile) writes the k
// pairs in ascending index order and fixes r on S.
// Recovery, all inside the same select launch (no host round trip):
//   * fewer than k candidates (the first call on a residual, or K* dropped by more than delta):
//     a stratified sample of |g + r| gives a lower threshold T2;
//   * more than the capacity: the stream pass's exact first-digit histogram of ALL candidates
//     gives T2 = the lower edge of the k-th key's bin;
//   then one rescan of the residual (4n bytes read; the first pass's recorded candidates are
//   overlaid from the buffer) rebuilds the candidate set at T2. Only if that also misses does the
//   exact full-array select run (~3 x 4n bytes). Every path gives the same bytes; the per-call path
//   and counters are reported through lowdiff_compress_counters.
// Nothing on this path is a dense contraction: no tensor cores.
#include <stdio.h>

#include <cooperative_groups.h>

#include "common.cuh"
#include "internal.h"

namespace cg = cooperative_groups;

namespace lowdiff {
namespace {

constexpr int kTile = 4096;            // elements per streaming tile: 256 thr x 4 vectors x 4
constexpr int kMaxSelectBlocks = 4 * 148;
constexpr int kSmallThreads = 1024;             // small select: one CTA
constexpr uint32_t kSmallMaxCand = 1u << 15;    // candidate counts it takes (above: the grid kernel)
constexpr uint32_t kNoForce = 0xFFFFFFFFu;
// digit p = (key >> shift(p)) & (bins(p) - 1): 12 + 10 + 9 bits of the 31-bit key
__host__ __device__ constexpr int bins(int p) { return p == 0 ? 4096 : (p == 1 ? 1024 : 512); }
__host__ __device__ constexpr int shift(int p) { return p == 0 ? 19 : (p == 1 ? 9 : 0); }
constexpr uint32_t kMaxChunks = 4096;            // fast select: chunks of tiles with a kept count each

// Persistent per-residual state (the first 256 bytes of the workspace; never cleared by a call).
// It is valid only for the (n, k, residual, dtypes) it was written for; anything else (a fresh or
// reused workspace) reads as "cold" and the call takes the recovery path once.
constexpr uint64_t kStateMagic = 0x4C44435354415445ull;   // "LDCSTATE"
struct __align__(256) State {
  uint64_t magic, n, k, resid, tag;
  uint32_t kstar;           // the previous call's exact k-th key
  float delta;              // relative margin below it for the next threshold
  uint64_t calls, rescans, fallbacks, nonfinite_calls, last_nonfinite, fast_calls;
  uint32_t last_cand, last_path;
};
struct StateKey {
  uint64_t n, k, resid, tag;
  float band_lo, band_hi;   // the margin controller's target band of first-pass candidates / k
};
constexpr float kDeltaInit = 1.0f / 64, kDeltaMin = 1.0f / 8192, kDeltaMax = 0.5f;

struct __align__(256) Ctl {
  uint32_t t_est;          // the first pass's threshold: candidates have key >= t_est
  uint32_t mode;           // path: 0/3 = first-pass candidates (3: fast select), 2 = rescan, 1 = full array
  uint32_t cand_count;     // candidates found by the streaming pass (may exceed capacity)
  uint32_t cand_count2;    // candidates found by the rescan
  uint32_t t2;             // the rescan's threshold
  uint32_t prefix;
  uint32_t kstar;          // the k-th largest key
  uint32_t small_done;     // the one-CTA select did this call (the grid kernel then returns)
  uint32_t fine_shift;     // the first pass's candidate histogram: bin = min((key - t_est) >> fine_shift, 4095)
  uint32_t nonfinite;      // elements with |a| = Inf or NaN (the streaming pass sees every a)
  uint32_t inbin_count;    // fast select: candidates in the k-th key's fine bin
  uint64_t m;              // K*-ties to keep (lowest indices first)
};

struct Layout {
  uint64_t state, ctl, hs, hc, hc2, h0, h1, h2, hl, ctot, zero_end, tiles, tiles2, cand_idx, cand_val, cand2_idx,
      cand2_val, tloc, tk, bits, inbin, boff, seg, pj, total;
  uint32_t num_tiles, cap;
};

Layout layout(uint64_t n, uint64_t k) {
  Layout L;
  L.num_tiles = (uint32_t)((n + kTile - 1) / kTile);
  uint64_t cap = 8 * k + 65536;
  L.cap = (uint32_t)(cap < n ? cap : n);
  uint64_t o = 0;
  L.state = o;    o += align256(sizeof(State));
  L.ctl = o;      o += align256(sizeof(Ctl));
  L.hs = o;       o += align256(4u * bins(0));   // sample (recovery)
  L.hc = o;       o += align256(4u * bins(0));   // first-pass candidates' fine bins (relative to T)
  L.hc2 = o;      o += align256(4u * bins(0));   // rescan candidates' first digit
  L.h0 = o;       o += align256(4u * bins(0));
  L.h1 = o;       o += align256(4u * bins(1));
  L.h2 = o;       o += align256(4u * bins(2));
  L.hl = o;       o += align256(4u * bins(0));
  L.ctot = o;     o += align256(8u * kMaxChunks);
  L.zero_end = o;
  L.tiles = o;    o += align256(8ull * L.num_tiles);
  L.tiles2 = o;   o += align256(8ull * L.num_tiles);
  L.cand_idx = o; o += align256(4ull * L.cap);
  L.cand_val = o; o += align256(4ull * L.cap);
  L.cand2_idx = o; o += align256(4ull * L.cap);
  L.cand2_val = o; o += align256(4ull * L.cap);
  L.tloc = o;     o += align256(8ull * L.num_tiles);   // per-tile (gt, eq) counts, then their scan
  L.tk = o;       o += align256(8ull * L.num_tiles);   // fast select: (>, ==) counts per tile
  L.bits = o;     o += align256(8ull * (L.cap / 32 + 1));   // fast select: (>, ==) bits per position
  L.inbin = o;    o += align256(8ull * L.cap);         // fast select: the undecided (position, value)
  L.boff = o;     o += align256(8ull * 3 * kMaxSelectBlocks);
  L.seg = o;      o += align256(16ull * L.num_tiles);  // small select: P at each tile's segment ends
  L.pj = o;       o += align256(8ull * (L.cap < kSmallMaxCand ? L.cap : kSmallMaxCand));   // P per position
  L.total = o;
  return L;
}

// ---- loads ----------------------------------------------------------------------------------
template <bool BF16>
__device__ __forceinline__ float4 load_g4(const void* g, uint64_t i) {   // i % 4 == 0
  if constexpr (BF16) {
    uint2 u = ld_stream_u2(reinterpret_cast<const uint2*>(static_cast<const uint16_t*>(g) + i));
    return make_float4(__uint_as_float(u.x << 16), __uint_as_float(u.x & 0xFFFF0000u),
                       __uint_as_float(u.y << 16), __uint_as_float(u.y & 0xFFFF0000u));
  } else {
    return ld_stream_f4(reinterpret_cast<const float4*>(static_cast<const float*>(g) + i));
  }
}
template <bool BF16>
__device__ __forceinline__ float load_g1(const void* g, uint64_t i) {
  if constexpr (BF16) return __uint_as_float(((uint32_t) static_cast<const uint16_t*>(g)[i]) << 16);
  else return static_cast<const float*>(g)[i];
}

// ---- threshold state ------------------------------------------------------------------------
__device__ __forceinline__ bool state_valid(const State* st, const StateKey& sk) {
  return st->magic == kStateMagic && st->n == sk.n && st->k == sk.k && st->resid == sk.resid &&
         st->tag == sk.tag;
}
// The first pass's threshold: K*_prev lowered by delta (in magnitude); "no candidates" when cold.
__device__ __forceinline__ uint32_t pass1_threshold(const State* st, const StateKey& sk, uint32_t force_t) {
  if (force_t != kNoForce) return force_t;                 // test hook
  if (!state_valid(st, sk)) return 0xFFFFFFFFu;           // cold: every key is below it
  const uint32_t K = st->kstar;
  if (K >= 0x7F800000u) return 0x7F800000u;               // non-finite k-th key: keep them all
  const float t = __uint_as_float(K) * (1.0f - st->delta);
  return __float_as_uint(t) & 0x7FFFFFFFu;
}
// The first pass's candidate histogram is relative to T: bin = min((key - T) >> s, 4095), with s
// the smallest shift whose bins 0..4094 reach K*_prev (1 + 2 delta): around the expected k-th key
// the bins are a few key units wide, so the select finds K* with one pass over the candidates.
// Cold or forced thresholds use s = 19 (the bins then cover every key >= T).
__device__ __forceinline__ uint32_t fine_shift(const State* st, const StateKey& sk, uint32_t T, uint32_t force_t) {
  if (force_t != kNoForce || !state_valid(st, sk)) return 19;
  const uint32_t K = st->kstar;
  if (K >= 0x7F800000u || T >= 0x7F800000u) return 19;
  uint32_t top = __float_as_uint(__uint_as_float(K) * (1.0f + 2.0f * st->delta)) & 0x7FFFFFFFu;
  if (top >= 0x7F800000u) top = 0x7F7FFFFFu;
  const uint64_t range = top > T ? top - T : 1;
  uint32_t sh = 0;
  while (sh < 19 && (4095ull << sh) < range) ++sh;
  return sh;
}
__device__ __forceinline__ uint32_t fine_bin(uint32_t key, uint32_t T, uint32_t s) {   // key >= T
  const uint32_t d = (key - T) >> s;
  return d < 4095u ? d : 4095u;
}

// After the select (one thread): counters, and the margin controller on the first pass's
// candidate count: fewer than k -> widen, above the capacity -> narrow, else aim at the band
// (1.05-1.5 k by default: fewer candidates make the select cheaper, scripts/band_sweep.sh).
__device__ void state_update(State* st, const StateKey& sk, uint64_t k, uint32_t cap, uint32_t cc,
                             uint32_t path, uint32_t kstar, uint64_t nonfinite) {
  const bool warm = state_valid(st, sk);
  if (!warm) {
    st->magic = kStateMagic; st->n = sk.n; st->k = sk.k; st->resid = sk.resid; st->tag = sk.tag;
    st->delta = kDeltaInit;
    st->calls = st->rescans = st->fallbacks = st->nonfinite_calls = st->fast_calls = 0;
  } else {
    float d = st->delta;
    if (cc < k) d = d * 2.0f;
    else if (cc > cap) d = d * 0.5f;
    else if ((double)cc > (double)sk.band_hi * (double)k) d = d * 0.75f;
    else if ((double)cc < (double)sk.band_lo * (double)k) d = d * 1.5f;
    st->delta = d < kDeltaMin ? kDeltaMin : (d > kDeltaMax ? kDeltaMax : d);
  }
  st->calls += 1;
  st->rescans += path == 2;
  st->fallbacks += path == 1;
  st->fast_calls += path == 3;
  st->nonfinite_calls += nonfinite > 0;
  st->last_nonfinite = nonfinite;
  st->kstar = kstar;
  st->last_cand = cc;
  st->last_path = path;
}

// ---- histogram "find": the bin holding the need-th largest key (1-based) --------------------
// h: global histogram (nb bins, nb % 256 == 0). Walks bins from the top. Returns the bin
// (or -1 if the total is below `need`) and, via *above, the count in strictly higher bins.
// stage (optional): NB words of shared memory; the histogram is then read coalesced into it first
// (every CTA of a grid reads the same lines: thread-contiguous global reads cost 4x the L2 requests)
template <int NB>
__device__ int find_bin_desc(const uint32_t* h, uint64_t need, uint64_t* above_out, uint64_t* smem_scan,
                             uint32_t* stage = nullptr) {
  __shared__ int s_bin;
  __shared__ uint64_t s_above;
  constexpr int PER = NB / kThreads;               // 16, 4 or 2 bins per thread, loaded as vectors
  const int lo = NB - (threadIdx.x + 1) * PER;     // this thread's bins: [lo, lo + PER)
  uint32_t c[PER];
  if (stage) {
    for (int j = threadIdx.x; j < NB / 4; j += kThreads)
      reinterpret_cast<uint4*>(stage)[j] = __ldcg(reinterpret_cast<const uint4*>(h) + j);
    __syncthreads();
#pragma unroll
    for (int q = 0; q < PER; ++q) c[q] = stage[lo + q];
  } else {
#pragma unroll
    for (int q = 0; q < PER; q += 2) {
      const uint2 u = __ldcg(reinterpret_cast<const uint2*>(h + lo + q));
      c[q] = u.x; c[q + 1] = u.y;
    }
  }
  uint64_t sum = 0;
#pragma unroll
  for (int q = 0; q < PER; ++q) sum += c[q];
  if (threadIdx.x == 0) { s_bin = -1; s_above = 0; }
  uint64_t total;
  uint64_t above = block_exclusive_scan(sum, smem_scan, &total);   // syncs inside
  if (above < need && above + sum >= need) {
#pragma unroll
    for (int q = PER - 1; q >= 0; --q) {
      if (above + c[q] >= need) { s_bin = lo + q; s_above = above; break; }
      above += c[q];
    }
  }
  __syncthreads();
  if (s_bin < 0) { *above_out = total; return -1; }
  *above_out = s_above;
  return s_bin;
}

// ---- stratified sample of keys (recovery) ---------------------------------------------------
// Runs after the streaming pass, which stored r = a = g + r for every element it did not record
// (recorded candidates hold their as-if-selected residual: a bias of < k keys), so the sample
// reads the residual alone. Samples are 8-element (32-byte, sector-aligned) micro-chunks spread
// evenly over [0, n) with a per-call phase, so small parameter segments are represented in
// proportion. Exhaustive mode (small n) visits every micro-chunk. This thread's share:
// micro-chunks first, first + step, ...
__device__ __forceinline__ void sample_accumulate(const float* r, uint64_t n, uint32_t num_micro, double stride,
                                                  double phase, int exhaustive, uint32_t* sh, uint32_t first,
                                                  uint32_t step, uint32_t* shf = nullptr, uint32_t T = 0,
                                                  uint32_t t_lo = 0, uint32_t sf = 0) {
  // shf (optional): keys in [t_lo, T) by their distance below T, bins of 2^sf key units
  auto fine = [&](uint32_t key) {
    if (shf && key < T && key >= t_lo) {
      const uint32_t j = (T - 1 - key) >> sf;      // stored reversed: bin 4095 - j (top = just below T)
      atomicAdd(&shf[4095u - (j < 4095u ? j : 4095u)], 1u);
    }
  };
  const uint64_t n8 = n / 8;
  for (uint32_t m = first; m < num_micro; m += step) {
    uint64_t c8 = exhaustive ? m : (uint64_t)(((double)m + phase) * stride);
    if (!exhaustive && c8 >= n8) c8 = n8 ? n8 - 1 : 0;
    const uint64_t i = c8 * 8;
    if (i + 8 <= n) {
      const float4 r0 = __ldcg(reinterpret_cast<const float4*>(r + i));
      const float4 r1 = __ldcg(reinterpret_cast<const float4*>(r + i + 4));
      const float a[8] = {r0.x, r0.y, r0.z, r0.w, r1.x, r1.y, r1.z, r1.w};
#pragma unroll
      for (int e = 0; e < 8; ++e) {
        atomicAdd(&sh[mag_key(a[e]) >> shift(0)], 1u);
        fine(mag_key(a[e]));
      }
    } else {
      for (uint64_t j = i; j < n; ++j) {
        atomicAdd(&sh[mag_key(__ldcg(r + j)) >> shift(0)], 1u);
        fine(mag_key(__ldcg(r + j)));
      }
    }
  }
}

// A threshold from the finished sample histogram hs (block-wide; every thread gets it).
// Exhaustive -> the lower edge of the bin holding the need_exact-th largest key (exact);
// sampled -> `factor` x the expected sample count above the k-th key (+8), placed inside its
// 6 %-wide bin by an exponential-density model of this bin and the next one up, moved 20 %
// toward the lower edge as a safety margin.
__device__ __forceinline__ uint32_t threshold_from_sample(const uint32_t* hs, uint64_t n, uint64_t k,
                                                          uint64_t need_exact, double factor, uint32_t num_micro,
                                                          int exhaustive, uint64_t* s_scan) {
  __shared__ uint32_t s_t;
  const uint64_t S = exhaustive ? n : (uint64_t)num_micro * 8;
  const uint64_t need = exhaustive ? need_exact : (uint64_t)(factor * (double)k * (double)S / (double)n) + 8;
  uint64_t above;
  const int b = find_bin_desc<bins(0)>(hs, need, &above, s_scan);
  if (threadIdx.x == 0) {
    uint32_t t = (b < 0) ? 0u : ((uint32_t)b << shift(0));
    if (b >= 0 && !exhaustive) {
      const double c0 = (double)__ldcg(hs + b);
      const double c1 = (b + 1 < bins(0)) ? (double)__ldcg(hs + b + 1) : 0.0;
      const double f = (double)(need - above) / (c0 > 0 ? c0 : 1.0);   // share of the bin needed, (0, 1]
      double x;                                                        // position from the bin's bottom
      if (c1 >= c0 || c0 < 2) {
        x = 1.0 - f;
      } else {
        const double lam = log(c0 / (c1 > 0.5 ? c1 : 0.5));
        const double el = exp(-lam);
        x = -log(f * (1.0 - el) + el) / lam;
      }
      x = 0.8 * (x < 0 ? 0 : (x > 1 ? 1 : x));
      uint32_t off = (uint32_t)(x * (double)(1u << shift(0)));
      if (off >= (1u << shift(0))) off = (1u << shift(0)) - 1;
      t += off;
    }
    s_t = t;
  }
  __syncthreads();
  return s_t;
}

// End of a streaming tile: the tile's candidates go to the buffer (if it has room) and the
// residual is stored. A candidate that was recorded is stored as if it were selected (r = 0, or
// a - fp32(bf16(a)) for bf16 values, reading #8): the select kernel then writes r = a back only
// for the candidates it rejects (~0.3 k), instead of scattering the k selected ones (a scattered
// 4-byte store costs a 32-byte DRAM read-modify-write).
__device__ __forceinline__ float selected_residual(float a, int vbf16) {
  return vbf16 ? a - __bfloat162float(__float2bfloat16_rn(a)) : 0.0f;
}
__device__ __forceinline__ void tile_tail(float (&a)[4][4], uint32_t flags, uint32_t total,
                                          const uint32_t (&vec_base)[4], uint64_t excl, uint32_t b,
                                          uint32_t cap, uint64_t base, uint64_t n, bool full, int vbf16,
                                          float* __restrict__ r, uint32_t* __restrict__ cand_idx,
                                          float* __restrict__ cand_val) {
  const int tid = threadIdx.x;
  const bool rec = total && (uint64_t)b + total <= cap;
  if (rec && flags) {
#pragma unroll
    for (int c = 0; c < 4; ++c) {
      uint32_t pos = b + vec_base[c] + (uint32_t)((excl >> (16 * c)) & 0xFFFF);
#pragma unroll
      for (int e = 0; e < 4; ++e)
        if (flags & (1u << (c * 4 + e))) {
          cand_idx[pos] = (uint32_t)(base + c * 1024 + tid * 4 + e);
          cand_val[pos] = a[c][e];
          ++pos;
        }
    }
  }
  const uint32_t sel = rec ? flags : 0u;
#pragma unroll
  for (int c = 0; c < 4; ++c) {
    float o[4];
#pragma unroll
    for (int e = 0; e < 4; ++e) o[e] = (sel >> (c * 4 + e)) & 1u ? selected_residual(a[c][e], vbf16) : a[c][e];
    const uint64_t i = base + c * 1024 + tid * 4;
    if (full) {
      __stcs(reinterpret_cast<float4*>(r + i), make_float4(o[0], o[1], o[2], o[3]));
    } else {
#pragma unroll
      for (int e = 0; e < 4; ++e)
        if (i + e < n) r[i + e] = o[e];
    }
  }
}

// Order-preserving compaction of one 4096-element tile: one block scan of 4 x 16-bit per-vector
// counts. Returns the tile total; vec_base / excl locate this thread's flagged elements.
__device__ __forceinline__ uint32_t tile_scan(uint32_t flags, uint64_t* s_scan_par, uint32_t (&vec_base)[4],
                                              uint64_t& excl) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint64_t packed = 0;
#pragma unroll
  for (int c = 0; c < 4; ++c) packed |= (uint64_t)__popc((flags >> (4 * c)) & 0xFu) << (16 * c);
  uint64_t incl = packed;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    uint64_t y = __shfl_up_sync(0xFFFFFFFFu, incl, o);
    if (lane >= o) incl += y;
  }
  if (lane == 31) s_scan_par[warp] = incl;
  __syncthreads();
  uint64_t warp_off = 0, tot = 0;
#pragma unroll
  for (int w = 0; w < kThreads / 32; ++w) {
    uint64_t t = s_scan_par[w];
    warp_off += (w < warp) ? t : 0;
    tot += t;
  }
  excl = warp_off + incl - packed;
  uint32_t total = 0;
#pragma unroll
  for (int c = 0; c < 4; ++c) { vec_base[c] = total; total += (uint32_t)((tot >> (16 * c)) & 0xFFFF); }
  return total;
}

// ---- K1: the fused streaming pass -----------------------------------------------------------
template <bool BF16>
__global__ void __launch_bounds__(kThreads) stream_kernel(const void* __restrict__ g,
                                                          float* __restrict__ r, uint64_t n,
                                                          uint32_t num_tiles, Ctl* ctl,
                                                          uint2* __restrict__ tile_info,
                                                          uint32_t* __restrict__ cand_idx,
                                                          float* __restrict__ cand_val, uint32_t cap,
                                                          int vbf16, uint32_t* __restrict__ hc,
                                                          uint64_t* __restrict__ tk,
                                                          const State* st, StateKey sk, uint32_t force_t) {
  __shared__ uint64_t s_scan[2][kThreads / 32];
  __shared__ uint32_t s_base[2];
  __shared__ uint32_t s_h[bins(0)];               // fine histogram of this CTA's candidates
  for (int j = threadIdx.x; j < bins(0); j += kThreads) s_h[j] = 0;
  const uint32_t T = pass1_threshold(st, sk, force_t);
  const uint32_t FS = fine_shift(st, sk, T, force_t);
  if (blockIdx.x == 0 && threadIdx.x == 0) { ctl->t_est = T; ctl->fine_shift = FS; }
  const int tid = threadIdx.x;
  uint32_t nonfinite = 0;
  int par = 0;
  for (uint32_t tile = blockIdx.x; tile < num_tiles; tile += gridDim.x, par ^= 1) {
    const uint64_t base = (uint64_t)tile * kTile;
    float a[4][4];
    uint32_t flags = 0;
    if (base + kTile <= n) {
      float4 gv[4], rv[4];
#pragma unroll
      for (int c = 0; c < 4; ++c) {
        const uint64_t i = base + c * 1024 + tid * 4;
        gv[c] = load_g4<BF16>(g, i);
        rv[c] = *reinterpret_cast<const float4*>(r + i);
      }
#pragma unroll
      for (int c = 0; c < 4; ++c) {
        a[c][0] = gv[c].x + rv[c].x; a[c][1] = gv[c].y + rv[c].y;
        a[c][2] = gv[c].z + rv[c].z; a[c][3] = gv[c].w + rv[c].w;
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          flags |= (mag_key(a[c][e]) >= T ? 1u : 0u) << (c * 4 + e);
          nonfinite += mag_key(a[c][e]) >= 0x7F800000u;
        }
      }
    } else {
#pragma unroll
      for (int c = 0; c < 4; ++c)
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          const uint64_t i = base + c * 1024 + tid * 4 + e;
          a[c][e] = 0.f;
          if (i < n) {
            a[c][e] = load_g1<BF16>(g, i) + r[i];
            flags |= (mag_key(a[c][e]) >= T ? 1u : 0u) << (c * 4 + e);
            nonfinite += mag_key(a[c][e]) >= 0x7F800000u;
          }
        }
    }
    if (flags) {                                   // the select's first digit, for free
#pragma unroll
      for (int c = 0; c < 4; ++c)
#pragma unroll
        for (int e = 0; e < 4; ++e)
          if ((flags >> (c * 4 + e)) & 1u) atomicAdd(&s_h[fine_bin(mag_key(a[c][e]), T, FS)], 1u);
    }
    uint32_t vec_base[4];
    uint64_t excl;
    const uint32_t total = tile_scan(flags, s_scan[par], vec_base, excl);
    if (tid == 0) {
      uint32_t b = total ? atomicAdd(&ctl->cand_count, total) : 0u;
      s_base[par] = b;
      tile_info[tile] = make_uint2(b, total);
      tk[tile] = 0;
    }
    __syncthreads();
    tile_tail(a, flags, total, vec_base, excl, s_base[par], cap, base, n, base + kTile <= n, vbf16, r,
              cand_idx, cand_val);
  }
  if (nonfinite) atomicAdd(&ctl->nonfinite, nonfinite);
  __syncthreads();
  for (int j = threadIdx.x; j < bins(0); j += kThreads)
    if (s_h[j]) atomicAdd(hc + j, s_h[j]);
}

// ---- K1': the streaming pass with 1-D TMA bulk copies (LOWDIFF_STREAM_TMA=1; measured, not the
// default: DESIGN.md §5) -----------------------------------------------------------------------
// Same per-tile work as stream_kernel, but the g and r tiles of this CTA's next kStages tiles are
// in flight as cp.async.bulk copies (one elected thread, completion on an mbarrier per stage)
// while the current tile is scanned. Full tiles only; the ragged last tile takes direct loads.
#ifndef LOWDIFF_STREAM_STAGES
#define LOWDIFF_STREAM_STAGES 2
#endif
constexpr int kStages = LOWDIFF_STREAM_STAGES;
template <bool BF16>
__global__ void __launch_bounds__(kThreads) stream_tma_kernel(const void* __restrict__ g,
                                                              float* __restrict__ r, uint64_t n,
                                                              uint32_t num_tiles, Ctl* ctl,
                                                              uint2* __restrict__ tile_info,
                                                              uint32_t* __restrict__ cand_idx,
                                                              float* __restrict__ cand_val, uint32_t cap,
                                                              int vbf16, uint32_t* __restrict__ hc,
                                                              uint64_t* __restrict__ tk,
                                                              const State* st, StateKey sk, uint32_t force_t) {
  __shared__ uint32_t s_h[bins(0)];
  for (int j = threadIdx.x; j < bins(0); j += kThreads) s_h[j] = 0;
  constexpr uint32_t kGB = kTile * (BF16 ? 2 : 4), kRB = kTile * 4, kSB = kGB + kRB;
  extern __shared__ __align__(128) uint8_t s_tiles[];          // kStages x {g tile, r tile}
  __shared__ __align__(8) uint64_t s_bar[kStages];
  __shared__ uint64_t s_scan[2][kThreads / 32];
  __shared__ uint32_t s_base[2];
  const uint32_t T = pass1_threshold(st, sk, force_t);
  const uint32_t FS = fine_shift(st, sk, T, force_t);
  if (blockIdx.x == 0 && threadIdx.x == 0) { ctl->t_est = T; ctl->fine_shift = FS; }
  const int tid = threadIdx.x;
  uint32_t nonfinite = 0;
  const uint32_t full_tiles = (uint32_t)(n / kTile);
  auto issue = [&](uint32_t it) {                              // this CTA's it-th tile -> its stage
    const uint32_t tile = blockIdx.x + it * gridDim.x;
    if (tile >= full_tiles) return;
    const uint32_t stg = it % kStages, bar = smem_u32(&s_bar[stg]);
    const uint32_t dst = smem_u32(s_tiles + stg * kSB);
    mbar_expect_tx(bar, kSB);
    bulk_g2s(dst, static_cast<const uint8_t*>(g) + (uint64_t)tile * kGB, kGB, bar);
    bulk_g2s(dst + kGB, reinterpret_cast<const uint8_t*>(r) + (uint64_t)tile * kRB, kRB, bar);
  };
  if (tid == 0) {
    for (int s = 0; s < kStages; ++s) mbar_init(smem_u32(&s_bar[s]), 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    for (uint32_t it = 0; it < (uint32_t)kStages; ++it) issue(it);
  }
  __syncthreads();
  int par = 0;
  uint32_t it = 0;
  for (uint32_t tile = blockIdx.x; tile < num_tiles; tile += gridDim.x, par ^= 1, ++it) {
    const uint64_t base = (uint64_t)tile * kTile;
    float a[4][4];
    uint32_t flags = 0;
    if (tile < full_tiles) {
      const uint32_t stg = it % kStages;
      mbar_wait(smem_u32(&s_bar[stg]), (it / kStages) & 1u);
      const uint8_t* sg = s_tiles + stg * kSB;
      const float* sr = reinterpret_cast<const float*>(sg + kGB);
#pragma unroll
      for (int c = 0; c < 4; ++c) {
        const int o = c * 1024 + tid * 4;
        float4 gv;
        if constexpr (BF16) {
          const uint2 u = *reinterpret_cast<const uint2*>(sg + 2 * o);
          gv = make_float4(__uint_as_float(u.x << 16), __uint_as_float(u.x & 0xFFFF0000u),
                           __uint_as_float(u.y << 16), __uint_as_float(u.y & 0xFFFF0000u));
        } else {
          gv = *reinterpret_cast<const float4*>(sg + 4 * o);
        }
        const float4 rv = *reinterpret_cast<const float4*>(sr + o);
        a[c][0] = gv.x + rv.x; a[c][1] = gv.y + rv.y; a[c][2] = gv.z + rv.z; a[c][3] = gv.w + rv.w;
      }
    } else {
#pragma unroll
      for (int c = 0; c < 4; ++c)
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          const uint64_t i = base + c * 1024 + tid * 4 + e;
          a[c][e] = i < n ? load_g1<BF16>(g, i) + r[i] : 0.f;
        }
    }
#pragma unroll
    for (int c = 0; c < 4; ++c) {
      const uint64_t i = base + c * 1024 + tid * 4;
#pragma unroll
      for (int e = 0; e < 4; ++e)
        if (tile < full_tiles || i + e < n) {
          flags |= (mag_key(a[c][e]) >= T ? 1u : 0u) << (c * 4 + e);
          nonfinite += mag_key(a[c][e]) >= 0x7F800000u;
        }
    }
    if (flags) {
#pragma unroll
      for (int c = 0; c < 4; ++c)
#pragma unroll
        for (int e = 0; e < 4; ++e)
          if ((flags >> (c * 4 + e)) & 1u) atomicAdd(&s_h[fine_bin(mag_key(a[c][e]), T, FS)], 1u);
    }
    uint32_t vec_base[4];
    uint64_t excl;
    const uint32_t total = tile_scan(flags, s_scan[par], vec_base, excl);   // every thread is done with the stage
    if (tid == 0) {
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      issue(it + kStages);                            // refill the stage just consumed
      uint32_t b = total ? atomicAdd(&ctl->cand_count, total) : 0u;
      s_base[par] = b;
      tile_info[tile] = make_uint2(b, total);
      tk[tile] = 0;
    }
    __syncthreads();
    tile_tail(a, flags, total, vec_base, excl, s_base[par], cap, base, n, tile < full_tiles, vbf16, r,
              cand_idx, cand_val);
  }
  if (nonfinite) atomicAdd(&ctl->nonfinite, nonfinite);
  __syncthreads();
  for (int j = threadIdx.x; j < bins(0); j += kThreads)
    if (s_h[j]) atomicAdd(hc + j, s_h[j]);
}

// ---- K2: exact radix select over the candidates (or the full array) ------------------------
struct SelArgs {
  float* r;
  uint64_t n, k;
  Ctl* ctl;
  State* st;
  StateKey sk;
  const uint32_t* cidx1; const float* cval1; const uint2* tinfo1;   // first pass
  uint32_t* cidx2; float* cval2; uint2* tinfo2;                     // rescan
  uint32_t num_tiles, cap;
  uint32_t *hs, *hc, *hc2, *h0, *h1, *h2;
  uint64_t* tloc;
  uint64_t* tk;            // fast select: packed (> K*, == K*) counts per tile
  uint64_t* ctot;          // fast select: the same per chunk of chunk_tiles tiles
  uint32_t* hl;            // fast select: low key bits of the undecided
  uint32_t* gbits;         // fast select: "> K*" bit per candidate position
  uint32_t* ebits;         // fast select: "== K*" bit per candidate position
  uint64_t* inbin;         // fast select: (position, value) of the undecided
  uint32_t chunk_tiles, num_chunks;
  uint64_t* boff;
  uint8_t* pairs;
  uint32_t num_micro;       // recovery sample
  double stride, phase;
  int exhaustive;
  uint32_t force_t2;        // test hook: the rescan's threshold
  int fast;                 // the fast select may run (LOWDIFF_FAST_SELECT=0: always the general path)
};

// One cooperative launch runs the three digit passes (12 + 10 + 9 bits of the 31-bit key) with a
// grid barrier after each histogram; every CTA then redoes the tiny 'find' on the L2-resident
// histogram itself, so no second barrier or serial tail is needed per pass.
template <int PASS>
__device__ __forceinline__ void select_pass(const float* __restrict__ src, uint64_t N, uint32_t* sh,
                                            uint32_t* hist, uint32_t& prefix, uint64_t& need,
                                            uint64_t* s_scan, cg::grid_group& grid, bool count = true) {
  constexpr int NB = bins(PASS);
  constexpr int SH = shift(PASS);
  if (count) {
  for (int b = threadIdx.x; b < NB; b += kThreads) sh[b] = 0;
  __syncthreads();
  // Warp-aggregated increments: the candidates' keys crowd into few bins, so lanes with the same
  // bin are combined (__match_any_sync) into one shared-memory atomic.
  const int lane = threadIdx.x & 31;
  const uint64_t stride = (uint64_t)gridDim.x * kThreads;
  constexpr int U = 4;                             // loads in flight per thread
  for (uint64_t base = (uint64_t)blockIdx.x * kThreads + (threadIdx.x & ~31u); base < N; base += U * stride) {
    uint32_t keys[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const uint64_t i = base + u * stride + lane;
      keys[u] = i < N ? mag_key(src[i]) : 0u;
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      if (base + u * stride >= N) break;           // warp-uniform
      const uint64_t i = base + u * stride + lane;
      const uint32_t key = keys[u];
      const bool take = i < N && (PASS == 0 || (key >> shift(PASS > 0 ? PASS - 1 : 0)) == prefix);
      const uint32_t act = __ballot_sync(0xFFFFFFFFu, take);
      if (take) {
        const uint32_t bin = (key >> SH) & (NB - 1);
        const uint32_t peers = __match_any_sync(act, bin);
        if (lane == __ffs(peers) - 1) atomicAdd(&sh[bin], (uint32_t)__popc(peers));
      }
    }
  }
  __syncthreads();
  for (int b = threadIdx.x; b < NB; b += kThreads)
    if (sh[b]) atomicAdd(hist + b, sh[b]);
  grid.sync();
  }
  uint64_t above;
  const int d = find_bin_desc<NB>(hist, need, &above, s_scan);
  need -= above;
  prefix = (PASS == 0) ? (uint32_t)d : ((prefix << (PASS == 1 ? 10 : 9)) | (uint32_t)d);
  __syncthreads();
}

// Chunked block scan of packed (count > K*, count == K*) values over positions [a, e) of a block's
// chunk: writes the block-local exclusive prefix to out[p]; returns the chunk total.
template <typename ValueFn>
__device__ __forceinline__ uint64_t chunk_scan(uint64_t a, uint64_t e, ValueFn value, uint64_t* out,
                                               uint64_t* s_scan) {
  uint64_t carry = 0;
  for (uint64_t base = a; base < e; base += (uint64_t)kThreads * 4) {
    uint64_t v[4], sum = 0;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const uint64_t p = base + threadIdx.x * 4 + j;
      v[j] = p < e ? value(p) : 0;
      sum += v[j];
    }
    uint64_t tot;
    uint64_t run = carry + block_exclusive_scan(sum, s_scan, &tot);
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const uint64_t p = base + threadIdx.x * 4 + j;
      if (p < e) out[p] = run;
      run += v[j];
    }
    carry += tot;
  }
  return carry;
}

// Exclusive prefix of the blocks' chunk totals (each block sums bsum[0, blockIdx.x)).
__device__ __forceinline__ uint64_t block_offset(const uint64_t* bsum, uint64_t* s_scan) {
  uint64_t v[kMaxSelectBlocks / kThreads + 1];     // independent loads, issued together
#pragma unroll
  for (int q = 0; q < kMaxSelectBlocks / kThreads + 1; ++q) {
    const uint32_t b = threadIdx.x + q * kThreads;
    v[q] = b < blockIdx.x ? __ldcg(bsum + b) : 0;
  }
  uint64_t part = 0;
#pragma unroll
  for (int q = 0; q < kMaxSelectBlocks / kThreads + 1; ++q) part += v[q];
  uint64_t tot;
  block_exclusive_scan(part, s_scan, &tot);
  return tot;
}

// Put a = g + r back into the residual for every recorded candidate of a buffer (the pass that
// recorded them stored r as if they were selected). Grid-stride over tiles.
__device__ __forceinline__ void restore_recorded(float* r, const uint2* tinfo, const uint32_t* cidx,
                                                 const float* cval, uint32_t num_tiles, uint32_t cap) {
  const uint64_t stride = (uint64_t)gridDim.x * kThreads;
  for (uint64_t t = (uint64_t)blockIdx.x * kThreads + threadIdx.x; t < num_tiles; t += stride) {
    const uint2 ti = tinfo[t];
    if (ti.y && (uint64_t)ti.x + ti.y <= cap)
      for (uint32_t j = 0; j < ti.y; ++j) r[cidx[ti.x + j]] = cval[ti.x + j];
  }
}

// Recovery rescan: rebuild the candidate set at threshold T2 from the residual, with the first
// pass's recorded candidates overlaid from its buffer (their r holds the as-if-selected value).
// Writes the rescan buffer, its tile table and first-digit histogram, and fixes r wherever an
// element's recorded state changes (recorded now, not before: as-if-selected; before, not now: a).
__device__ void rescan(const SelArgs& A, uint32_t T2, int vbf16, float* s_ov, uint32_t* s_bits, uint32_t* s_h,
                       uint64_t (*s_scan)[kThreads / 32], uint32_t* s_base) {
  const int tid = threadIdx.x;
  const uint64_t n = A.n;
  for (int j = tid; j < bins(0); j += kThreads) s_h[j] = 0;
  __syncthreads();
  int par = 0;
  for (uint32_t tile = blockIdx.x; tile < A.num_tiles; tile += gridDim.x, par ^= 1) {
    const uint64_t base = (uint64_t)tile * kTile;
    const bool full = base + kTile <= n;
    float a[4][4];
    if (full) {
#pragma unroll
      for (int c = 0; c < 4; ++c) {
        const float4 v = __ldcg(reinterpret_cast<const float4*>(A.r + base + c * 1024 + tid * 4));
        a[c][0] = v.x; a[c][1] = v.y; a[c][2] = v.z; a[c][3] = v.w;
      }
    } else {
#pragma unroll
      for (int c = 0; c < 4; ++c)
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          const uint64_t i = base + c * 1024 + tid * 4 + e;
          a[c][e] = i < n ? A.r[i] : 0.f;
        }
    }
    const uint2 s1 = A.tinfo1[tile];
    uint32_t old = 0;
    if (s1.y && (uint64_t)s1.x + s1.y <= A.cap) {       // block-uniform
      if (tid < kTile / 32) s_bits[tid] = 0;
      __syncthreads();
      for (uint32_t j = tid; j < s1.y; j += kThreads) {
        const uint32_t o = A.cidx1[s1.x + j] - (uint32_t)base;
        s_ov[o] = A.cval1[s1.x + j];
        atomicOr(&s_bits[o >> 5], 1u << (o & 31));
      }
      __syncthreads();
#pragma unroll
      for (int c = 0; c < 4; ++c)
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          const uint32_t o = c * 1024 + tid * 4 + e;
          if ((s_bits[o >> 5] >> (o & 31)) & 1u) { a[c][e] = s_ov[o]; old |= 1u << (c * 4 + e); }
        }
    }
    uint32_t flags = 0;
#pragma unroll
    for (int c = 0; c < 4; ++c)
#pragma unroll
      for (int e = 0; e < 4; ++e)
        if (full || base + c * 1024 + tid * 4 + e < n) flags |= (mag_key(a[c][e]) >= T2 ? 1u : 0u) << (c * 4 + e);
    if (flags) {
#pragma unroll
      for (int c = 0; c < 4; ++c)
#pragma unroll
        for (int e = 0; e < 4; ++e)
          if ((flags >> (c * 4 + e)) & 1u) atomicAdd(&s_h[mag_key(a[c][e]) >> shift(0)], 1u);
    }
    uint32_t vec_base[4];
    uint64_t excl;
    const uint32_t total = tile_scan(flags, s_scan[par], vec_base, excl);
    if (tid == 0) {
      const uint32_t b = total ? atomicAdd(&A.ctl->cand_count2, total) : 0u;
      s_base[par] = b;
      A.tinfo2[tile] = make_uint2(b, total);
    }
    __syncthreads();
    const uint32_t b = s_base[par];
    const bool rec = total && (uint64_t)b + total <= A.cap;
    if (rec && flags) {
#pragma unroll
      for (int c = 0; c < 4; ++c) {
        uint32_t pos = b + vec_base[c] + (uint32_t)((excl >> (16 * c)) & 0xFFFF);
#pragma unroll
        for (int e = 0; e < 4; ++e)
          if (flags & (1u << (c * 4 + e))) {
            A.cidx2[pos] = (uint32_t)(base + c * 1024 + tid * 4 + e);
            A.cval2[pos] = a[c][e];
            ++pos;
          }
      }
    }
    const uint32_t sel = rec ? flags : 0u;
    uint32_t diff = sel ^ old;
    while (diff) {
      const int bit = __ffs(diff) - 1;
      diff &= diff - 1;
      const int c = bit >> 2, e = bit & 3;
      const float v = a[c][e];
      A.r[base + c * 1024 + tid * 4 + e] = ((sel >> bit) & 1u) ? selected_residual(v, vbf16) : v;
    }
  }
  __syncthreads();
  for (int j = tid; j < bins(0); j += kThreads)
    if (s_h[j]) atomicAdd(A.hc2 + j, s_h[j]);
}

// ---- K2 fast path: warm first pass, the k-th key in a narrow fine bin ------------------------
// The stream pass histogrammed the candidates into fine bins relative to T (bin width 2^s keys,
// s <= 12). The bin b* holding the k-th largest key splits the candidates: bins above b* are
// surely > K*, bins below surely < K* (rejected), those in b* are undecided until K* is known.
//   phase 1 (balanced over buffer positions): per position a "> K*" bit and a "== K*" bit (one
//     warp ballot per 32 positions), packed (>, ==) counts per tile and per chunk of tiles
//     (warp-aggregated 64-bit atomics); the undecided go to a list plus a histogram of their low
//     s key bits; the surely rejected get r = a back.                     -- grid barrier --
//   phase 2 (every CTA): K* and the kept tie count m from the low-bit histogram; each CTA resolves
//     a slice of the undecided list into the bits and counts (< K*: r = a). -- grid barrier --
//   phase 3 (balanced over positions): for the candidate at buffer position p in tile t,
//     (gt, eq) before it = (chunk offset) + (a warp-wide sum over t's chunk before t) + (bits in t's
//     segment before p); kept iff > K*, or == K* with eq < m; slot = gt + min(eq, m).
// The candidates of one tile are contiguous in the buffer and in index order, so "before" is
// "at a lower index". Two grid barriers, no tile scan (the general path has five).
__device__ __forceinline__ uint64_t warp_sum64(uint64_t v) {
#pragma unroll
  for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xFFFFFFFFu, v, o);
  return v;
}

#ifdef LOWDIFF_SEL_TIMING
// experiment instrumentation (not in the product build): per-CTA %globaltimer stamps at the phase
// boundaries of the fast select, printed by sel_timing_print for one chosen call
__device__ uint64_t g_seltime[8][1024];
__device__ __forceinline__ void sel_stamp(int i) {
  if (threadIdx.x == 0 && blockIdx.x < 1024) {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    g_seltime[i][blockIdx.x] = t;
  }
}
__global__ void sel_timing_print(const State* st, uint32_t grid, uint64_t when) {
  if (st->calls != when) return;
  uint64_t t0 = ~0ull;
  for (uint32_t b = 0; b < grid; ++b) t0 = min(t0, g_seltime[0][b]);
  for (int i = 0; i < 8; ++i) {
    uint64_t lo = ~0ull, hi = 0, sum = 0;
    for (uint32_t b = 0; b < grid; ++b) {
      const uint64_t t = g_seltime[i][b] - t0;
      lo = min(lo, t); hi = max(hi, t); sum += t;
    }
    printf("sel stamp %d: min %.2f us  mean %.2f us  max %.2f us\n", i, lo * 1e-3, sum * 1e-3 / grid, hi * 1e-3);
  }
}
#define SEL_STAMP(i) sel_stamp(i)
#else
#define SEL_STAMP(i)
#endif

template <bool VBF16>
__device__ void fast_select(const SelArgs& A, uint32_t T, uint32_t S, uint32_t bst, uint64_t above,
                            uint32_t cc, uint8_t* s_raw, uint64_t* s_scan, cg::grid_group& grid) {
  Ctl* ctl = A.ctl;
  const uint64_t k = A.k;
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t lowmask = (1u << S) - 1;
  const uint32_t num_tiles = A.num_tiles;
  // chunking of the tile counts: tiles holding >= 32 candidates (C2, C4) go through long runs with a
  // warp-wide prefix over chunks of 32q tiles; sparser tiles take the finest chunks kMaxChunks allows
  // so each lane can sum its own tile's prefix (measured: C3 select 45.8 -> 37.6 us; the finer
  // chunks cost the dense-tile configurations their longer chunk-offset prologue)
  // (tiles of >= 32 candidates take the per-lane prefix too while the fine chunks stay <= 16 tiles:
  // C2 compress 81 -> 75 us per call; only C4/C5-sized tile counts keep the long warp runs)
  const bool dense_tiles = cc / (num_tiles ? num_tiles : 1) >= 32 && (num_tiles + kMaxChunks - 1) / kMaxChunks > 16;
  const uint32_t CH = dense_tiles || num_tiles == 0 ? A.chunk_tiles : (num_tiles + kMaxChunks - 1) / kMaxChunks;
  const uint32_t nch = (num_tiles + CH - 1) / CH;
  constexpr uint64_t kGt = 1ull << 32;             // packed count: (> K*) << 32 | (== K*)
  float* r = A.r;
  const uint64_t nwarps = (uint64_t)gridDim.x * (kThreads / 32);
  const uint64_t wid = ((uint64_t)blockIdx.x * kThreads + threadIdx.x) >> 5;
  // ---- phase 1: classify (4 words per warp in flight) ----
  SEL_STAMP(1);
  constexpr uint32_t kStage = 2 * 4 * kTile / 8;   // undecided entries staged per CTA (s_raw)
  uint64_t* s_stage = reinterpret_cast<uint64_t*>(s_raw);
  __shared__ uint32_t s_ucnt;
  if (threadIdx.x == 0) s_ucnt = 0;
  __syncthreads();
#ifndef LOWDIFF_SEL_U1
#define LOWDIFF_SEL_U1 4
#endif
  constexpr int U1 = LOWDIFF_SEL_U1;
  for (uint64_t base0 = wid * 32; base0 < cc; base0 += U1 * nwarps * 32) {   // warp-uniform
  float av[U1];
  uint32_t iv[U1];
#pragma unroll
  for (int v = 0; v < U1; ++v) {
    const uint64_t pv = base0 + v * nwarps * 32 + lane;
    av[v] = pv < cc ? A.cval1[pv] : 0.f;
    iv[v] = pv < cc ? A.cidx1[pv] : 0u;
  }
#pragma unroll
  for (int u = 0; u < U1; ++u) {
    const uint64_t base = base0 + u * nwarps * 32;
    if (base >= cc) break;                         // warp-uniform
    const uint64_t p = base + lane;
    const bool in = p < cc;
    const float a = av[u];
    const uint32_t idx = iv[u];
    const uint32_t key = mag_key(a);
    const uint32_t fb = in ? fine_bin(key, T, S) : 0u;
    const bool sure = in && fb > bst, und = in && fb == bst;
    if (in && fb < bst) r[idx] = a;                // surely rejected: keeps all of a
    const uint32_t sk = __ballot_sync(0xFFFFFFFFu, sure);
    if (lane == 0) { A.gbits[base >> 5] = sk; A.ebits[base >> 5] = 0u; }
    if (sure) {                                    // one atomic per tile (and chunk) per warp
      const uint32_t tile = idx / kTile;
      const uint32_t peers = __match_any_sync(sk, tile);
      if (lane == __ffs(peers) - 1) {
        atomicAdd(reinterpret_cast<unsigned long long*>(&A.tk[tile]), (unsigned long long)__popc(peers) << 32);
        atomicAdd(reinterpret_cast<unsigned long long*>(&A.ctot[tile / CH]), (unsigned long long)__popc(peers) << 32);
      }
    }
    const uint32_t ub = __ballot_sync(0xFFFFFFFFu, und);
    if (ub) {
      // staged in shared memory and appended to the global list once per CTA (one global counter
      // for every undecided word serialised phase 1 at C4); the global counter only on overflow
      uint32_t slot0 = 0;
      if (lane == __ffs(ub) - 1) slot0 = atomicAdd(&s_ucnt, (uint32_t)__popc(ub));
      slot0 = __shfl_sync(0xFFFFFFFFu, slot0, __ffs(ub) - 1);
      const bool staged = slot0 + __popc(ub) <= kStage;   // (warp-uniform)
      if (!staged) {
        if (lane == __ffs(ub) - 1) slot0 = atomicAdd(&ctl->inbin_count, (uint32_t)__popc(ub));
        slot0 = __shfl_sync(0xFFFFFFFFu, slot0, __ffs(ub) - 1);
      }
      if (und) {
        const uint64_t ent = ((uint64_t)p << 32) | __float_as_uint(a);
        const uint32_t sl = slot0 + __popc(ub & ((1u << lane) - 1));
        if (staged) s_stage[sl] = ent;
        else A.inbin[sl] = ent;
        atomicAdd(&A.hl[(key - T) & lowmask], 1u);
      }
    }
  }
  }
  __syncthreads();
  {
    const uint32_t ns = min(s_ucnt, kStage);
    __shared__ uint32_t s_g0;
    if (threadIdx.x == 0 && ns) s_g0 = atomicAdd(&ctl->inbin_count, ns);
    __syncthreads();
    for (uint32_t i = threadIdx.x; i < ns; i += kThreads) A.inbin[s_g0 + i] = s_stage[i];
  }
  SEL_STAMP(2);
  grid.sync();
  SEL_STAMP(3);
  // ---- phase 2: K*, m; resolve this CTA's slice of the undecided ----
  __shared__ uint32_t s_K;
  __shared__ uint64_t s_m;
  const uint64_t need = k - above;                 // rank of K* inside bin b* (>= 1)
  {
    const uint32_t NB = 1u << S;
    const uint32_t per = NB > kThreads ? NB / kThreads : 1;
    const bool act = threadIdx.x * per < NB;
    const uint32_t lo = act ? NB - (threadIdx.x + 1) * per : 0;
    uint32_t* s_hl = reinterpret_cast<uint32_t*>(s_raw);  // coalesced copy (every CTA reads it)
    for (uint32_t j = threadIdx.x; j < NB; j += kThreads) s_hl[j] = __ldcg(A.hl + j);
    __syncthreads();
    uint64_t sum = 0;
    for (uint32_t q = 0; q < per && act; ++q) sum += s_hl[lo + q];
    uint64_t tot;
    uint64_t ab = block_exclusive_scan(sum, s_scan, &tot);
    if (act && ab < need && ab + sum >= need) {
      for (int q = (int)per - 1; q >= 0; --q) {
        const uint32_t c = s_hl[lo + q];
        if (ab + c >= need) { s_K = T + (bst << S) + lo + q; s_m = need - ab; break; }
        ab += c;
      }
    }
    __syncthreads();
  }
  const uint32_t K = s_K;
  const uint64_t m = s_m;
  const uint32_t n_in = __ldcg(&ctl->inbin_count);
  for (uint64_t i = (uint64_t)blockIdx.x * kThreads + threadIdx.x; i < n_in; i += (uint64_t)gridDim.x * kThreads) {
    const uint64_t e = __ldcg(A.inbin + i);
    const uint32_t p = (uint32_t)(e >> 32);
    const float a = __uint_as_float((uint32_t)e);
    const uint32_t key = mag_key(a), idx = A.cidx1[p];
    if (key >= K) {
      const uint64_t inc = key > K ? kGt : 1ull;
      atomicOr(key > K ? &A.gbits[p >> 5] : &A.ebits[p >> 5], 1u << (p & 31));
      atomicAdd(reinterpret_cast<unsigned long long*>(&A.tk[idx / kTile]), (unsigned long long)inc);
      atomicAdd(reinterpret_cast<unsigned long long*>(&A.ctot[idx / kTile / CH]), (unsigned long long)inc);
    } else {
      r[idx] = a;                                  // below K*: keeps all of a
    }
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    ctl->mode = 3; ctl->kstar = K; ctl->m = m;
    state_update(A.st, A.sk, k, A.cap, cc, 3, K, ctl->nonfinite);
  }
  SEL_STAMP(4);
  grid.sync();
  SEL_STAMP(5);
  // ---- phase 3: chunk offsets (every CTA), then the ordered emission ----
  uint64_t* s_coff = reinterpret_cast<uint64_t*>(s_raw);          // <= 4096 chunks
  {
    const uint32_t per = (nch + kThreads - 1) / kThreads;         // <= 16
    // coalesced into shared memory first (every CTA reads the same lines: thread-contiguous global
    // reads cost 4x the L2 sector requests), then each thread scans its contiguous run
    for (uint32_t c = threadIdx.x; c < nch; c += kThreads) s_coff[c] = __ldcg(A.ctot + c);
    __syncthreads();
    uint64_t v[16], gsum = 0, esum = 0;
#pragma unroll
    for (int q = 0; q < 16; ++q) {
      const uint32_t c = threadIdx.x * per + q;
      v[q] = (q < (int)per && c < nch) ? s_coff[c] : 0ull;
      gsum += v[q] >> 32;
      esum += v[q] & 0xFFFFFFFFull;
    }
    uint64_t tot;
    uint64_t run = block_exclusive_scan((gsum << 32) | esum, s_scan, &tot);   // both halves < 2^32
#pragma unroll
    for (int q = 0; q < 16; ++q) {
      const uint32_t c = threadIdx.x * per + q;
      if (q < (int)per && c < nch) s_coff[c] = run;
      run += v[q];
    }
  }
  __syncthreads();
  SEL_STAMP(6);
  uint8_t* pairs = A.pairs;
  uint32_t* out_idx = reinterpret_cast<uint32_t*>(pairs);
  uint8_t* out_val = pairs + pad16(4 * k);
  if (blockIdx.x == 0 && threadIdx.x < 16) {       // zero the 16-byte padding of both sections
    const uint64_t ip = 4 * k, ie = pad16(4 * k);
    if (ip + threadIdx.x < ie) pairs[ip + threadIdx.x] = 0;
    const uint64_t vp = pad16(4 * k) + (VBF16 ? 2 : 4) * k, ve = pad16(4 * k) + pad16((VBF16 ? 2 : 4) * k);
    if (vp + threadIdx.x < ve) pairs[vp + threadIdx.x] = 0;
  }
  // Warps take runs of W consecutive 32-position words (runs strided over the grid), carrying the
  // packed (gt, eq) count of the current tile from word to word: a tile's prefix (chunk offset + a
  // warp-wide sum over its chunk) is computed once per tile a run meets, the segment carry before
  // the run (a warp-wide popcount over earlier words) once per run. Long runs amortise that when
  // tiles hold many candidates, but serialise the warp.
  const uint32_t lt = (1u << lane) - 1;
  // (measured: one word per run when tiles hold < 32 candidates, C2/C3; one contiguous range per
  // warp above, C4)
  const uint64_t W = dense_tiles ? ((cc + nwarps * 32 - 1) / (nwarps * 32)) : 1;
  const bool lane_prefix = !dense_tiles && CH <= 16;   // (uniform)
  for (uint64_t run0 = wid * 32 * W; run0 < cc; run0 += nwarps * 32 * W) {   // warp-uniform
  const uint64_t p_end = run0 + 32 * W < cc ? run0 + 32 * W : cc;
  uint32_t cur_t = 0xFFFFFFFFu;                    // the tile continuing from the previous word
  uint64_t cur_before = 0;                         // its packed (gt, eq) before the current word
  auto tile_prefix = [&](uint32_t tt) -> uint64_t {   // packed count in tiles before tt (warp-wide)
    const uint32_t cb = tt / CH * CH;
    uint64_t part = 0;
    for (uint32_t j = cb + lane; j < tt; j += 32) part += __ldcg(A.tk + j);
    return warp_sum64(part) + s_coff[tt / CH];
  };
  // the next word's loads are issued before the current word is processed
  uint32_t n_idx = 0, n_gw = 0, n_ew = 0;
  float n_a = 0.f;
  auto load_word = [&](uint64_t bw) {
    const uint64_t pw = bw + lane;
    n_idx = pw < p_end ? A.cidx1[pw] : 0u;
    n_a = pw < p_end ? A.cval1[pw] : 0.f;
    n_gw = bw < p_end ? __ldcg(A.gbits + (bw >> 5)) : 0u;
    n_ew = bw < p_end ? __ldcg(A.ebits + (bw >> 5)) : 0u;
  };
  load_word(run0);
  for (uint64_t base = run0; base < p_end; base += 32) {   // warp-uniform
    const uint64_t p = base + lane;
    const bool in = p < p_end;
    const uint32_t idx = n_idx, gw = n_gw, ew = n_ew;
    const float a = n_a;
    if (base + 32 < p_end) load_word(base + 32);
    const uint32_t t = in ? idx / kTile : 0xFFFFFFFFu;
    uint64_t before = 0;
    if (lane_prefix) {
      // one word per run and short chunks: each lane sums its own tile's prefix (chunk offset +
      // < CH tile counts, independent loads; lanes of one tile repeat it) — no warp-wide loop over
      // the word's distinct tiles. Only the word's first tile can have begun in an earlier word.
      const uint32_t peers = __match_any_sync(0xFFFFFFFFu, t);
      const uint32_t first = (uint32_t)__ffs(peers) - 1;
      uint64_t b0 = 0;
      if (in) {
        const uint32_t cb = t / CH * CH;
        b0 = s_coff[t / CH];
        // the < CH <= 16 tile counts before t: predicated, unrolled, so the loads go out together
        // (a rolled loop serialised them: one round trip per tile)
        uint64_t tv[15];
#pragma unroll
        for (int q = 0; q < 15; ++q) tv[q] = cb + q < t ? __ldcg(A.tk + cb + q) : 0ull;
#pragma unroll
        for (int q = 0; q < 15; ++q) b0 += tv[q];
      }
      const uint32_t sx0 = __shfl_sync(0xFFFFFFFFu, in ? A.tinfo1[t].x : 0u, 0);
      if (sx0 < base) {                            // warp-uniform (lane 0 is always in)
        uint64_t c = 0;
        for (uint64_t w = (sx0 >> 5) + lane; w < (base >> 5); w += 32) {
          uint32_t g1 = __ldcg(A.gbits + w), e1 = __ldcg(A.ebits + w);
          if (w == (sx0 >> 5)) { g1 &= ~((1u << (sx0 & 31)) - 1); e1 &= ~((1u << (sx0 & 31)) - 1); }
          c += ((uint64_t)__popc(g1) << 32) | __popc(e1);
        }
        c = warp_sum64(c);
        if (first == 0) b0 += c;                    // lane 0's tile: its lanes start at lane 0
      }
      const uint32_t msk = lt & ~((1u << first) - 1);
      before = b0 + (((uint64_t)__popc(gw & msk)) << 32) + __popc(ew & msk);
    }
    uint32_t pend = lane_prefix ? 0u : __ballot_sync(0xFFFFFFFFu, in);
    uint32_t last_t = 0xFFFFFFFFu;
    uint64_t last_before = 0;
    while (pend) {                                 // warp-uniform: each distinct tile of this word
      const int l0 = __ffs(pend) - 1;
      const uint32_t tt = __shfl_sync(0xFFFFFFFFu, t, l0);
      const uint32_t same = __ballot_sync(0xFFFFFFFFu, t == tt);
      pend &= ~same;
      uint64_t b0;                                 // packed count before this word's first lane of tt
      if (tt == cur_t) {
        b0 = cur_before;
      } else {
        b0 = tile_prefix(tt);
        const uint32_t sx = A.tinfo1[tt].x;
        if (sx < base) {                           // only at the range start: the segment began earlier
          uint64_t c = 0;
          for (uint64_t w = (sx >> 5) + lane; w < (base >> 5); w += 32) {
            uint32_t g1 = __ldcg(A.gbits + w), e1 = __ldcg(A.ebits + w);
            if (w == (sx >> 5)) { g1 &= ~((1u << (sx & 31)) - 1); e1 &= ~((1u << (sx & 31)) - 1); }
            c += ((uint64_t)__popc(g1) << 32) | __popc(e1);
          }
          b0 += warp_sum64(c);
        }
      }
      const uint32_t lanes_lt_first = (1u << l0) - 1;   // tt's lanes are contiguous from l0
      if ((same >> lane) & 1u) {
        const uint32_t msk = lt & ~lanes_lt_first;
        before = b0 + (((uint64_t)__popc(gw & msk)) << 32) + __popc(ew & msk);
      }
      last_t = tt;
      last_before = b0 + (((uint64_t)__popc(gw & same)) << 32) + __popc(ew & same);
    }
    if (!lane_prefix) {
      cur_t = last_t;                              // the word's last tile may continue
      cur_before = last_before;
    }
    const bool isg = in && ((gw >> lane) & 1u), ise = in && ((ew >> lane) & 1u);
    const uint64_t gtb = before >> 32, eqb = before & 0xFFFFFFFFull;
    if (isg || (ise && eqb < m)) {
      const uint64_t pos = gtb + (eqb < m ? eqb : m);
      out_idx[pos] = idx;
      if constexpr (VBF16) reinterpret_cast<__nv_bfloat16*>(out_val)[pos] = __float2bfloat16_rn(a);
      else reinterpret_cast<float*>(out_val)[pos] = a;
    } else if (ise) {
      r[idx] = a;                                  // a tie beyond the m kept: keeps all of a
    }
  }
  }
}

template <bool VBF16>
__global__ void __launch_bounds__(kThreads, 4) select_kernel(SelArgs A) {
  cg::grid_group grid = cg::this_grid();
  __shared__ __align__(16) uint8_t s_raw[2 * 4 * kTile];    // general: histogram | recovery overlay
  __shared__ uint64_t s_scan[2][kThreads / 32];
  uint32_t* sh = reinterpret_cast<uint32_t*>(s_raw);
  Ctl* ctl = A.ctl;
  if (ctl->small_done) return;                     // the one-CTA select did this call (uniform)
  SEL_STAMP(0);
  const uint64_t n = A.n, k = A.k;
  const uint32_t cap = A.cap, num_tiles = A.num_tiles;
  const uint32_t cc = ctl->cand_count;
  const uint32_t T = ctl->t_est, FS = ctl->fine_shift;
  // the candidate set the select runs on: the first pass's, unless it missed
  const uint32_t* cidx = A.cidx1;
  const float* cval = A.cval1;
  const uint2* tinfo = A.tinfo1;
  const uint32_t* hfirst = A.hc;
  uint64_t N = cc;
  uint32_t mode = 0;
  if (cc >= k && cc <= cap) {
    uint64_t above;
    const int bst = find_bin_desc<bins(0)>(A.hc, k, &above, s_scan[0], sh);
    const uint32_t inb = bst >= 0 ? __ldcg(A.hc + bst) : ~0u;
    if (A.fast && bst >= 0 && bst < 4095 && FS <= 12 && inb <= cap) {
      fast_select<VBF16>(A, T, FS, (uint32_t)bst, above, cc, s_raw, s_scan[0], grid);
      SEL_STAMP(7);
      return;
    }
  }
  if (cc < k || cc > cap) {                        // recovery (uniform)
    float* s_ov = reinterpret_cast<float*>(s_raw + 4 * kTile);
    __shared__ uint32_t s_bits[kTile / 32];
    __shared__ uint32_t s_base[2];
    __shared__ uint32_t s_t2;
    bool try_rescan = true;
    if (cc > cap) {
      // too many: the k-th key's bin in the exact fine histogram of ALL candidates
      uint64_t above;
      const int bk = find_bin_desc<bins(0)>(A.hc, k, &above, s_scan[0]);
      const uint64_t lo_edge = bk < 0 ? 0ull : (uint64_t)T + ((uint64_t)bk << FS);
      const uint64_t cnt = bk < 0 ? ~0ull : above + __ldcg(A.hc + bk);
      if (threadIdx.x == 0) s_t2 = (uint32_t)(lo_edge < 0x7FFFFFFFull ? lo_edge : 0x7FFFFFFFull);
      try_rescan = cnt <= cap;
    } else {
      // too few: a stratified sample of the keys (the first pass's candidates read as their
      // as-if-selected residual: a bias of < k keys, covered by the 2x margin; exhaustive
      // sampling asks for the k - cc still missing instead). Warm calls (T finite) also histogram
      // the sampled keys in the eighth below T finely, relative to T: in error-feedback steady
      // state the keys pile up right below the threshold, and the k-th key usually missed T by a
      // hair, so T2 is placed where the sample counts max(2 (k - cc), 64 samples' worth) keys in
      // [T2, T) — the coarse bins alone put T2 percents lower, past the candidate capacity (C5
      // with a 4-gradient cycle: 3 of 6 rescans overflowed into the full-array select).
      const bool warm = T < 0x7F800000u;
      const uint32_t t_lo = warm ? (__float_as_uint(__uint_as_float(T) * 0.875f) & 0x7FFFFFFFu) : 0u;
      uint32_t sf = 0;
      while (warm && (4096ull << sf) < (uint64_t)(T - t_lo)) ++sf;
      uint32_t* shf = reinterpret_cast<uint32_t*>(s_raw + 4 * kTile);   // (the overlay space, free here)
      for (int j = threadIdx.x; j < bins(0); j += kThreads) { sh[j] = 0; shf[j] = 0; }
      __syncthreads();
      sample_accumulate(A.r, n, A.num_micro, A.stride, A.phase, A.exhaustive, sh,
                        blockIdx.x * kThreads + threadIdx.x, gridDim.x * kThreads,
                        warm ? shf : nullptr, T, t_lo, sf);
      __syncthreads();
      for (int j = threadIdx.x; j < bins(0); j += kThreads) {
        if (sh[j]) atomicAdd(A.hs + j, sh[j]);
        if (shf[j]) atomicAdd(A.hl + j, shf[j]);
      }
      grid.sync();
      uint32_t t2 = threshold_from_sample(A.hs, n, k, k - cc, 2.0, A.num_micro, A.exhaustive, s_scan[0]);
      if (t2 >= T) t2 = __float_as_uint(__uint_as_float(T) * 0.875f) & 0x7FFFFFFFu;
      if (warm) {
        // fine placement: bin 4095 - j of hl counts sampled keys in [T - (j+1) 2^sf, T - j 2^sf);
        // the bin holding the need-th sampled key below T, from the top
        const uint64_t S = A.exhaustive ? n : (uint64_t)A.num_micro * 8;
        uint64_t need = (uint64_t)(2.0 * (double)(k - cc) * (double)S / (double)n) + 1;
        if (need < 64) need = 64;
        uint64_t above;
        const int bf = find_bin_desc<bins(0)>(A.hl, need, &above, s_scan[0]);
        if (bf >= 0) {
          const uint64_t tf = (uint64_t)T - ((uint64_t)(4096 - bf) << sf);
          const uint32_t tfine = tf > t_lo ? (uint32_t)tf : t_lo;
          if (tfine > t2) t2 = tfine;              // the finer (higher) of the two placements
        }
      }
      if (threadIdx.x == 0) s_t2 = t2;
    }
    __syncthreads();
    uint32_t T2 = s_t2;
    if (A.force_t2 != kNoForce) T2 = A.force_t2;   // test hook
    if (try_rescan) {
      rescan(A, T2, VBF16 ? 1 : 0, s_ov, s_bits, sh, s_scan, s_base);
      grid.sync();
      const uint32_t cc2 = __ldcg(&ctl->cand_count2);
      if (cc2 >= k && cc2 <= cap) {
        cidx = A.cidx2; cval = A.cval2; tinfo = A.tinfo2; hfirst = A.hc2; N = cc2; mode = 2;
      } else {
        restore_recorded(A.r, A.tinfo2, A.cidx2, A.cval2, num_tiles, cap);
        mode = 1;
      }
    } else {
      restore_recorded(A.r, A.tinfo1, A.cidx1, A.cval1, num_tiles, cap);
      mode = 1;
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) ctl->t2 = T2;
    if (mode == 1) { N = n; grid.sync(); }
  }
  const float* src = mode == 1 ? A.r : cval;
  uint32_t prefix = 0;
  uint64_t need = k;
  // the rescan built its set's first-digit histogram; the first pass's is relative to T (fine)
  select_pass<0>(src, N, sh, mode == 2 ? const_cast<uint32_t*>(hfirst) : A.h0, prefix, need, s_scan[0], grid,
                 mode != 2);
  select_pass<1>(src, N, sh, A.h1, prefix, need, s_scan[0], grid);
  select_pass<2>(src, N, sh, A.h2, prefix, need, s_scan[0], grid);
  const uint32_t K = prefix;
  const uint64_t m = need;                         // K*-ties to keep (lowest indices first)
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    ctl->mode = mode;
    ctl->kstar = K;
    ctl->m = m;
    state_update(A.st, A.sk, k, cap, cc, mode, K, ctl->nonfinite);
  }
  // ---- fused ordered emission ----
  // A streaming tile's candidates sit contiguously in the buffer, in index order (candidate modes),
  // or the tile is its own 4096 residual elements (full mode). A group of g lanes (a power of two
  // covering the mean segment length, 4..32) owns one tile at a time:
  //  (A) per tile: (count > K*, count == K*) over its segment -> tcnt[t]
  //  (B) exclusive scan of tcnt over tiles (block chunks + block offsets)
  //  (C) per tile again: ballot prefixes inside the segment give each kept candidate its slot
  // output position of a kept candidate = (# > K* before it) + min(# == K* before it, m).
  const uint32_t G = gridDim.x, b = blockIdx.x, lane = threadIdx.x & 31;
  uint32_t ts_log = 0;
  while (((uint64_t)G << ts_log) < num_tiles) ++ts_log;
  uint32_t glog = 2;
  while (glog < 5 && ((uint64_t)num_tiles << glog) < N) ++glog;
  float* r = A.r;
  const float* vsrc = mode == 1 ? r : cval;
  auto segment = [&](uint64_t t) -> uint2 {      // (first buffer position, length) of tile t
    if (mode != 1) return tinfo[t];
    const uint64_t b0 = t * kTile;
    return make_uint2((uint32_t)b0, (uint32_t)((n - b0) < (uint64_t)kTile ? n - b0 : kTile));
  };
  const uint32_t g = 1u << glog, gl = lane & (g - 1), gshift = lane & ~(g - 1);
  const uint32_t gmask = g == 32 ? 0xFFFFFFFFu : ((1u << g) - 1);
  const uint64_t tpw = 32u >> glog;                // tiles per warp per round
  const uint64_t wstride = (uint64_t)G * (kThreads / 32) * tpw;
  const uint64_t tfirst = (((uint64_t)b * kThreads + threadIdx.x) >> 5) * tpw + (lane >> glog);
  uint64_t* tcnt = A.tloc;
  uint64_t* boff = A.boff;
  // (A)
  for (uint64_t tw = tfirst - (lane >> glog); tw < num_tiles; tw += wstride) {   // warp-uniform
    const uint64_t t = tw + (lane >> glog);
    const uint2 ti = t < num_tiles ? segment(t) : make_uint2(0u, 0u);
    uint32_t gt = 0, eq = 0;
#pragma unroll 4
    for (uint32_t j = gl; j < ti.y; j += g) {
      const uint32_t key = mag_key(vsrc[(uint64_t)ti.x + j]);
      gt += key > K;
      eq += key == K;
    }
    for (uint32_t o = g >> 1; o; o >>= 1) {        // reduce inside the group
      gt += __shfl_xor_sync(0xFFFFFFFFu, gt, o);
      eq += __shfl_xor_sync(0xFFFFFFFFu, eq, o);
    }
    if (gl == 0 && t < num_tiles) tcnt[t] = ((uint64_t)gt << 32) | eq;
  }
  grid.sync();
  // (B)
  const uint64_t t0 = (uint64_t)b << ts_log, t1 = (t0 + (1ull << ts_log) < num_tiles) ? t0 + (1ull << ts_log) : num_tiles;
  const uint64_t ttot = t0 < t1 ? chunk_scan(t0, t1, [&](uint64_t t) { return tcnt[t]; }, tcnt, s_scan[0]) : 0;
  if (threadIdx.x == 0) boff[b] = ttot;
  grid.sync();
  const uint64_t toff = block_offset(boff, s_scan[0]);
  __syncthreads();
  if (threadIdx.x == 0) boff[G + b] = toff;
  grid.sync();
  // (C)
  uint8_t* pairs = A.pairs;
  uint32_t* out_idx = reinterpret_cast<uint32_t*>(pairs);
  uint8_t* out_val = pairs + pad16(4 * k);
  if (b == 0 && threadIdx.x < 16) {                // zero the 16-byte padding of both sections
    const uint64_t ip = 4 * k, ie = pad16(4 * k);
    if (ip + threadIdx.x < ie) pairs[ip + threadIdx.x] = 0;
    const uint64_t vp = pad16(4 * k) + (VBF16 ? 2 : 4) * k, ve = pad16(4 * k) + pad16((VBF16 ? 2 : 4) * k);
    if (vp + threadIdx.x < ve) pairs[vp + threadIdx.x] = 0;
  }
  const uint32_t lt = (1u << gl) - 1;
  // the next round's tile (segment, prefix) is loaded while the current one is emitted, and the
  // group's loads of two iterations are issued together: the loop is load-latency bound
  auto tinfo_at = [&](uint64_t tw, uint2& ti, uint64_t& tp) {
    const uint64_t t = tw + (lane >> glog);
    const bool tv = t < num_tiles;
    ti = tv ? segment(t) : make_uint2(0u, 0u);
    tp = tv ? tcnt[t] + __ldcg(boff + G + (t >> ts_log)) : 0;
  };
  uint64_t tw = tfirst - (lane >> glog);
  uint2 ti = make_uint2(0u, 0u);
  uint64_t tp = 0;
  if (tw < num_tiles) tinfo_at(tw, ti, tp);
  for (; tw < num_tiles; tw += wstride) {          // warp-uniform
    uint2 nti = make_uint2(0u, 0u);
    uint64_t ntp = 0;
    if (tw + wstride < num_tiles) tinfo_at(tw + wstride, nti, ntp);
    uint64_t gtb = tp >> 32, eqb = tp & 0xFFFFFFFFull;
    const uint32_t len_max = __reduce_max_sync(0xFFFFFFFFu, ti.y);
    for (uint32_t j0 = 0; j0 < len_max; j0 += 2 * g) {
      float a2[2];
      uint32_t id2[2];
      bool in2[2];
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const uint32_t j = j0 + h * g + gl;
        in2[h] = j < ti.y;
        a2[h] = in2[h] ? vsrc[(uint64_t)ti.x + j] : 0.f;
        id2[h] = in2[h] ? (mode == 1 ? ti.x + j : cidx[(uint64_t)ti.x + j]) : 0u;
      }
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        if (j0 + h * g >= len_max) break;          // warp-uniform
        const float a = a2[h];
        const uint32_t idx = id2[h];
        const bool in = in2[h];
        const uint32_t key = mag_key(a);
        const bool isg = in && key > K, ise = in && key == K;
        const uint32_t bg = (__ballot_sync(0xFFFFFFFFu, isg) >> gshift) & gmask;
        const uint32_t be = (__ballot_sync(0xFFFFFFFFu, ise) >> gshift) & gmask;
        const uint64_t myeq = eqb + __popc(be & lt);
        if (isg || (ise && myeq < m)) {
          const uint64_t pos = gtb + __popc(bg & lt) + (myeq < m ? myeq : m);
          out_idx[pos] = idx;
          if constexpr (VBF16) {
            const __nv_bfloat16 hb = __float2bfloat16_rn(a);
            reinterpret_cast<__nv_bfloat16*>(out_val)[pos] = hb;
            if (mode == 1) r[idx] = a - __bfloat162float(hb);   // exact (Sterbenz), reading #8
          } else {
            reinterpret_cast<float*>(out_val)[pos] = a;
            if (mode == 1) r[idx] = 0.0f;
          }
        } else if (in && mode != 1) {
          r[idx] = a;                              // a rejected candidate keeps all of a
        }
        gtb += __popc(bg);
        eqb += __popc(be);
      }
    }
    ti = nti;
    tp = ntp;
  }
}


// ---- K2': small problems (<= 2^15 candidates): the same select + ordered emission in ONE CTA ----
// The grid kernel's ~10 dependent phases each pay a grid barrier; for a few thousand candidates
// (C1) one CTA does every phase behind __syncthreads. Work is split by candidate-buffer position:
//   digits : shared-memory histograms of the candidates (12 bits from the stream pass, 10, 9)
//   S      : exclusive prefix P(j) over buffer positions of packed (key > K*, key == K*); a tile's
//            candidates are one contiguous segment, so P at its first and one-past-last position
//            bound its counts
//   B      : exclusive scan of the per-tile counts in index order
//   C      : candidate j of tile t: (# > K* before it) = tile offset + P_gt(j) - P_gt(seg start),
//            likewise for ties; kept iff key > K* or a tie among the first m -> slot; rejected
//            candidates get r = a back (the stream pass stored them as selected).
__device__ __forceinline__ uint64_t small_block_scan(uint64_t x, uint64_t* smem, uint64_t* total) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint64_t incl = x;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint64_t y = __shfl_up_sync(0xFFFFFFFFu, incl, o);
    if (lane >= o) incl += y;
  }
  if (lane == 31) smem[warp] = incl;
  __syncthreads();
  if (warp == 0) {
    const uint64_t v = smem[lane];
    uint64_t w = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint64_t y = __shfl_up_sync(0xFFFFFFFFu, w, o);
      if (lane >= o) w += y;
    }
    smem[lane] = w - v;                            // exclusive warp offsets
    if (lane == 31) smem[32] = w;
  }
  __syncthreads();
  const uint64_t r = smem[warp] + incl - x;
  *total = smem[32];
  __syncthreads();
  return r;
}

// the bin of the need-th largest key (1-based) of a shared-memory histogram
template <int NB>
__device__ __forceinline__ int small_find(const uint32_t* h, uint64_t need, uint64_t* above_out, uint64_t* smem) {
  __shared__ int s_bin;
  __shared__ uint64_t s_above;
  constexpr int PER = NB >= kSmallThreads ? NB / kSmallThreads : 1;
  const bool act = (int)threadIdx.x * PER < NB;
  const int lo = NB - ((int)threadIdx.x + 1) * PER;
  uint32_t c[PER];
  uint64_t sum = 0;
#pragma unroll
  for (int q = 0; q < PER; ++q) {
    c[q] = act ? h[lo + q] : 0u;
    sum += c[q];
  }
  if (threadIdx.x == 0) { s_bin = -1; s_above = 0; }
  uint64_t total;
  uint64_t above = small_block_scan(sum, smem, &total);
  if (act && above < need && above + sum >= need) {
#pragma unroll
    for (int q = PER - 1; q >= 0; --q) {
      if (above + c[q] >= need) { s_bin = lo + q; s_above = above; break; }
      above += c[q];
    }
  }
  __syncthreads();
  *above_out = s_bin < 0 ? total : s_above;
  return s_bin;
}

template <bool VBF16>
__global__ void __launch_bounds__(kSmallThreads, 1)
select_small_kernel(float* __restrict__ r, uint64_t k, Ctl* ctl, const float* __restrict__ cand_val,
                    const uint32_t* __restrict__ cand_idx, const uint2* __restrict__ tile_info,
                    uint32_t num_tiles, uint32_t cap, const uint32_t* __restrict__ hc,
                    uint64_t* __restrict__ toff, ulonglong2* __restrict__ seg, uint64_t* __restrict__ pj,
                    uint8_t* __restrict__ pairs, State* st, StateKey sk) {
  const uint32_t cc = ctl->cand_count;
  if (!(cc >= k && cc <= cap && cc <= kSmallMaxCand)) return;   // the grid kernel does this call
  __shared__ uint32_t s_h0[bins(0)], s_h1[bins(1)], s_h2[bins(2)];
  __shared__ uint64_t s_scan[33];
  const uint32_t tid = threadIdx.x, lane = tid & 31;
  for (int b = tid; b < bins(0); b += kSmallThreads) s_h0[b] = 0;
  for (int b = tid; b < bins(1); b += kSmallThreads) s_h1[b] = 0;
  for (int b = tid; b < bins(2); b += kSmallThreads) s_h2[b] = 0;
  __syncthreads();
  uint64_t need = k, above;
  auto digit = [&](uint32_t* sh, int NBITS, uint32_t pfx, int pshift, int dshift) {
    for (uint32_t jw = tid & ~31u; jw < cc; jw += kSmallThreads) {   // warp-uniform trip count
      const uint32_t j = jw + lane;
      const uint32_t key = j < cc ? mag_key(cand_val[j]) : 0xFFFFFFFFu;
      const bool take = key != 0xFFFFFFFFu && (key >> pshift) == pfx;
      const uint32_t act = __ballot_sync(0xFFFFFFFFu, take);
      if (take) {                                  // lanes with the same bin: one shared atomic
        const uint32_t bin = (key >> dshift) & ((1u << NBITS) - 1);
        const uint32_t peers = __match_any_sync(act, bin);
        if (lane == __ffs(peers) - 1) atomicAdd(&sh[bin], (uint32_t)__popc(peers));
      }
    }
    __syncthreads();
  };
  // Warm first pass: the stream pass's histogram is fine and relative to T, so the k-th key's bin
  // b* is found there and ONE pass over the candidates in b* (their low s key bits) gives K*.
  const uint32_t T = ctl->t_est, FS = ctl->fine_shift;
  uint32_t K;
  bool fine = false;
  if (FS <= 12) {
    for (int b = tid; b < bins(0); b += kSmallThreads) s_h0[b] = __ldcg(hc + b);
    __syncthreads();
    const int bst = small_find<bins(0)>(s_h0, need, &above, s_scan);
    fine = bst >= 0 && bst < 4095;                 // (uniform) K* below the top (overflow) bin
    if (fine) {
      need -= above;
      __syncthreads();
      for (int b = tid; b < bins(0); b += kSmallThreads) s_h0[b] = 0;
      __syncthreads();
      const uint32_t lowmask = (1u << FS) - 1;
      for (uint32_t jw = tid & ~31u; jw < cc; jw += kSmallThreads) {   // warp-uniform trip count
        const uint32_t j = jw + lane;
        const uint32_t key = j < cc ? mag_key(cand_val[j]) : 0u;
        const bool take = j < cc && fine_bin(key, T, FS) == (uint32_t)bst;
        const uint32_t act = __ballot_sync(0xFFFFFFFFu, take);
        if (take) {
          const uint32_t bin = (key - T) & lowmask;
          const uint32_t peers = __match_any_sync(act, bin);
          if (lane == __ffs(peers) - 1) atomicAdd(&s_h0[bin], (uint32_t)__popc(peers));
        }
      }
      __syncthreads();
      const uint32_t d = (uint32_t)small_find<bins(0)>(s_h0, need, &above, s_scan);
      need -= above;
      K = T + ((uint32_t)bst << FS) + d;
    } else {
      need = k;
      __syncthreads();
      for (int b = tid; b < bins(0); b += kSmallThreads) s_h0[b] = 0;
      __syncthreads();
    }
  }
  if (!fine) {                                     // the general 3-digit radix select
    digit(s_h0, 12, 0u, 31, shift(0));
    const uint32_t d0 = (uint32_t)small_find<bins(0)>(s_h0, need, &above, s_scan);
    need -= above;
    digit(s_h1, 10, d0, shift(0), shift(1));
    const uint32_t d1 = (uint32_t)small_find<bins(1)>(s_h1, need, &above, s_scan);
    need -= above;
    const uint32_t p1 = (d0 << 10) | d1;
    digit(s_h2, 9, p1, shift(1), shift(2));
    const uint32_t d2 = (uint32_t)small_find<bins(2)>(s_h2, need, &above, s_scan);
    need -= above;
    K = (p1 << 9) | d2;
  }
  const uint64_t m = need;                         // K*-ties to keep (lowest indices first)
  if (tid == 0) {
    ctl->mode = 0; ctl->kstar = K; ctl->m = m; ctl->small_done = 1;
    state_update(st, sk, k, cap, cc, 0, K, ctl->nonfinite);
  }
  auto flag = [&](uint32_t j) -> uint64_t {        // packed (key > K*, key == K*) of position j
    const uint32_t key = mag_key(cand_val[j]);
    return ((uint64_t)(key > K) << 32) | (uint64_t)(key == K);
  };
  // S: P(j) over buffer positions, chunks of kSmallThreads x 4; segment boundaries record P
  constexpr int kU = 4;
  uint64_t base = 0;
  for (uint32_t c0 = 0; c0 < cc; c0 += kSmallThreads * kU) {
    uint64_t f[kU], sum = 0;
    uint32_t ti[kU];
    const uint32_t jf = c0 + tid * kU;
    const uint32_t tbefore = (jf == 0 || jf > cc) ? 0xFFFFFFFFu : cand_idx[jf - 1] / kTile;
    const uint32_t tafter = jf + kU >= cc ? 0xFFFFFFFFu : cand_idx[jf + kU] / kTile;
#pragma unroll
    for (int u = 0; u < kU; ++u) {
      const uint32_t j = jf + u;
      f[u] = j < cc ? flag(j) : 0;
      ti[u] = j < cc ? cand_idx[j] / kTile : 0xFFFFFFFFu;
      sum += f[u];
    }
    uint64_t ctot;
    uint64_t run = base + small_block_scan(sum, s_scan, &ctot);
#pragma unroll
    for (int u = 0; u < kU; ++u) {
      const uint32_t j = jf + u;
      if (j < cc) {
        pj[j] = run;
        const uint32_t tprev = u ? ti[u - 1] : tbefore;
        const uint32_t tnext = u < kU - 1 ? ti[u + 1] : tafter;
        if (tprev != ti[u]) seg[ti[u]].x = run;                     // P at the segment's start
        if (tnext != ti[u]) seg[ti[u]].y = run + f[u];              // P one past its end
      }
      run += f[u];
    }
    base += ctot;
  }
  __syncthreads();
  // B: exclusive scan of the per-tile (gt, eq) counts in tile order
  auto tcount = [&](uint32_t t) -> uint64_t {
    if (tile_info[t].y == 0) return 0;
    const ulonglong2 sg = seg[t];
    return sg.y - sg.x;
  };
  base = 0;
  for (uint32_t c0 = 0; c0 < num_tiles; c0 += kSmallThreads * kU) {
    uint64_t v[kU], sum = 0;
#pragma unroll
    for (int u = 0; u < kU; ++u) {
      const uint32_t t = c0 + tid * kU + u;
      v[u] = t < num_tiles ? tcount(t) : 0;
      sum += v[u];
    }
    uint64_t ctot;
    uint64_t run = base + small_block_scan(sum, s_scan, &ctot);
#pragma unroll
    for (int u = 0; u < kU; ++u) {
      const uint32_t t = c0 + tid * kU + u;
      if (t < num_tiles) toff[t] = run;
      run += v[u];
    }
    base += ctot;
  }
  __syncthreads();
  // C: emission
  uint32_t* out_idx = reinterpret_cast<uint32_t*>(pairs);
  uint8_t* out_val = pairs + pad16(4 * k);
  if (tid < 16) {                                  // zero the 16-byte padding of both sections
    const uint64_t ip = 4 * k, ie = pad16(4 * k);
    if (ip + tid < ie) pairs[ip + tid] = 0;
    const uint64_t vp = pad16(4 * k) + (VBF16 ? 2 : 4) * k, ve = pad16(4 * k) + pad16((VBF16 ? 2 : 4) * k);
    if (vp + tid < ve) pairs[vp + tid] = 0;
  }
  for (uint32_t j = tid; j < cc; j += kSmallThreads) {
    const float a = cand_val[j];
    const uint32_t idx = cand_idx[j], t = idx / kTile, key = mag_key(a);
    const uint64_t before = toff[t] + (pj[j] - seg[t].x);        // packed (# > K*, # == K*) before j
    const uint64_t gtb = before >> 32, eqb = before & 0xFFFFFFFFull;
    if (key > K || (key == K && eqb < m)) {
      const uint64_t pos = gtb + (eqb < m ? eqb : m);
      out_idx[pos] = idx;
      if constexpr (VBF16) reinterpret_cast<__nv_bfloat16*>(out_val)[pos] = __float2bfloat16_rn(a);
      else reinterpret_cast<float*>(out_val)[pos] = a;
    } else {
      r[idx] = a;                                  // a rejected candidate keeps all of a
    }
  }
}

int g_stream_blocks_f32 = 0, g_stream_blocks_bf16 = 0;
uint32_t g_force_t = kNoForce;          // test hooks: override the first-pass / rescan thresholds
uint32_t g_force_t2 = kNoForce;

int device_sms() {
  static int sms = 0;
  if (!sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || sms < 1) sms = kNumSMs;
  }
  return sms;
}

int g_tma_blocks_f32 = 0, g_tma_blocks_bf16 = 0;
int stream_tma_smem(bool bf16) { return kStages * kTile * ((bf16 ? 2 : 4) + 4); }
int stream_tma_blocks(bool bf16) {
  int& cache = bf16 ? g_tma_blocks_bf16 : g_tma_blocks_f32;
  if (!cache) {
    const int smem = stream_tma_smem(bf16);
    int per_sm = 0;
    if (bf16) {
      cudaFuncSetAttribute(stream_tma_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, stream_tma_kernel<true>, kThreads, smem);
    } else {
      cudaFuncSetAttribute(stream_tma_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, stream_tma_kernel<false>, kThreads, smem);
    }
    cache = (per_sm > 0 ? per_sm : 1) * device_sms();
  }
  return cache;
}

int stream_blocks(bool bf16) {
  int& cache = bf16 ? g_stream_blocks_bf16 : g_stream_blocks_f32;
  if (!cache) {
    int per_sm = 0;
    if (bf16) cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, stream_kernel<true>, kThreads, 0);
    else cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, stream_kernel<false>, kThreads, 0);
    cache = (per_sm > 0 ? per_sm : 4) * device_sms();
  }
  return cache;
}

const void* select_fn(bool vbf) {
  return vbf ? (const void*)select_kernel<true> : (const void*)select_kernel<false>;
}

// CTAs per SM the cooperative select may use: its occupancy limit over all four variants
int select_max_per_sm() {
  static int sel_max = 0;
  if (!sel_max) {
    sel_max = kMaxSelectBlocks;
    for (int q = 0; q < 2; ++q) {
      int a = 0;
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&a, select_fn(q), kThreads, 0);
      if (a < sel_max) sel_max = a;
    }
    if (sel_max < 1) sel_max = 1;
    const int cap = kMaxSelectBlocks / device_sms();
    if (sel_max > (cap < 1 ? 1 : cap)) sel_max = cap < 1 ? 1 : cap;
  }
  return sel_max;
}

}  // namespace

uint64_t compress_ws_bytes(uint64_t n, uint64_t k) { return layout(n, k).total; }

void compress_force_threshold(int which, int enable, uint32_t key) {
  (which == 0 ? g_force_t : g_force_t2) = enable ? key : kNoForce;
}

lowdiff_status compress_stats(const void* ws, uint64_t n, uint64_t k, uint64_t out[10], cudaStream_t s) {
  const Layout L = layout(n, k);
  Ctl c;
  LD_CUDA(cudaMemcpyAsync(&c, static_cast<const uint8_t*>(ws) + L.ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, s),
          "stats copy");
  LD_CUDA(cudaStreamSynchronize(s), "stats sync");
  out[0] = c.t_est; out[1] = c.cand_count; out[2] = c.mode; out[3] = c.kstar; out[4] = c.m;
  out[5] = L.cap;
  out[6] = c.fine_shift;
  out[7] = c.inbin_count;
  out[8] = c.t2;
  out[9] = c.cand_count2;
  return LOWDIFF_OK;
}

lowdiff_status compress_counters(const void* ws, cudaStream_t s, uint64_t out[9]) {
  State st;
  LD_CUDA(cudaMemcpyAsync(&st, ws, sizeof(State), cudaMemcpyDeviceToHost, s), "counters copy");
  LD_CUDA(cudaStreamSynchronize(s), "counters sync");
  if (st.magic != kStateMagic) {
    for (int i = 0; i < 9; ++i) out[i] = 0;
    return LOWDIFF_OK;
  }
  out[0] = st.calls; out[1] = st.rescans; out[2] = st.fallbacks; out[3] = st.nonfinite_calls;
  out[4] = st.last_nonfinite; out[5] = st.last_cand; out[6] = st.kstar;
  out[7] = (uint64_t)((double)st.delta * 4294967296.0);     // delta in 2^-32 units
  out[8] = st.fast_calls;
  return LOWDIFF_OK;
}

lowdiff_status compress_run(const void* grad, int gdt, float* residual, uint64_t n, uint64_t k,
                            void* pairs, int vdt, void* ws, cudaStream_t s) {
  const Layout L = layout(n, k);
  uint8_t* w = static_cast<uint8_t*>(ws);
  Ctl* ctl = reinterpret_cast<Ctl*>(w + L.ctl);
  State* st = reinterpret_cast<State*>(w + L.state);
  LD_CUDA(cudaMemsetAsync(w + L.ctl, 0, L.zero_end - L.ctl, s), "memset compress workspace");
  // the margin controller's band of first-pass candidates / k (measured: scripts/band_sweep.sh,
  // profiles/r02/band.txt): 1.05-1.5 k; 1.02-1.2 k for large, dense selections (k >= 2^20 and
  // k >= n/200) — each rejected candidate costs a scattered residual store, ~0.8 M per call at C4
  // (C4 659 -> 643 us per call). Sparser selections lose to extra rescans with the tight band (C5:
  // 49 rescans in 1,200 error-feedback calls instead of 1-4; C2, C3 slower).
  // LOWDIFF_CAND_BAND="lo,hi" overrides (experiments).
  static float env_lo = -1.f, env_hi = -1.f;
  if (env_lo < 0.f) {
    env_lo = env_hi = 0.f;
    if (const char* e = getenv("LOWDIFF_CAND_BAND")) {
      float a = 0.f, b = 0.f;
      if (sscanf(e, "%f,%f", &a, &b) == 2 && a >= 1.0f && b > a) { env_lo = a; env_hi = b; }
    }
  }
  const bool big_k = k >= (1ull << 20) && 200 * k >= n;
  const float band_lo = env_lo > 0.f ? env_lo : (big_k ? 1.02f : 1.05f);
  const float band_hi = env_lo > 0.f ? env_hi : (big_k ? 1.2f : 1.5f);
  const StateKey sk{n, k, (uint64_t)(uintptr_t)residual, (uint64_t)(gdt | (vdt << 8)), band_lo, band_hi};

  // recovery sample size: >= 512 expected keys above the k-th (S >= 512 n / k: the 2x target is
  // then > 10 sigma of the count above k), >= 64 Ki, power of 2; every micro-chunk when S >= n/2
  uint64_t S = 65536;
  while ((double)S * (double)k < 512.0 * (double)n && S < (1ull << 26)) S <<= 1;
  const int exhaustive = (S >= n / 2) ? 1 : 0;
  const uint32_t micro = exhaustive ? (uint32_t)((n + 7) / 8) : (uint32_t)(S / 8);
  const double stride = exhaustive ? 1.0 : (double)(n / 8) / (double)micro;
  static uint64_t calls = 0;                       // per-call phase (golden-ratio sequence)
  const double phase = exhaustive ? 0.0 : (double)((++calls * 0x9E3779B97F4A7C15ull) >> 11) * 0x1p-53;
  static int use_tma = -1;
  if (use_tma < 0) {
    const char* e = getenv("LOWDIFF_STREAM_TMA");
    use_tma = e ? atoi(e) : 0;
  }

  uint2* tiles = reinterpret_cast<uint2*>(w + L.tiles);
  uint32_t* cidx = reinterpret_cast<uint32_t*>(w + L.cand_idx);
  float* cval = reinterpret_cast<float*>(w + L.cand_val);
  const bool bf = gdt == LOWDIFF_BF16;
  const int vbf = vdt == LOWDIFF_BF16 ? 1 : 0;
  uint32_t* hcand = reinterpret_cast<uint32_t*>(w + L.hc);
  uint64_t* tk = reinterpret_cast<uint64_t*>(w + L.tk);
  if (use_tma) {
    int grid = stream_tma_blocks(bf);
    if ((uint32_t)grid > L.num_tiles) grid = (int)L.num_tiles;
    const int smem = stream_tma_smem(bf);
    if (bf)
      LD_LAUNCH("compress_stream", s, stream_tma_kernel<true>, grid, kThreads, smem, grad, residual, n,
                L.num_tiles, ctl, tiles, cidx, cval, L.cap, vbf, hcand, tk, st, sk, g_force_t);
    else
      LD_LAUNCH("compress_stream", s, stream_tma_kernel<false>, grid, kThreads, smem, grad, residual, n,
                L.num_tiles, ctl, tiles, cidx, cval, L.cap, vbf, hcand, tk, st, sk, g_force_t);
  } else {
    int grid = stream_blocks(bf);
    if ((uint32_t)grid > L.num_tiles) grid = (int)L.num_tiles;
    if (bf)
      LD_LAUNCH("compress_stream", s, stream_kernel<true>, grid, kThreads, 0, grad, residual, n,
                L.num_tiles, ctl, tiles, cidx, cval, L.cap, vbf, hcand, tk, st, sk, g_force_t);
    else
      LD_LAUNCH("compress_stream", s, stream_kernel<false>, grid, kThreads, 0, grad, residual, n,
                L.num_tiles, ctl, tiles, cidx, cval, L.cap, vbf, hcand, tk, st, sk, g_force_t);
  }

  const int sel_max = select_max_per_sm();
  // CTAs per SM: more hide the latency of the emission loop at large k, fewer make the grid
  // syncs and histogram flushes cheaper at small k (measured, profiles/README.md; round 2 with the
  // fast select: 3 per SM for 2^14 <= k < 2^18, C2 74.8 -> 73.1 us, C3 289 -> 287.1 us per call;
  // C1's k = 2697 keeps 2: 19.1 vs 20.5 us)
  int want = k >= (1u << 18) ? 4 : (k >= (1u << 14) ? 3 : 2);
  if (const char* e = getenv("LOWDIFF_SELECT_PER_SM")) want = atoi(e);
  if (want < 1) want = 1;
  if (want > sel_max) want = sel_max;
  int sel_grid = want * device_sms();
  if (sel_grid > kMaxSelectBlocks) sel_grid = kMaxSelectBlocks;
  if (const char* e = getenv("LOWDIFF_SELECT_GRID")) {   // experiments: explicit CTA count
    const int gq = atoi(e);
    if (gq >= 1 && gq <= sel_max * device_sms() && gq <= kMaxSelectBlocks) sel_grid = gq;
  }
  SelArgs A;
  A.r = residual; A.n = n; A.k = k; A.ctl = ctl; A.st = st; A.sk = sk;
  A.cidx1 = cidx; A.cval1 = cval; A.tinfo1 = tiles;
  A.cidx2 = reinterpret_cast<uint32_t*>(w + L.cand2_idx);
  A.cval2 = reinterpret_cast<float*>(w + L.cand2_val);
  A.tinfo2 = reinterpret_cast<uint2*>(w + L.tiles2);
  A.num_tiles = L.num_tiles; A.cap = L.cap;
  A.hs = reinterpret_cast<uint32_t*>(w + L.hs);
  A.hc = hcand;
  A.hc2 = reinterpret_cast<uint32_t*>(w + L.hc2);
  A.h0 = reinterpret_cast<uint32_t*>(w + L.h0);
  A.h1 = reinterpret_cast<uint32_t*>(w + L.h1);
  A.h2 = reinterpret_cast<uint32_t*>(w + L.h2);
  A.tloc = reinterpret_cast<uint64_t*>(w + L.tloc);
  A.tk = tk;
  A.ctot = reinterpret_cast<uint64_t*>(w + L.ctot);
  A.hl = reinterpret_cast<uint32_t*>(w + L.hl);
  A.gbits = reinterpret_cast<uint32_t*>(w + L.bits);
  A.ebits = A.gbits + (L.cap / 32 + 1);
  A.inbin = reinterpret_cast<uint64_t*>(w + L.inbin);
  {
    const uint32_t q = (L.num_tiles + 32u * kMaxChunks - 1) / (32u * kMaxChunks);
    A.chunk_tiles = 32u * (q ? q : 1u);            // dense tiles; fast_select picks finer for sparse
    A.num_chunks = (L.num_tiles + A.chunk_tiles - 1) / A.chunk_tiles;
  }
  A.boff = reinterpret_cast<uint64_t*>(w + L.boff);
  A.pairs = static_cast<uint8_t*>(pairs);
  A.num_micro = micro; A.stride = stride; A.phase = phase; A.exhaustive = exhaustive;
  A.force_t2 = g_force_t2;
  static int use_fast = -1;
  if (use_fast < 0) {
    const char* e = getenv("LOWDIFF_FAST_SELECT");
    use_fast = e ? atoi(e) : 1;
  }
  A.fast = use_fast;
  ProfScope prof("compress_select", s);
  // the one-CTA select for tiny k: opt-in (LOWDIFF_SELECT_SMALL=1, read per call); measured, the
  // grid select is faster even at C1 (20.2 vs 21.7 us per compress call, graph-timed)
  const char* use_small_env = getenv("LOWDIFF_SELECT_SMALL");
  const int use_small = use_small_env ? atoi(use_small_env) : 0;
  if (use_small && 4 * k <= kSmallMaxCand) {   // a few thousand candidates: one CTA does it all
    ulonglong2* seg = reinterpret_cast<ulonglong2*>(w + L.seg);
    uint64_t* pj = reinterpret_cast<uint64_t*>(w + L.pj);
    if (vbf)
      select_small_kernel<true><<<1, kSmallThreads, 0, s>>>(residual, k, ctl, cval, cidx, tiles, L.num_tiles, L.cap,
                                                             hcand, A.tloc, seg, pj, A.pairs, st, sk);
    else
      select_small_kernel<false><<<1, kSmallThreads, 0, s>>>(residual, k, ctl, cval, cidx, tiles, L.num_tiles, L.cap,
                                                              hcand, A.tloc, seg, pj, A.pairs, st, sk);
    note_launch();
  }
  void* args[] = {(void*)&A};
  LD_CUDA(cudaLaunchCooperativeKernel(select_fn(vbf), sel_grid, kThreads, args, 0, s), "select launch");
  note_launch();
#ifdef LOWDIFF_SEL_TIMING
  {
    static uint64_t when = 0;
    if (!when) { const char* e = getenv("LOWDIFF_SEL_TIMING_CALL"); when = e ? strtoull(e, nullptr, 10) : 410; }
    sel_timing_print<<<1, 1, 0, s>>>(st, (uint32_t)sel_grid, when);
  }
#endif
  return cuda_status(cudaGetLastError(), "compress launch");
}

}  // namespace lowdiff
