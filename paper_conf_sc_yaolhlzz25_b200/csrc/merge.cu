// Multiway index merge engine (sm_100a) — serves two steps of the path:
//   * coalesce after the sparse all-gather: Sync(G~_{i,t}) (Alg.1 line 5)
//       P rank lists -> sorted unique union in [lo, hi), rank-ascending fp32 fold, / P
//   * batch merge of B differentials (§4.2 Step 2; "tensor addition or dictionary
//       accumulation") -> one record (SUM: iteration-ascending fold; STACK: per-index
//       iteration lists)
//
// Sort-free design. The index range [lo, hi) is cut into fine windows of
// W = 4096 consecutive parameter indices.
//   K2a  starts: for every list, the position of each fine window's first entry (one streaming
//        pass over the entries).
//   K2p  plan: consecutive fine windows are grouped G at a time (G from the host's density
//        estimate, ~1K entries per group); a group whose entry count fits the shared-memory
//        capacity becomes one "sparse" work item, a heavier group is split into its fine windows
//        ("dense" items). Items are in index order.
//   K2b  merge: persistent, ticket-ordered CTAs take one item each.
//        sparse item: the lists' entries are loaded to shared memory and each entry's position
//          in (index, list) order is computed by binary searches in the other lists' segments
//          (the lists are sorted); runs of equal indices are folded in list order.
//        dense item: the entries are folded into a W-slot shared-memory accumulator list by
//          list, so the fp32 fold order is the definition's (rank / iteration ascending) with
//          no float atomics, and occupied slots are compacted in index order.
//        Items are independent: each writes its entries (STACK) at their final positions (the
//        item's entry offset is the sum of its lists' start positions) and its unique heads to a
//        staging array at that same offset.
//   K2q  scan of the items' unique counts;  K2m  compaction of the staged heads.
//   K2c  pack: sections -> the byte-exact record (header | lr[] | idx | val  or  off | it | val).
#include "common.cuh"
#include "internal.h"
#include "starts.cuh"

namespace lowdiff {
namespace {

constexpr int kW = 4096;                    // parameter indices per fine window
constexpr int kSlotsPerThread = kW / kThreads;
constexpr int kCap = 2048;                  // entries a sparse item may hold (shared memory)
constexpr int kPosPerThread = kCap / kThreads;
constexpr int kPlanThreads = 1024;

struct __align__(256) MCtl {
  uint32_t ticket;
  uint32_t num_items;
  uint64_t nnz;      // unique indices (written by the scan kernel)
  uint64_t nent;     // entries (written by the scan kernel)
};

// Workspace. The merge kernel writes each item's unique heads into staging arrays at the item's
// ENTRY offset (known from the starts table alone, so items need no ordering between them); a
// scan over the items' unique counts and a compaction then place them densely.
struct MLayout {
  uint64_t ctl, ebnd, zero_end, starts, items, ucnt, epre, upre, sidx, sval, wit, went, total;
  uint32_t num_w;
};

MLayout mlayout(int L, uint64_t max_entries, uint64_t lo, uint64_t hi, bool record) {
  MLayout M;
  M.num_w = (uint32_t)((hi - lo + kW - 1) / kW);
  uint64_t o = 0;
  M.ctl = o;    o += align256(sizeof(MCtl));
  M.zero_end = o;
  M.ebnd = o;   o += align256(8ull * L);         // per-list entry range of [lo, hi) (coalesce)
  M.starts = o; o += align256(4ull * L * (M.num_w + 1));
  M.items = o;  o += align256(8ull * M.num_w);
  M.ucnt = o;   o += align256(4ull * M.num_w);   // unique count per item
  M.epre = o;   o += align256(4ull * M.num_w);   // entry offset per item
  M.upre = o;   o += align256(4ull * M.num_w);   // unique offset per item (scan)
  M.sidx = o;   o += align256(4 * max_entries);  // staged heads: idx
  M.sval = o;   o += align256(4 * max_entries);  // staged heads: value (SUM/coalesce) or off (STACK)
  M.wit = M.went = 0;
  if (record) {                                   // entries at their record order (STACK); the heads
                                                  // are compacted straight into the record
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

// ---- K2p: work-item plan (one CTA) -----------------------------------------------------------------
// items[i] = (first fine window, number of fine windows).
__global__ void __launch_bounds__(kPlanThreads) plan_kernel(int L, const uint32_t* __restrict__ starts,
                                                            uint32_t num_w, uint32_t G, uint32_t sparse_max,
                                                            int keep_groups, MCtl* ctl, uint2* __restrict__ items,
                                                            uint32_t* __restrict__ gcnt) {
  __shared__ uint64_t s_scan[kPlanThreads / 32];
  const int tid = threadIdx.x;
  const uint32_t num_g = (num_w + G - 1) / G;
  if (keep_groups) {                               // bitmap-sized groups stay whole: item g = group g
    for (uint32_t g = tid; g < num_g; g += kPlanThreads)
      items[g] = make_uint2(g * G, (g * G + G < num_w ? G : num_w - g * G));
    if (tid == 0) ctl->num_items = num_g;
    return;
  }
  // per group (block-strided: every thread's loads in flight at once) the entry count decides
  // whole / split into windows -> gcnt; then each thread sums a contiguous chunk of gcnt, one block
  // scan places every item (index order)
  auto count = [&](uint32_t g) -> uint32_t {
    const uint32_t fs = g * G, fe = fs + G < num_w ? fs + G : num_w;
    uint64_t e = 0;
    int l = 0;
    for (; l + 4 <= L; l += 4) {                   // 8 independent loads in flight
      uint32_t a2[4], b2[4];
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const uint32_t* st = starts + (uint64_t)(l + q) * (num_w + 1);
        a2[q] = st[fe]; b2[q] = st[fs];
      }
#pragma unroll
      for (int q = 0; q < 4; ++q) e += a2[q] - b2[q];
    }
    for (; l < L; ++l) {
      const uint32_t* st = starts + (uint64_t)l * (num_w + 1);
      e += st[fe] - st[fs];
    }
    return (e <= (uint64_t)sparse_max || fe - fs == 1) ? 1u : fe - fs;
  };
  for (uint32_t g = tid; g < num_g; g += kPlanThreads) gcnt[g] = count(g);
  __syncthreads();
  const uint32_t per = (num_g + kPlanThreads - 1) / kPlanThreads;
  const uint32_t g0 = tid * per, g1 = g0 + per < num_g ? g0 + per : num_g;
  uint32_t mine = 0;
  for (uint32_t g = g0; g < g1; ++g) mine += gcnt[g];
  uint64_t tot;
  uint32_t off = (uint32_t)block_exclusive_scan_n<kPlanThreads>(mine, s_scan, &tot);
  for (uint32_t g = g0; g < g1; ++g) {
    const uint32_t cnt = gcnt[g], fs = g * G, fe = fs + G < num_w ? fs + G : num_w;
    if (cnt == 1) items[off] = make_uint2(fs, fe - fs);
    else
      for (uint32_t q = 0; q < cnt; ++q) items[off + q] = make_uint2(fs + q, 1u);
    off += cnt;
  }
  if (tid == 0) ctl->num_items = (uint32_t)tot;
}

// ---- K2b: item merge ------------------------------------------------------------------------------
struct DenseSmem {
  float acc[kW];                 // SUM: running fold; STACK: slot entry cursor (u32)
  uint32_t cnt[kW];              // entries per slot
};
struct SparseSmem {
  uint64_t sk[2][kCap];          // (idx - w0) << 40 | list << 32 | load position; merge ping-pong
};
constexpr int kBmLists = 32;                // lists the bitmap path handles
constexpr int kWords = kW / 32;             // bitmap words per fine window
constexpr int kBmWords = 4096;              // list x word capacity of a bitmap item (16 KB)
constexpr int kBmMaxWords = 512;            // words (4 windows) per bitmap item
struct BitmapSmem {
  uint32_t bm[kBmWords];           // per list, the item's occupied slots (list-major)
  uint64_t wpre[kBmMaxWords];      // per word: (# unique slots before it) << 32 | # entries before it
  uint4 pl[kBmMaxWords];           // per word, L <= 15: bit planes of the per-slot list count
                                   // (x = 1s, y = 2s, z = 4s, w = 8s); L > 15: x = slots of any list
};
union ItemSmem {
  DenseSmem d;
  SparseSmem s;
  BitmapSmem b;
};

#ifndef LOWDIFF_MERGE_MINB
#define LOWDIFF_MERGE_MINB 6                    // CTAs per SM the item engine is compiled for (37 KB smem each)
#endif
template <int KIND, bool BF16>
__global__ void __launch_bounds__(kThreads, LOWDIFF_MERGE_MINB) merge_kernel(const __grid_constant__ ListSet ls, uint64_t lo,
                                                         uint32_t num_w, const uint32_t* __restrict__ starts,
                                                         const uint2* __restrict__ items, MCtl* ctl,
                                                         uint32_t* __restrict__ ucnt, uint32_t* __restrict__ epre,
                                                         uint32_t* __restrict__ stg_idx,
                                                         uint32_t* __restrict__ stg_val,
                                                         uint8_t* __restrict__ out_it,
                                                         float* __restrict__ out_ent, uint32_t sparse_max,
                                                         uint32_t bitmap_min) {
  __shared__ ItemSmem sm;
  __shared__ uint32_t s_beg[kMaxLists], s_len[kMaxLists], s_off[kMaxLists + 1];
  __shared__ uint64_t s_scan[kThreads / 32];
  __shared__ uint32_t s_ticket, s_e0;
  const int tid = threadIdx.x;
  const int L = ls.L;
  const uint32_t num_items = ctl->num_items;
  for (int j = tid; j < kW; j += kThreads) sm.d.cnt[j] = 0;
  bool dense_clean = true;                         // cnt[] is all zero
  while (true) {
    if (tid == 0) s_ticket = atomicAdd(&ctl->ticket, 1u);
    __syncthreads();
    const uint32_t item = s_ticket;
    if (item >= num_items) break;
    const uint2 it = items[item];
    const uint64_t w0 = lo + (uint64_t)it.x * kW;
    // per-list segments of this item; their prefix (list order); the item's entry offset
    uint32_t len = 0, beg = 0;
    if (tid < L) {
      const uint32_t* st = starts + (uint64_t)tid * (num_w + 1);
      beg = st[it.x];
      len = st[it.x + it.y] - beg;
      s_beg[tid] = beg;
      s_len[tid] = len;
    }
    uint64_t tot_e;
    const uint64_t packed = block_exclusive_scan(((uint64_t)beg << 32) | len, s_scan, &tot_e);
    if (tid < L) s_off[tid] = (uint32_t)packed;
    if (tid == 0) {
      s_off[L] = (uint32_t)tot_e;
      s_e0 = (uint32_t)(tot_e >> 32);              // sum over lists of the item's first position
    }
    __syncthreads();
    const uint32_t E = (uint32_t)tot_e;
    const uint32_t e0 = s_e0;
    uint64_t tot;
    auto list_of = [&](uint32_t x) -> int {        // list l with s_off[l] <= x < s_off[l+1]
      int a = 0, b = L - 1;
      while (a < b) {
        const int mid = (a + b + 1) >> 1;
        if (s_off[mid] <= x) a = mid; else b = mid - 1;
      }
      return a;
    };
    const uint32_t NW = it.y * kWords;            // bitmap words of this item
    const bool bm_shape = KIND == kMergeStack && L <= kBmLists && (uint32_t)L * NW <= (uint32_t)kBmWords &&
                          NW <= (uint32_t)kBmMaxWords;
    if (bm_shape && (E >= bitmap_min * it.y || (E > sparse_max && it.y > 1))) {
      // ---- bitmap item (STACK, dense enough): per list a bitmap of the item's occupied slots;
      //      per word the (unique, entry) counts and their exclusive scan; then every entry finds
      //      its final position with popcounts alone:
      //        pos = e0 + entries in earlier words + entries of this word at lower slots
      //              + lists before its own with the same slot (iteration order)
      //      and the first entry of a slot (rank 0) writes the unique head. No sorting.
      for (uint32_t j = tid; j < (uint32_t)L * NW; j += kThreads) sm.b.bm[j] = 0;
      __syncthreads();
      // warp w walks lists w, w + 8, ... (no per-entry list lookup; round 2: the binary search over
      // the lists' offsets was ~20 % of the kernel's issue slots), 4 entries per lane in flight
      const int bw_warp = tid >> 5, bw_lane = tid & 31;
      for (int l = bw_warp; l < L; l += kThreads / 32) {
        const uint32_t* li = ls.list[l].idx + s_beg[l];
        const uint32_t len = s_len[l];
        for (uint32_t j0 = bw_lane; j0 < len; j0 += 128) {
          uint32_t sl[4];
#pragma unroll
          for (int u = 0; u < 4; ++u) sl[u] = j0 + 32 * u < len ? li[j0 + 32 * u] - (uint32_t)w0 : 0xFFFFFFFFu;
#pragma unroll
          for (int u = 0; u < 4; ++u)
            if (sl[u] != 0xFFFFFFFFu) atomicOr(&sm.b.bm[l * NW + (sl[u] >> 5)], 1u << (sl[u] & 31));
        }
      }
      __syncthreads();
      // each thread owns q consecutive words: their counts, a block scan, then the per-word prefix.
      // Up to 15 lists the word's per-slot list counts are kept as 4 bit planes (a carry-save sum of
      // the lists' bitmaps), so an entry's count of entries at lower slots of its word is 4
      // popcounts instead of a loop over the lists, and only a slot held by >= 2 lists walks the
      // lists for its iteration rank (round 2; C4: ~2 % of the slots)
      const bool planes = L <= 15;
      constexpr int kQ = (kBmMaxWords + kThreads - 1) / kThreads;
      const uint32_t q = (NW + kThreads - 1) / kThreads, w_a = tid * q, w_e = min(NW, w_a + q);
      uint64_t cw[kQ];
      uint64_t mine = 0;
#pragma unroll
      for (int i = 0; i < kQ; ++i) {
        const uint32_t wd = w_a + i;
        cw[i] = 0;
        if (wd >= w_e) continue;
        uint32_t c, u;
        if (planes) {
          uint32_t p0 = 0, p1 = 0, p2 = 0, p3 = 0;
          for (int l = 0; l < L; ++l) {
            const uint32_t b = sm.b.bm[l * NW + wd];
            const uint32_t c0 = p0 & b;
            p0 ^= b;
            const uint32_t c1 = p1 & c0;
            p1 ^= c0;
            const uint32_t c2 = p2 & c1;
            p2 ^= c1;
            p3 ^= c2;
          }
          sm.b.pl[wd] = make_uint4(p0, p1, p2, p3);
          c = __popc(p0) + 2 * __popc(p1) + 4 * __popc(p2) + 8 * __popc(p3);
          u = __popc(p0 | p1 | p2 | p3);
        } else {
          uint32_t orv = 0;
          c = 0;
          for (int l = 0; l < L; ++l) {
            const uint32_t bw = sm.b.bm[l * NW + wd];
            orv |= bw;
            c += __popc(bw);
          }
          sm.b.pl[wd].x = orv;
          u = __popc(orv);
        }
        cw[i] = ((uint64_t)u << 32) | c;
        mine += cw[i];
      }
      uint64_t run = block_exclusive_scan(mine, s_scan, &tot);
#pragma unroll
      for (int i = 0; i < kQ; ++i) {
        if (w_a + i >= w_e) continue;
        sm.b.wpre[w_a + i] = run;
        run += cw[i];
      }
      __syncthreads();
      for (int a = bw_warp; a < L; a += kThreads / 32) {   // the same walk: list a's entries
        const uint64_t eb = s_beg[a];
        const uint32_t* li = ls.list[a].idx + eb;
        const uint32_t len = s_len[a];
        for (uint32_t j0 = bw_lane; j0 < len; j0 += 128) {   // 4 entries' (idx, val) loads in flight
        uint32_t sl[4];
        float vv[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const uint32_t e = j0 + 32 * u;
          sl[u] = e < len ? li[e] - (uint32_t)w0 : 0xFFFFFFFFu;
          vv[u] = e < len ? list_val<BF16>(ls, a, eb + e) : 0.f;
        }
#pragma unroll
        for (int u = 0; u < 4; ++u) {
        if (sl[u] == 0xFFFFFFFFu) break;
        const uint32_t slot = sl[u];
        const uint32_t wd = slot >> 5, bit = 1u << (slot & 31), below = bit - 1u;
        uint32_t cb = 0, rank = 0, orw;
        if (planes) {
          const uint4 P = sm.b.pl[wd];
          cb = __popc(P.x & below) + 2 * __popc(P.y & below) + 4 * __popc(P.z & below) + 8 * __popc(P.w & below);
          orw = P.x | P.y | P.z | P.w;
          if ((P.y | P.z | P.w) & bit)             // a slot of >= 2 lists: its lists before this one
            for (int l = 0; l < a; ++l) rank += (sm.b.bm[l * NW + wd] & bit) ? 1u : 0u;
        } else {
          for (int l = 0; l < L; ++l) {
            const uint32_t bw = sm.b.bm[l * NW + wd];
            cb += __popc(bw & below);
            rank += (l < a && (bw & bit)) ? 1u : 0u;
          }
          orw = sm.b.pl[wd].x;
        }
        const uint64_t pw = sm.b.wpre[wd];
        const uint32_t pos = e0 + (uint32_t)pw + cb + rank;
        out_it[pos] = (uint8_t)a;
        out_ent[pos] = vv[u];
        if (rank == 0) {
          const uint32_t uu = e0 + (uint32_t)(pw >> 32) + __popc(orw & below);
          stg_idx[uu] = (uint32_t)(w0 + slot);
          stg_val[uu] = pos;                       // off[] = the head's entry position
        }
        }
        }
      }
      tot >>= 32;                                  // unique slots of the item
      dense_clean = false;                         // the bitmap arrays alias cnt[]
    } else if (E <= sparse_max) {
      // ---- sparse item: load the lists' segments (each sorted by index) as runs of unique
      //      composite keys (index, list), then merge runs pairwise, ceil(log2 L) rounds: a key's
      //      rank in the merged run = its rank in its own run + the number of smaller keys in the
      //      partner run (binary search). Equal indices end up in list (rank / iteration) order.
      for (uint32_t x = tid; x < E; x += kThreads) {
        int a = 0, b = L - 1;                      // list l with s_off[l] <= x < s_off[l+1]
        while (a < b) {
          const int mid = (a + b + 1) >> 1;
          if (s_off[mid] <= x) a = mid; else b = mid - 1;
        }
        const uint64_t e = s_beg[a] + (x - s_off[a]);
        const uint32_t key = ls.list[a].idx[e] - (uint32_t)w0;
        sm.s.sk[0][x] = ((uint64_t)key << 40) | ((uint64_t)a << 32) | x;
      }
      __syncthreads();
      int cur = 0;
      for (int w = 1; w < L; w <<= 1, cur ^= 1) {  // runs of w lists -> runs of 2w lists
        const uint64_t* A = sm.s.sk[cur];
        uint64_t* Bo = sm.s.sk[cur ^ 1];
        for (uint32_t x = tid; x < E; x += kThreads) {
          const uint64_t key = A[x];
          const int q = (int)((key >> 32) & 0xFFu) / w;   // own run
          const int pq = q ^ 1;                            // partner run
          const uint32_t own_s = s_off[q * w];
          const uint32_t ps = s_off[pq * w < L ? pq * w : L];
          const uint32_t pe = s_off[(pq + 1) * w < L ? (pq + 1) * w : L];
          uint32_t pos = ps, len = pe - ps;               // lower_bound of key in A[ps, pe)
          while (len > 0) {
            const uint32_t half = len >> 1;
            if (A[pos + half] < key) { pos += half + 1; len -= half + 1; } else { len = half; }
          }
          Bo[s_off[(q & ~1) * w] + (x - own_s) + (pos - ps)] = key;
        }
        __syncthreads();
      }
      const uint64_t* S = sm.s.sk[cur];
      auto val_of = [&](uint64_t skr) -> float {  // the value of a key, from its list (L2-warm)
        const int l = (int)((skr >> 32) & 0xFFu);
        return list_val<BF16>(ls, l, s_beg[l] + ((uint32_t)skr - s_off[l]));
      };
      uint32_t my_u = 0;
#pragma unroll
      for (int j = 0; j < kPosPerThread; ++j) {
        const uint32_t r = tid * kPosPerThread + j;
        if (r < E && (r == 0 || (S[r - 1] >> 40) != (S[r] >> 40))) ++my_u;
      }
      uint32_t u = e0 + (uint32_t)block_exclusive_scan(my_u, s_scan, &tot);
#pragma unroll
      for (int j = 0; j < kPosPerThread; ++j) {
        const uint32_t r = tid * kPosPerThread + j;
        if (r >= E) break;
        const uint64_t skr = S[r];
        const uint32_t key = (uint32_t)(skr >> 40);
        const bool head = r == 0 || (S[r - 1] >> 40) != key;
        if (KIND == kMergeStack) {
          if (head) {
            stg_idx[u] = (uint32_t)(w0 + key);
            stg_val[u] = e0 + r;                   // off[] = the head's entry position
            ++u;
          }
          out_it[e0 + r] = (uint8_t)(skr >> 32);
          out_ent[e0 + r] = val_of(skr);
        } else if (head) {
          float sum = val_of(skr);                 // fold the run in list order
          for (uint32_t r2 = r + 1; r2 < E && (S[r2] >> 40) == key; ++r2)
            sum = sum + val_of(S[r2]);
          stg_idx[u] = (uint32_t)(w0 + key);
          stg_val[u] = __float_as_uint(sum);
          ++u;
        }
      }
      dense_clean = false;                         // the sparse arrays alias cnt[]
    } else {
      // ---- dense item: exactly one fine window, any number of entries ----
      if (!dense_clean) {
        for (int j = tid; j < kW; j += kThreads) sm.d.cnt[j] = 0;
        __syncthreads();
      }
      if (KIND == kMergeStack) {
        for (int l = 0; l < L; ++l)                // integer counts: order-free
          for (uint32_t e = s_beg[l] + tid; e < s_beg[l] + s_len[l]; e += kThreads)
            atomicAdd(&sm.d.cnt[ls.list[l].idx[e] - w0], 1u);
      } else {
        for (int l = 0; l < L; ++l) {              // fp32 fold in list (rank/iteration) order
          if (s_len[l] == 0) continue;             // block-uniform
          for (uint32_t e = s_beg[l] + tid; e < s_beg[l] + s_len[l]; e += kThreads) {
            const uint32_t slot = ls.list[l].idx[e] - (uint32_t)w0;
            const float v = list_val<BF16>(ls, l, e);
            const uint32_t c = sm.d.cnt[slot];
            sm.d.acc[slot] = c ? sm.d.acc[slot] + v : v;
            sm.d.cnt[slot] = c + 1;
          }
          __syncthreads();
        }
      }
      __syncthreads();
      uint64_t my_u = 0, my_e = 0;
#pragma unroll
      for (int j = 0; j < kSlotsPerThread; ++j) {
        const uint32_t c = sm.d.cnt[tid * kSlotsPerThread + j];
        my_u += c ? 1 : 0;
        my_e += c;
      }
      const uint64_t local = block_exclusive_scan((my_u << 32) | my_e, s_scan, &tot);
      uint32_t u = e0 + (uint32_t)(local >> 32);
      uint32_t e = e0 + (uint32_t)local;
      tot >>= 32;
#pragma unroll 4
      for (int j = 0; j < kSlotsPerThread; ++j) {
        const int slot = tid * kSlotsPerThread + j;
        const uint32_t c = sm.d.cnt[slot];
        if (!c) continue;
        stg_idx[u] = (uint32_t)(w0 + slot);
        if (KIND == kMergeStack) {
          stg_val[u] = e;                                             // off[]
          reinterpret_cast<uint32_t*>(sm.d.acc)[slot] = e;            // entry cursor
        } else {
          stg_val[u] = __float_as_uint(sm.d.acc[slot]);
        }
        ++u;
        e += c;
      }
      if (KIND == kMergeStack) {
        __syncthreads();
        for (int l = 0; l < L; ++l) {              // entries in iteration order per slot
          if (s_len[l] == 0) continue;
          for (uint32_t x = s_beg[l] + tid; x < s_beg[l] + s_len[l]; x += kThreads) {
            const uint32_t slot = ls.list[l].idx[x] - (uint32_t)w0;
            const uint32_t pos = reinterpret_cast<uint32_t*>(sm.d.acc)[slot];
            out_it[pos] = (uint8_t)l;
            out_ent[pos] = list_val<BF16>(ls, l, x);
            reinterpret_cast<uint32_t*>(sm.d.acc)[slot] = pos + 1;
          }
          __syncthreads();
        }
      }
#pragma unroll
      for (int j = 0; j < kSlotsPerThread; ++j) sm.d.cnt[tid * kSlotsPerThread + j] = 0;
      dense_clean = true;
    }
    if (tid == 0) {
      ucnt[item] = (uint32_t)tot;
      epre[item] = e0;
    }
    __syncthreads();
  }
}

// ---- K2q: exclusive scan of the items' unique counts; totals (one CTA) ------------------------
__global__ void __launch_bounds__(kPlanThreads) ucount_scan_kernel(const __grid_constant__ ListSet ls,
                                                                   uint32_t num_w,
                                                                   const uint32_t* __restrict__ starts,
                                                                   MCtl* ctl, const uint32_t* __restrict__ ucnt,
                                                                   uint32_t* __restrict__ upre,
                                                                   uint64_t* d_out_nnz) {
  __shared__ uint64_t s_scan[kPlanThreads / 32];
  const int tid = threadIdx.x;
  const uint32_t num_items = ctl->num_items;
  // each thread a contiguous chunk of items (4 loads in flight), one block scan of the chunk sums
  const uint32_t per = (num_items + kPlanThreads - 1) / kPlanThreads;
  const uint32_t i0 = tid * per, i1 = i0 + per < num_items ? i0 + per : num_items;
  uint32_t mine = 0;
  for (uint32_t i = i0; i < i1; i += 4) {
    uint32_t v[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) v[q] = i + q < i1 ? ucnt[i + q] : 0u;
#pragma unroll
    for (int q = 0; q < 4; ++q) mine += v[q];
  }
  uint64_t tot;
  uint32_t run = (uint32_t)block_exclusive_scan_n<kPlanThreads>(mine, s_scan, &tot);
  for (uint32_t i = i0; i < i1; i += 4) {
    uint32_t v[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) v[q] = i + q < i1 ? ucnt[i + q] : 0u;
#pragma unroll
    for (int q = 0; q < 4; ++q)
      if (i + q < i1) { upre[i + q] = run; run += v[q]; }
  }
  if (tid == 0) {
    uint64_t nent = 0;
    for (int l = 0; l < ls.L; ++l) {
      const uint32_t* st = starts + (uint64_t)l * (num_w + 1);
      nent += st[num_w] - st[0];
    }
    ctl->nnz = tot;
    ctl->nent = nent;
    if (d_out_nnz) *d_out_nnz = tot;
  }
}

// ---- K2m: compaction of the staged heads (one warp per item) ----------------------------------
__global__ void __launch_bounds__(kThreads) compact_kernel(const MCtl* ctl, const uint32_t* __restrict__ ucnt,
                                                           const uint32_t* __restrict__ epre,
                                                           const uint32_t* __restrict__ upre,
                                                           const uint32_t* __restrict__ stg_idx,
                                                           const uint32_t* __restrict__ stg_val,
                                                           float inv_div, int divide, uint32_t* __restrict__ out_idx,
                                                           uint32_t* __restrict__ out_val, uint8_t* __restrict__ rec,
                                                           uint64_t rec_cap, uint32_t B, int stack) {
  const uint32_t num_items = ctl->num_items;
  if (rec) {
    // batch merge (round 2): the heads go straight to the record's idx and val/off sections, whose
    // offsets are known once the unique count is (ucount_scan_kernel ran before); the packer then
    // only writes the header, lr[], the padding, off[nnz] and the entry sections
    const uint64_t nnz = ctl->nnz, nent = ctl->nent;
    const uint64_t o_idx = 80 + pad16(4ull * B), o_v = o_idx + pad16(4 * nnz);
    const uint64_t total = stack ? o_v + pad16(4 * (nnz + 1)) + pad16(nent) + pad16(4 * nent)
                                 : o_v + pad16(4 * nnz);
    if (total > rec_cap) return;                     // the packer reports the size; nothing is written
    out_idx = reinterpret_cast<uint32_t*>(rec + o_idx);
    out_val = reinterpret_cast<uint32_t*>(rec + o_v);
  }
  const int lane = threadIdx.x & 31;
  (void)inv_div;
  for (uint32_t i = (blockIdx.x * kThreads + threadIdx.x) >> 5; i < num_items; i += (gridDim.x * kThreads) >> 5) {
    const uint32_t c = ucnt[i], src = epre[i], dst = upre[i];
    for (uint32_t x0 = 0; x0 < c; x0 += 128) {       // 4 loads in flight per lane
      uint32_t iv[4], vv[4];
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const uint32_t x = x0 + q * 32 + lane;
        if (x < c) { iv[q] = stg_idx[src + x]; vv[q] = stg_val[src + x]; }
      }
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const uint32_t x = x0 + q * 32 + lane;
        if (x >= c) break;
        uint32_t v = vv[q];
        if (divide) v = __float_as_uint(__fdiv_rn(__uint_as_float(v), inv_div));   // "/ P" (coalesce)
        out_idx[dst + x] = iv[q];
        out_val[dst + x] = v;
      }
    }
  }
}

// ---- K2s: coalesce of a single list (P = 1): the union is the list itself, /1 is exact --------
// Warp-parallel lower bound (32 probes per round) of `v` in a sorted list of `len`.
__device__ uint64_t warp_lower_bound(const uint32_t* idx, uint64_t len, uint64_t v) {
  const int lane = threadIdx.x & 31;
  uint64_t lo = 0, hi = len;                       // answer in [lo, hi]
  while (hi - lo > 32) {
    const uint64_t step = (hi - lo + 31) / 32;
    const uint64_t p = lo + (uint64_t)lane * step;
    const bool less = p < hi && (uint64_t)idx[p] < v;
    const uint32_t m = __ballot_sync(0xFFFFFFFFu, less);
    const int c = __popc(m);                       // probes below v (a prefix of the lanes)
    const uint64_t nlo = c ? lo + (uint64_t)(c - 1) * step + 1 : lo;
    const uint64_t nhi = lo + (uint64_t)c * step;
    lo = nlo;
    hi = nhi < hi ? nhi : hi;
  }
  const uint64_t p = lo + lane;
  const bool less = p < hi && (uint64_t)idx[p] < v;
  return lo + __popc(__ballot_sync(0xFFFFFFFFu, less));
}

template <bool BF16>
__global__ void __launch_bounds__(kThreads) single_list_kernel(const uint32_t* __restrict__ idx,
                                                               const void* __restrict__ val, uint64_t len,
                                                               uint64_t lo, uint64_t hi,
                                                               uint32_t* __restrict__ out_idx,
                                                               float* __restrict__ out_val,
                                                               uint64_t* d_out_nnz) {
  __shared__ uint64_t s_first, s_last;
  if (threadIdx.x < 32) {
    const uint64_t f = (len == 0 || idx[0] >= lo) ? 0 : warp_lower_bound(idx, len, lo);
    const uint64_t l = (len == 0 || idx[len - 1] < hi) ? len : warp_lower_bound(idx, len, hi);
    if (threadIdx.x == 0) {
      s_first = f;
      s_last = l;
      if (blockIdx.x == 0) *d_out_nnz = l - f;
    }
  }
  __syncthreads();
  const uint64_t first = s_first, cnt = s_last - s_first;
  uint64_t done = 0;
  if ((first & 3) == 0) {                          // aligned: 4 entries per thread, 128-bit idx I/O
    const uint64_t c4 = cnt / 4;
    for (uint64_t q = (uint64_t)blockIdx.x * kThreads + threadIdx.x; q < c4; q += (uint64_t)gridDim.x * kThreads) {
      const uint64_t e = q * 4;
      *reinterpret_cast<uint4*>(out_idx + e) = *reinterpret_cast<const uint4*>(idx + first + e);
      float v[4];
      if constexpr (BF16) {
        const uint2 u = *reinterpret_cast<const uint2*>(static_cast<const uint16_t*>(val) + first + e);
        v[0] = __uint_as_float(u.x << 16); v[1] = __uint_as_float(u.x & 0xFFFF0000u);
        v[2] = __uint_as_float(u.y << 16); v[3] = __uint_as_float(u.y & 0xFFFF0000u);
      } else {
        const float4 t = *reinterpret_cast<const float4*>(static_cast<const float*>(val) + first + e);
        v[0] = t.x; v[1] = t.y; v[2] = t.z; v[3] = t.w;
      }
      *reinterpret_cast<float4*>(out_val + e) =          // the definition's "/ P" with P = 1 (exact)
          make_float4(__fdiv_rn(v[0], 1.0f), __fdiv_rn(v[1], 1.0f), __fdiv_rn(v[2], 1.0f), __fdiv_rn(v[3], 1.0f));
    }
    done = c4 * 4;
  }
  for (uint64_t e = done + (uint64_t)blockIdx.x * kThreads + threadIdx.x; e < cnt; e += (uint64_t)gridDim.x * kThreads) {
    out_idx[e] = idx[first + e];
    float v;
    if constexpr (BF16) v = __uint_as_float(((uint32_t) static_cast<const uint16_t*>(val)[first + e]) << 16);
    else v = static_cast<const float*>(val)[first + e];
    out_val[e] = __fdiv_rn(v, 1.0f);               // the definition's "/ P" with P = 1 (exact)
  }
}

// ---- K2c: record packer ---------------------------------------------------------------------
struct PackArgs {
  uint32_t mode, B, nranks;
  uint64_t n, lo, hi, t_first, cap;
  float lr[256];
};

__global__ void __launch_bounds__(kThreads) pack_kernel(const __grid_constant__ PackArgs a, const MCtl* ctl,
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
  const uint64_t o_heads_end = a.mode == LOWDIFF_MERGE_SUM ? total : o_it;   // idx + val/off: compact_kernel
  if (blockIdx.x == 0 && threadIdx.x < 8) {        // their zero padding (whole words) and off[nnz] = nent
    uint32_t* w32 = reinterpret_cast<uint32_t*>(rec);
    const int t = threadIdx.x;
    const uint64_t e_idx = o_idx + 4 * nnz, e_v = o_v + 4 * (a.mode == LOWDIFF_MERGE_SUM ? nnz : nnz + 1);
    if (e_idx / 4 + t < o_v / 4 && t < 4) w32[e_idx / 4 + t] = 0u;
    if (t >= 4 && e_v / 4 + (t - 4) < o_heads_end / 4) w32[e_v / 4 + (t - 4)] = 0u;
    if (t == 0 && a.mode != LOWDIFF_MERGE_SUM) w32[o_v / 4 + nnz] = (uint32_t)nent;
  }
  const uint64_t chunks = total / 16;
  for (uint64_t c = (uint64_t)blockIdx.x * kThreads + threadIdx.x; c < chunks;
       c += (uint64_t)gridDim.x * kThreads) {
    const uint64_t off = c * 16;
    if (off >= o_idx && off < o_heads_end) continue;   // written by compact_kernel (+ the padding above)
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

// bytes [0, len) of a 16-byte aligned buffer <- 0
__global__ void __launch_bounds__(kThreads) zero_kernel(uint8_t* __restrict__ p, uint64_t len) {
  const uint64_t n16 = len / 16, stride = (uint64_t)gridDim.x * kThreads;
  const uint64_t t = (uint64_t)blockIdx.x * kThreads + threadIdx.x;
  for (uint64_t i = t; i < n16; i += stride) reinterpret_cast<uint4*>(p)[i] = make_uint4(0u, 0u, 0u, 0u);
  for (uint64_t i = n16 * 16 + t; i < len; i += stride) p[i] = 0;
}

lowdiff_status merge_run(const ListSet& ls, MergeKind kind, uint64_t lo, uint64_t hi, int average,
                         uint64_t max_entries, uint32_t* out_idx, float* out_val, uint64_t out_cap,
                         uint64_t* d_out_nnz, const float* lr, uint64_t n, uint64_t t_first,
                         uint32_t nranks, void* d_record, uint64_t record_cap,
                         uint64_t* d_record_bytes, void* ws, cudaStream_t s) {
  (void)out_cap;
  const bool record = kind != kCoalesce;
  if (kind == kCoalesce && ls.L == 1) {
    uint64_t g = (ls.list[0].len / 4 + kThreads - 1) / kThreads;
    if (g > 4ull * kNumSMs) g = 4ull * kNumSMs;
    if (g < 1) g = 1;
    if (ls.bf16)
      LD_LAUNCH("coalesce", s, single_list_kernel<true>, (int)g, kThreads, 0, ls.list[0].idx, ls.list[0].val,
                ls.list[0].len, lo, hi, out_idx, out_val, d_out_nnz);
    else
      LD_LAUNCH("coalesce", s, single_list_kernel<false>, (int)g, kThreads, 0, ls.list[0].idx, ls.list[0].val,
                ls.list[0].len, lo, hi, out_idx, out_val, d_out_nnz);
    return cuda_status(cudaGetLastError(), "coalesce launch");
  }
  const MLayout M = mlayout(ls.L, max_entries, lo, hi, record);
  uint8_t* w = static_cast<uint8_t*>(ws);
  MCtl* ctl = reinterpret_cast<MCtl*>(w + M.ctl);
  uint32_t* starts = reinterpret_cast<uint32_t*>(w + M.starts);
  uint2* items = reinterpret_cast<uint2*>(w + M.items);
  // zeroed by a kernel, not cudaMemsetAsync: a memset may synchronise implicitly with the device's
  // other streams, which would serialise this merge behind a peer-memory wait (lowdiff_p2p_*) of
  // another rank simulated on the same device
  {
    uint64_t g = (M.zero_end / 16 + kThreads - 1) / kThreads;
    if (g > 2ull * kNumSMs) g = 2ull * kNumSMs;
    if (g < 1) g = 1;
    LD_LAUNCH("merge_zero", s, zero_kernel, (int)g, kThreads, 0, w, M.zero_end);
  }

  uint64_t per_list = max_entries / (ls.L ? ls.L : 1) + 1;
  uint64_t gx = (per_list + kThreads - 1) / kThreads;
  if (gx > 8ull * kNumSMs) gx = 8ull * kNumSMs;
  if (gx < 1) gx = 1;
  // coalesce: the gathered lists span the whole index range, so the shard's entry range of each
  // list is found first and only it is scanned (batch merge: the lists are the shard's already)
  uint32_t* ebnd = kind == kCoalesce ? reinterpret_cast<uint32_t*>(w + M.ebnd) : nullptr;
  if (ebnd) LD_LAUNCH("starts", s, bounds_kernel, ls.L, 64, 0, ls, lo, hi, ebnd);
  bool al16 = !ebnd;
  for (int l = 0; l < ls.L && al16; ++l) al16 = (reinterpret_cast<uintptr_t>(ls.list[l].idx) & 15u) == 0;
  if (al16) {                                      // 16-byte loads, 2 steps in flight
    uint64_t g4 = (per_list / 4 + 1 + 2 * kThreads - 1) / (2 * kThreads);
    if (g4 > 8ull * kNumSMs) g4 = 8ull * kNumSMs;
    if (g4 < 1) g4 = 1;
    LD_LAUNCH("starts", s, starts4_kernel<kW>, dim3((unsigned)g4, (unsigned)ls.L), kThreads, 0, ls, lo, hi,
              M.num_w, starts);
  } else {
    LD_LAUNCH("starts", s, starts_kernel<kW>, dim3((unsigned)gx, (unsigned)ls.L), kThreads, 0, ls, lo, hi,
              M.num_w, starts, (const uint32_t*)ebnd);
  }

  // group size: up to kCap/2 entries per group at the average density (power of two); the
  // entries actually present (max_entries is a capacity) make groups smaller than this bound
  const double per_w = (double)max_entries / (double)M.num_w;
  uint32_t G = 1;
  while (G < 4096 && (double)(2 * G) * per_w <= kCap / 2) G <<= 1;     // key < 2^24
  uint32_t sparse_max = kCap;       // items with more entries take the dense (one window) path
  if (const char* e = getenv("LOWDIFF_MERGE_SPARSE_MAX")) sparse_max = (uint32_t)atoi(e);
  if (sparse_max > (uint32_t)kCap) sparse_max = kCap;
  // STACK merges of dense-enough differentials: one window per item through the bitmap path
  uint32_t bitmap_min = 96;         // entries per window from which the bitmap path is used
  if (const char* e = getenv("LOWDIFF_MERGE_BITMAP_MIN")) bitmap_min = (uint32_t)atoi(e);
  // (measured: with 32 lists the popcount work per entry grows past the sparse run merging, so
  // the bitmap path is used up to 16 lists; groups stay small enough to leave >= 4 items per CTA)
  int keep_groups = 0;
  const uint32_t merge_ctas = 6u * kNumSMs;
  if (kind == kMergeStack && ls.L <= 16 && per_w >= (double)bitmap_min) {
    G = 1;                          // groups of bitmap size: as many windows as fit (power of 2)
    uint32_t gmax = 1u << 30;                       // experiments: LOWDIFF_MERGE_BMG caps the windows per item
    if (const char* e = getenv("LOWDIFF_MERGE_BMG")) gmax = (uint32_t)atoi(e);
    while (2 * G <= gmax && 2 * G * kWords <= (uint32_t)kBmMaxWords && (uint32_t)ls.L * 2 * G * kWords <= (uint32_t)kBmWords &&
           M.num_w / (2 * G) >= 4 * merge_ctas)
      G <<= 1;
    keep_groups = 1;
  }
  LD_LAUNCH("merge_plan", s, plan_kernel, 1, kPlanThreads, 0, ls.L, starts, M.num_w, G, sparse_max, keep_groups, ctl,
            items, reinterpret_cast<uint32_t*>(w + M.ucnt));

  const int grid = (int)(M.num_w < 6u * kNumSMs ? M.num_w : 6u * kNumSMs);   // 6 CTAs/SM (37 KB smem)
  uint32_t* ucnt = reinterpret_cast<uint32_t*>(w + M.ucnt);
  uint32_t* epre = reinterpret_cast<uint32_t*>(w + M.epre);
  uint32_t* upre = reinterpret_cast<uint32_t*>(w + M.upre);
  uint32_t* sidx = reinterpret_cast<uint32_t*>(w + M.sidx);
  uint32_t* sval = reinterpret_cast<uint32_t*>(w + M.sval);
  uint8_t* oit = record ? w + M.wit : nullptr;
  float* oent = record ? reinterpret_cast<float*>(w + M.went) : nullptr;
  const char* cls = record ? "merge" : "coalesce";
  if (kind == kCoalesce && ls.bf16)
    LD_LAUNCH(cls, s, (merge_kernel<kCoalesce, true>), grid, kThreads, 0, ls, lo, M.num_w, starts, items, ctl,
              ucnt, epre, sidx, sval, oit, oent, sparse_max, bitmap_min);
  else if (kind == kCoalesce)
    LD_LAUNCH(cls, s, (merge_kernel<kCoalesce, false>), grid, kThreads, 0, ls, lo, M.num_w, starts, items, ctl,
              ucnt, epre, sidx, sval, oit, oent, sparse_max, bitmap_min);
  else if (kind == kMergeSum && ls.bf16)
    LD_LAUNCH(cls, s, (merge_kernel<kMergeSum, true>), grid, kThreads, 0, ls, lo, M.num_w, starts, items, ctl,
              ucnt, epre, sidx, sval, oit, oent, sparse_max, bitmap_min);
  else if (kind == kMergeSum)
    LD_LAUNCH(cls, s, (merge_kernel<kMergeSum, false>), grid, kThreads, 0, ls, lo, M.num_w, starts, items, ctl,
              ucnt, epre, sidx, sval, oit, oent, sparse_max, bitmap_min);
  else if (ls.bf16)
    LD_LAUNCH(cls, s, (merge_kernel<kMergeStack, true>), grid, kThreads, 0, ls, lo, M.num_w, starts, items, ctl,
              ucnt, epre, sidx, sval, oit, oent, sparse_max, bitmap_min);
  else
    LD_LAUNCH(cls, s, (merge_kernel<kMergeStack, false>), grid, kThreads, 0, ls, lo, M.num_w, starts, items, ctl,
              ucnt, epre, sidx, sval, oit, oent, sparse_max, bitmap_min);
  LD_LAUNCH(cls, s, ucount_scan_kernel, 1, kPlanThreads, 0, ls, M.num_w, starts, ctl, ucnt, upre,
            kind == kCoalesce ? d_out_nnz : nullptr);
  uint32_t* didx = record ? nullptr : out_idx;     // record: compact_kernel places the heads in it
  uint32_t* dval = record ? nullptr : reinterpret_cast<uint32_t*>(out_val);
  const int cgrid = (int)((M.num_w + 7) / 8 < 4u * kNumSMs ? (M.num_w + 7) / 8 : 4u * kNumSMs);
  LD_LAUNCH(cls, s, compact_kernel, cgrid, kThreads, 0, ctl, ucnt, epre, upre, sidx, sval, (float)ls.L,
            (kind == kCoalesce && average) ? 1 : 0, didx, dval,
            record ? static_cast<uint8_t*>(d_record) : nullptr, record ? record_cap : 0, (uint32_t)ls.L,
            kind == kMergeStack ? 1 : 0);
  if (kind == kCoalesce) return cuda_status(cudaGetLastError(), "coalesce launch");

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
  LD_LAUNCH("merge_pack", s, pack_kernel, (int)pg, kThreads, 0, pa, ctl, w + M.wit, reinterpret_cast<const uint32_t*>(w + M.went), static_cast<uint8_t*>(d_record),
            d_record_bytes);
  return cuda_status(cudaGetLastError(), "merge launch");
}

}  // namespace lowdiff
