// Shared device/host helpers of liblowdiff (sm_100a). Not part of the ABI.
#pragma once
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <stdint.h>

#include "lowdiff.h"

namespace lowdiff {

constexpr int kThreads = 256;              // block size of every streaming kernel
constexpr int kNumSMs = 148;               // B200

__host__ __device__ inline uint64_t pad16(uint64_t x) { return (x + 15u) & ~(uint64_t)15u; }

// |a| as an ordered u32 key: sign dropped, so +0 == -0 (reading #3).
__device__ __forceinline__ uint32_t mag_key(float a) { return __float_as_uint(a) & 0x7FFFFFFFu; }

// ---- memory-order helpers (decoupled look-back) ------------------------------------------
__device__ __forceinline__ void st_release(uint64_t* p, uint64_t v) {
  asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t ld_acquire(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ float4 ld_stream_f4(const float4* p) {   // read once: no L1 allocate
  float4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w) : "l"(p));
  return r;
}
__device__ __forceinline__ uint2 ld_stream_u2(const uint2* p) {
  uint2 r;
  asm volatile("ld.global.nc.L1::no_allocate.v2.u32 {%0,%1}, [%2];" : "=r"(r.x), "=r"(r.y) : "l"(p));
  return r;
}

// Decoupled look-back (single-pass prefix scan over tiles processed in ticket order).
// status[t] = (flag << 62) | value; flag 1 = tile aggregate, 2 = inclusive prefix.
// Called by ONE full warp; returns the exclusive prefix of `aggregate` over tiles < tile and
// publishes the inclusive prefix. Values must stay below 2^62.
constexpr uint64_t kLbMask = (1ull << 62) - 1;
__device__ inline uint64_t lookback_exclusive(uint64_t* status, uint32_t tile, uint64_t aggregate) {
  const int lane = threadIdx.x & 31;
  if (tile == 0) {
    if (lane == 0) st_release(status, (2ull << 62) | aggregate);
    return 0;
  }
  if (lane == 0) st_release(status + tile, (1ull << 62) | aggregate);
  uint64_t exclusive = 0;
  int64_t base = (int64_t)tile - 1;
  while (true) {
    const int64_t my = base - lane;
    uint64_t w;
    do {
      w = (my >= 0) ? ld_acquire(status + my) : (2ull << 62);
    } while (__any_sync(0xFFFFFFFFu, (w >> 62) == 0));
    const uint32_t incl = __ballot_sync(0xFFFFFFFFu, (w >> 62) == 2);
    uint64_t v = w & kLbMask;
    if (incl) {
      const int first = __ffs(incl) - 1;            // nearest predecessor holding a prefix
      if (lane > first) v = 0;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xFFFFFFFFu, v, o);
    exclusive += v;
    if (incl) break;
    base -= 32;
  }
  if (lane == 0) st_release(status + tile, (2ull << 62) | (exclusive + aggregate));
  return exclusive;
}

// Block-wide exclusive scan of a u64 (kThreads threads). `smem` holds >= kThreads/32 u64.
// Returns the exclusive prefix; *total receives the block total. Contains two __syncthreads.
__device__ inline uint64_t block_exclusive_scan(uint64_t x, uint64_t* smem, uint64_t* total) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint64_t incl = x;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    uint64_t y = __shfl_up_sync(0xFFFFFFFFu, incl, o);
    if (lane >= o) incl += y;
  }
  if (lane == 31) smem[warp] = incl;
  __syncthreads();
  uint64_t warp_off = 0, tot = 0;
#pragma unroll
  for (int w = 0; w < kThreads / 32; ++w) {
    uint64_t t = smem[w];
    if (w < warp) warp_off += t;
    tot += t;
  }
  __syncthreads();
  *total = tot;
  return warp_off + incl - x;
}

}  // namespace lowdiff
