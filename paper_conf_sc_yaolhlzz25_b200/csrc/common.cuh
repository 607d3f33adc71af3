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

// ---- streaming loads ---------------------------------------------------------------------
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
