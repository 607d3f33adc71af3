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

// ---- TMA 1-D bulk copies completing on an mbarrier (shared by the stream and replay kernels) --
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n"
      "LAB_WAIT:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra LAB_WAIT;\n}" :: "r"(bar), "r"(parity) : "memory");
}
__device__ __forceinline__ void bulk_g2s(uint32_t dst, const void* src, uint32_t bytes, uint32_t bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
               :: "r"(dst), "l"(src), "r"(bytes), "r"(bar) : "memory");
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

// The same for a block of NT threads (NT % 32 == 0, NT <= 1024); `smem` holds >= NT/32 u64.
template <int NT>
__device__ inline uint64_t block_exclusive_scan_n(uint64_t x, uint64_t* smem, uint64_t* total) {
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
  for (int w = 0; w < NT / 32; ++w) {
    uint64_t t = smem[w];
    if (w < warp) warp_off += t;
    tot += t;
  }
  __syncthreads();
  *total = tot;
  return warp_off + incl - x;
}

}  // namespace lowdiff
