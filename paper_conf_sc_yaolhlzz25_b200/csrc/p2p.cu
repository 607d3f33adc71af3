// lowdiff_p2p_* — Sync(G~_{i,t}) (Alg.1 line 5; "Allgather") fused with the
// coalesce over peer memory: every rank's packed pairs stay in an exchange window in its owner's
// HBM, mapped into every rank through CUDA IPC, and the coalesce (merge.cu, the same multiway
// merge lowdiff_coalesce runs) reads them there over NVLink / NVSwitch. Compared with
// ncclAllGather + coalesce this skips the (P-1) * pairs_bytes receive write and its re-read, and
// a rank pulls only what its coalesce touches.
//
// Synchronisation is a pair of epoch flags per rank in every window (include/lowdiff.h (2')):
// ready[r] = e+1 once rank r's slot e&1 holds its epoch-e pairs, done[r] = e+1 once rank r has
// finished reading every slot of epoch e. Writers release-store at system scope after a system
// fence; waiters acquire-load their own window. Each wait is one tiny kernel (one CTA, one thread
// per peer) with a bounded spin, so a missing peer ends in ETIMEOUT, never in a hung GPU.
#include <string.h>

#include <cstdlib>

#include "common.cuh"
#include "internal.h"

namespace lowdiff {
namespace {

constexpr int kMaxP2P = 64;

struct FlagPtrs {
  uint64_t* p[kMaxP2P];
};

__device__ __forceinline__ uint64_t ld_acquire_sys(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_sys(uint64_t* p, uint64_t v) {
  asm volatile("st.release.sys.global.u64 [%0], %1;" :: "l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t globaltimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}

// The epoch counter lives in this rank's window (device memory), so a captured CUDA graph replays
// with fresh flag values: every kernel reads e from it, the done-signal advances it.
enum WaitKind { kWaitDone = 0, kWaitReady = 1 };

// kWaitDone : until done[p] >= e-1 for every p != rank (skipped while e < 2)
// kWaitReady: until ready[p] >= e+1 for every p != rank; also checks that the slot the host picked
//             (parity) is the device epoch's, else flags error 2
__global__ void p2p_wait_kernel(const uint64_t* flags, const uint64_t* epoch, int P, int rank, int kind,
                                uint32_t parity, uint64_t timeout_ns, volatile uint32_t* err) {
  const int p = threadIdx.x;
  const uint64_t e = *reinterpret_cast<const volatile uint64_t*>(epoch);
  if (kind == kWaitReady && p == 0 && (uint32_t)(e & 1) != parity) *err = 2u;
  if (p >= P || p == rank) return;
  if (kind == kWaitDone && e < 2) return;
  const uint64_t target = kind == kWaitDone ? e - 1 : e + 1;
  const uint64_t* f = flags + (kind == kWaitDone ? P : 0) + p;
  const uint64_t t0 = globaltimer();
  while (ld_acquire_sys(f) < target) {
    if (globaltimer() - t0 > timeout_ns) {
      *err = 1u;
      __threadfence_system();
      return;
    }
    __nanosleep(200);
  }
}

// Release-store e+1 into one flag of every window (the copy or merge that precedes this kernel on
// the stream has completed: stream order, then a system-scope fence). `advance`: then e += 1.
__global__ void p2p_signal_kernel(const __grid_constant__ FlagPtrs f, uint64_t* epoch, int P, int advance) {
  const int p = threadIdx.x;
  const uint64_t e = *reinterpret_cast<volatile uint64_t*>(epoch);
  if (p < P) {
    __threadfence_system();
    st_release_sys(f.p[p], e + 1);
  }
  if (advance) {
    __syncthreads();
    if (p == 0) *reinterpret_cast<volatile uint64_t*>(epoch) = e + 1;
  }
}

// pairs -> local slot (16-byte vectors; both 16-byte aligned, pairs_bytes a multiple of 16). A
// kernel rather than cudaMemcpyAsync: a device-to-device memcpy may synchronise implicitly with
// other streams of the device, which would serialise it behind a peer's spinning wait kernel when
// several ranks share one device (the single-process mode).
__global__ void __launch_bounds__(kThreads) p2p_copy_kernel(const uint4* __restrict__ src, uint4* __restrict__ dst,
                                                            uint64_t n16) {
  for (uint64_t i = (uint64_t)blockIdx.x * kThreads + threadIdx.x; i < n16; i += (uint64_t)gridDim.x * kThreads)
    dst[i] = src[i];
}

typedef int (*MemGetAddressRange)(unsigned long long*, size_t*, unsigned long long);

lowdiff_status allocation_base(const void* ptr, uint8_t** base) {
  static MemGetAddressRange fn = nullptr;
  if (!fn) {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    cudaError_t e = cudaGetDriverEntryPoint("cuMemGetAddressRange", &f, cudaEnableDefault, &q);
    if (e != cudaSuccess || q != cudaDriverEntryPointSuccess || !f)
      return fail(LOWDIFF_ECUDA, "p2p: cuMemGetAddressRange entry point unavailable");
    fn = reinterpret_cast<MemGetAddressRange>(f);
  }
  unsigned long long b = 0;
  size_t sz = 0;
  if (fn(&b, &sz, reinterpret_cast<unsigned long long>(ptr)) != 0)
    return fail(LOWDIFF_ECUDA, "p2p: cuMemGetAddressRange failed (not device memory?)");
  *base = reinterpret_cast<uint8_t*>(b);
  return LOWDIFF_OK;
}

// window: u64 ready[P] | u64 done[P] | u64 epoch | pad to 256 | slot 0 | slot 1
uint64_t flags_bytes(int P) { return align256(16ull * P + 8); }
uint64_t slot_bytes(uint64_t k, lowdiff_dtype vdt) {
  return align256(pad16(4 * k) + pad16((vdt == LOWDIFF_BF16 ? 2ull : 4ull) * k));
}

}  // namespace
}  // namespace lowdiff

using namespace lowdiff;

struct lowdiff_p2p {
  int P, rank;
  uint64_t k;
  lowdiff_dtype vdt;
  uint64_t pb, slot_off[2];
  uint8_t* win[kMaxP2P];        // every rank's window, mapped here (own included)
  uint8_t* ipc_base[kMaxP2P];   // IPC-opened allocation bases (closed by destroy), or nullptr
  uint64_t epoch;
  uint64_t timeout_ns;
  uint32_t* h_err;              // mapped pinned word: 1 once a wait expired
  uint32_t* d_err;
  bool slot_acquired;           // lowdiff_p2p_slot enqueued the done-wait of the next epoch
};

namespace {

lowdiff_status p2p_common_init(lowdiff_p2p** out, void* window, int32_t nranks, int32_t rank, uint64_t k,
                               lowdiff_dtype vdt) {
  if (!out || !window || nranks < 2 || nranks > kMaxP2P || rank < 0 || rank >= nranks || k == 0 ||
      (uint64_t)nranks * k >= (1ull << 31) || (vdt != LOWDIFF_F32 && vdt != LOWDIFF_BF16) ||
      (reinterpret_cast<uintptr_t>(window) & 255u))
    return fail(LOWDIFF_EINVAL, "p2p_init: need 2 <= nranks <= %d, 0 <= rank < nranks, k >= 1, P*k < 2^31, "
                "a 256-byte aligned window", kMaxP2P);
  lowdiff_p2p* c = new lowdiff_p2p();
  c->P = nranks;
  c->rank = rank;
  c->k = k;
  c->vdt = vdt;
  c->pb = lowdiff_pairs_bytes(k, vdt);
  c->slot_off[0] = flags_bytes(nranks);
  c->slot_off[1] = flags_bytes(nranks) + slot_bytes(k, vdt);
  c->epoch = 0;
  c->slot_acquired = false;
  const char* to = getenv("LOWDIFF_P2P_TIMEOUT_MS");
  c->timeout_ns = (to && atoll(to) > 0 ? (uint64_t)atoll(to) : 20000ull) * 1000000ull;
  cudaError_t e = cudaHostAlloc(reinterpret_cast<void**>(&c->h_err), 4, cudaHostAllocMapped);
  if (e == cudaSuccess) e = cudaHostGetDevicePointer(reinterpret_cast<void**>(&c->d_err), c->h_err, 0);
  if (e != cudaSuccess) {
    delete c;
    return cuda_status(e, "p2p_init: mapped error word");
  }
  *c->h_err = 0;
  // zero this rank's flags (peers must not signal before every rank's init returned: the
  // caller's barrier after init guarantees it)
  e = cudaMemset(window, 0, flags_bytes(nranks));
  if (e == cudaSuccess) e = cudaDeviceSynchronize();
  if (e != cudaSuccess) {
    cudaFreeHost(c->h_err);
    delete c;
    return cuda_status(e, "p2p_init: zero flags");
  }
  *out = c;
  return LOWDIFF_OK;
}

}  // namespace

extern "C" {

uint64_t lowdiff_p2p_window_bytes(int32_t nranks, uint64_t k, lowdiff_dtype vdt) {
  if (nranks < 1 || nranks > kMaxP2P || k == 0) return 0;
  return flags_bytes(nranks) + 2 * slot_bytes(k, vdt);
}

lowdiff_status lowdiff_p2p_export_handle(const void* window, uint8_t* handle) {
  if (!window || !handle) return fail(LOWDIFF_EINVAL, "p2p_export_handle: null");
  uint8_t* base = nullptr;
  lowdiff_status s = allocation_base(window, &base);
  if (s) return s;
  cudaIpcMemHandle_t h;
  LD_CUDA(cudaIpcGetMemHandle(&h, base), "cudaIpcGetMemHandle");
  static_assert(sizeof(h) == 64, "IPC handle size");
  const uint64_t off = (uint64_t)(static_cast<const uint8_t*>(window) - base);
  memset(handle, 0, LOWDIFF_P2P_HANDLE_BYTES);
  memcpy(handle, &h, 64);
  memcpy(handle + 64, &off, 8);
  return LOWDIFF_OK;
}

lowdiff_status lowdiff_p2p_init(lowdiff_p2p** out, void* window, const uint8_t* handles, int32_t nranks,
                                int32_t rank, uint64_t k, lowdiff_dtype vdt) {
  if (!handles) return fail(LOWDIFF_EINVAL, "p2p_init: null handles");
  lowdiff_p2p* c = nullptr;
  lowdiff_status s = p2p_common_init(&c, window, nranks, rank, k, vdt);
  if (s) return s;
  for (int p = 0; p < nranks; ++p) {
    c->ipc_base[p] = nullptr;
    if (p == rank) {
      c->win[p] = static_cast<uint8_t*>(window);
      continue;
    }
    cudaIpcMemHandle_t h;
    uint64_t off;
    memcpy(&h, handles + (uint64_t)p * LOWDIFF_P2P_HANDLE_BYTES, 64);
    memcpy(&off, handles + (uint64_t)p * LOWDIFF_P2P_HANDLE_BYTES + 64, 8);
    void* base = nullptr;
    cudaError_t e = cudaIpcOpenMemHandle(&base, h, cudaIpcMemLazyEnablePeerAccess);
    if (e != cudaSuccess) {
      for (int q = 0; q < p; ++q)
        if (c->ipc_base[q]) cudaIpcCloseMemHandle(c->ipc_base[q]);
      cudaFreeHost(c->h_err);
      delete c;
      return cuda_status(e, "p2p_init: cudaIpcOpenMemHandle");
    }
    c->ipc_base[p] = static_cast<uint8_t*>(base);
    c->win[p] = static_cast<uint8_t*>(base) + off;
  }
  *out = c;
  return LOWDIFF_OK;
}

lowdiff_status lowdiff_p2p_init_local(lowdiff_p2p** out, void* const* windows, int32_t nranks, int32_t rank,
                                      uint64_t k, lowdiff_dtype vdt) {
  if (!windows || nranks < 2 || rank < 0 || rank >= nranks) return fail(LOWDIFF_EINVAL, "p2p_init_local");
  for (int p = 0; p < nranks; ++p)
    if (!windows[p] || (reinterpret_cast<uintptr_t>(windows[p]) & 255u))
      return fail(LOWDIFF_EINVAL, "p2p_init_local: window %d null or not 256-byte aligned", p);
  lowdiff_p2p* c = nullptr;
  lowdiff_status s = p2p_common_init(&c, windows[rank], nranks, rank, k, vdt);
  if (s) return s;
  for (int p = 0; p < nranks; ++p) {
    c->win[p] = static_cast<uint8_t*>(windows[p]);
    c->ipc_base[p] = nullptr;
  }
  *out = c;
  return LOWDIFF_OK;
}

lowdiff_status lowdiff_p2p_destroy(lowdiff_p2p* c) {
  if (!c) return LOWDIFF_OK;
  cudaError_t first = cudaSuccess;
  for (int p = 0; p < c->P; ++p)
    if (c->ipc_base[p]) {
      cudaError_t e = cudaIpcCloseMemHandle(c->ipc_base[p]);
      if (first == cudaSuccess) first = e;
    }
  cudaFreeHost(c->h_err);
  delete c;
  return first == cudaSuccess ? LOWDIFF_OK : cuda_status(first, "p2p_destroy: cudaIpcCloseMemHandle");
}

lowdiff_status lowdiff_p2p_status(const lowdiff_p2p* c) {
  if (!c) return fail(LOWDIFF_EINVAL, "p2p_status: null");
  const uint32_t err = *reinterpret_cast<volatile uint32_t*>(c->h_err);
  if (err == 2u)
    return fail(LOWDIFF_EINVAL, "p2p: slot parity differs from the device epoch (a captured graph replays an odd "
                "number of calls, or calls were skipped)");
  if (err)
    return fail(LOWDIFF_ETIMEOUT, "p2p: a peer wait expired after %llu ms (a rank did not make the matching call)",
                (unsigned long long)(c->timeout_ns / 1000000ull));
  return LOWDIFF_OK;
}

static uint64_t* epoch_ptr(const lowdiff_p2p* c) {
  return reinterpret_cast<uint64_t*>(c->win[c->rank]) + 2 * c->P;
}

static lowdiff_status p2p_wait(lowdiff_p2p* c, int kind, cudaStream_t s) {
  LD_LAUNCH("p2p_wait", s, p2p_wait_kernel, 1, 32 * ((c->P + 31) / 32), 0,
            reinterpret_cast<const uint64_t*>(c->win[c->rank]), epoch_ptr(c), c->P, c->rank, kind,
            (uint32_t)(c->epoch & 1), c->timeout_ns, c->d_err);
  return cuda_status(cudaGetLastError(), "p2p wait launch");
}

static lowdiff_status p2p_wait_done(lowdiff_p2p* c, cudaStream_t s) { return p2p_wait(c, kWaitDone, s); }

void* lowdiff_p2p_slot(lowdiff_p2p* c, lowdiff_stream_t stream) {
  if (!c) return nullptr;
  if (!c->slot_acquired) {
    if (p2p_wait_done(c, (cudaStream_t)stream)) return nullptr;
    c->slot_acquired = true;
  }
  return c->win[c->rank] + c->slot_off[c->epoch & 1];
}

lowdiff_status lowdiff_p2p_allgather_sparse(lowdiff_p2p* c, const void* pairs, uint64_t lo, uint64_t hi,
                                            int32_t average, uint32_t* out_idx, float* out_val, uint64_t out_cap,
                                            uint64_t* d_out_nnz, void* ws, uint64_t ws_bytes,
                                            lowdiff_stream_t stream) {
  if (!c) return fail(LOWDIFF_EINVAL, "p2p_allgather_sparse: null handle");
  const int P = c->P;
  uint64_t wsz = 0;
  lowdiff_status st = lowdiff_coalesce_workspace_size(P, c->k, c->vdt, lo, hi, &wsz);
  if (st) return st;
  if (!pairs || !out_idx || !out_val || !d_out_nnz || !ws || (reinterpret_cast<uintptr_t>(pairs) & 15u) ||
      (reinterpret_cast<uintptr_t>(out_idx) & 15u) || (reinterpret_cast<uintptr_t>(out_val) & 15u) ||
      (reinterpret_cast<uintptr_t>(ws) & 15u))
    return fail(LOWDIFF_EINVAL, "p2p_allgather_sparse: null or misaligned pointer");
  const uint64_t need = (uint64_t)P * c->k < hi - lo ? (uint64_t)P * c->k : hi - lo;
  if (out_cap < need)
    return fail(LOWDIFF_EINVAL, "p2p_allgather_sparse: out_cap %llu < min(P*k, hi-lo) = %llu",
                (unsigned long long)out_cap, (unsigned long long)need);
  if (ws_bytes < wsz) return fail(LOWDIFF_EWORKSPACE, "p2p_allgather_sparse: workspace too small");
  cudaStream_t s = (cudaStream_t)stream;
  const uint64_t e = c->epoch;
  const int slot = (int)(e & 1);
  uint8_t* mine = c->win[c->rank] + c->slot_off[slot];
  // 1-2: the local slot becomes writable, then holds this epoch's pairs
  if (pairs != mine) {
    if (!c->slot_acquired) {
      st = p2p_wait_done(c, s);
      if (st) return st;
    }
    const uint64_t n16 = c->pb / 16;
    uint64_t g = (n16 + kThreads - 1) / kThreads;
    if (g > 2ull * kNumSMs) g = 2ull * kNumSMs;
    LD_LAUNCH("p2p_copy", s, p2p_copy_kernel, (int)g, kThreads, 0, static_cast<const uint4*>(pairs),
              reinterpret_cast<uint4*>(mine), n16);
  } else if (!c->slot_acquired) {
    return fail(LOWDIFF_EINVAL, "p2p_allgather_sparse: pairs is the slot but lowdiff_p2p_slot was not called");
  }
  c->slot_acquired = false;
  // 3: publish ready[rank] = e+1 in every window
  FlagPtrs f;
  for (int p = 0; p < P; ++p) f.p[p] = reinterpret_cast<uint64_t*>(c->win[p]) + c->rank;
  LD_LAUNCH("p2p_signal", s, p2p_signal_kernel, 1, 32 * ((P + 31) / 32), 0, f, epoch_ptr(c), P, 0);
  // 4: every peer's slot holds epoch e
  st = p2p_wait(c, kWaitReady, s);
  if (st) return st;
  // 5: coalesce straight out of the owners' windows
  ListSet* ls = new ListSet();
  ls->L = P;
  ls->bf16 = c->vdt == LOWDIFF_BF16;
  for (int p = 0; p < P; ++p) {
    const uint8_t* b = c->win[p] + c->slot_off[slot];
    ls->list[p].idx = reinterpret_cast<const uint32_t*>(b);
    ls->list[p].val = b + pad16(4 * c->k);
    ls->list[p].d_len = nullptr;
    ls->list[p].len = c->k;
  }
  st = merge_run(*ls, kCoalesce, lo, hi, average, (uint64_t)P * c->k, out_idx, out_val, out_cap, d_out_nnz,
                 nullptr, 0, 0, 0, nullptr, 0, nullptr, ws, s);
  delete ls;
  if (st) return st;
  // 6: done reading epoch e: done[rank] = e+1 in every window
  for (int p = 0; p < P; ++p) f.p[p] = reinterpret_cast<uint64_t*>(c->win[p]) + P + c->rank;
  LD_LAUNCH("p2p_signal", s, p2p_signal_kernel, 1, 32 * ((P + 31) / 32), 0, f, epoch_ptr(c), P, 1);
  c->epoch = e + 1;
  return cuda_status(cudaGetLastError(), "p2p_allgather_sparse launch");
}

}  // extern "C"
