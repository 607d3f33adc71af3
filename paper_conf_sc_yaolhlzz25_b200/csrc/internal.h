// Host-side internals of liblowdiff: error plumbing, launch accounting, profiling events and
// the launchers each .cu file exports to api.cu. Not part of the ABI.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "dense_step.h"
#include "lowdiff.h"

namespace lowdiff {

lowdiff_status fail(lowdiff_status s, const char* fmt, ...);
lowdiff_status cuda_status(cudaError_t e, const char* what);

// Every kernel launch goes through LD_LAUNCH so it is counted and (optionally) timed.
void note_launch();
struct ProfScope {
  ProfScope(const char* cls, cudaStream_t s);
  ~ProfScope();
  const char* cls;
  cudaStream_t stream;
  int slot;
};

#define LD_LAUNCH(cls, stream, kernel, grid, block, smem, ...)                      \
  do {                                                                             \
    ::lowdiff::ProfScope _ld_prof(cls, stream);                                    \
    kernel<<<(grid), (block), (smem), (stream)>>>(__VA_ARGS__);                    \
    ::lowdiff::note_launch();                                                      \
  } while (0)

#define LD_CUDA(expr, what)                                                         \
  do {                                                                             \
    cudaError_t _e = (expr);                                                       \
    if (_e != cudaSuccess) return ::lowdiff::cuda_status(_e, what);                \
  } while (0)

inline uint64_t align256(uint64_t x) { return (x + 255u) & ~(uint64_t)255u; }

// ---- compress (compress.cu) ---------------------------------------------------------------
uint64_t compress_ws_bytes(uint64_t n, uint64_t k);
void compress_force_threshold(int which /* 0 first pass, 1 rescan */, int enable, uint32_t key);
lowdiff_status compress_stats(const void* ws, uint64_t n, uint64_t k, uint64_t out[10], cudaStream_t s);
lowdiff_status compress_counters(const void* ws, cudaStream_t s, uint64_t out[9]);
lowdiff_status compress_run(const void* grad, int gdt, float* residual, uint64_t n, uint64_t k,
                            void* pairs, int vdt, void* ws, cudaStream_t s);

// ---- multiway index merge engine (merge.cu): coalesce after the all-gather, batch merge -------
constexpr int kMaxLists = 256;
struct ListDesc {
  const uint32_t* idx;
  const void* val;          // fp32, or bf16 when ListSet::bf16
  const uint64_t* d_len;    // device length (nullptr => use len)
  uint64_t len;
};
struct ListSet {
  int L;
  int bf16;
  ListDesc list[kMaxLists];
};
enum MergeKind { kCoalesce = 0, kMergeSum = 1, kMergeStack = 2 };
uint64_t merge_ws_bytes(int L, uint64_t max_entries, uint64_t lo, uint64_t hi);
// Coalesce: writes out_idx/out_val/d_out_nnz directly. Merge: assembles a record into d_record.
lowdiff_status merge_run(const ListSet& lists, MergeKind kind, uint64_t lo, uint64_t hi,
                         int average, uint64_t max_entries, uint32_t* out_idx, float* out_val,
                         uint64_t out_cap, uint64_t* d_out_nnz,
                         /* record (merge only) */ const float* lr, uint64_t n, uint64_t t_first,
                         uint32_t nranks, void* d_record, uint64_t record_cap,
                         uint64_t* d_record_bytes, void* ws, cudaStream_t s);

// ---- replay (replay.cu) ---------------------------------------------------------------------
struct RecInfo {            // parsed on the host from the record header
  const uint8_t* d;         // device record base
  uint32_t mode, B;
  uint64_t nnz, nent;
  uint64_t off_lr, off_idx, off_val, off_off, off_it;   // section byte offsets
  const float* h_lr;        // host lr[B]
  const void* h_head_bytes = nullptr;   // host copy of the 80-byte header (validated against the device)
  // live update (lowdiff_update): a bare (idx, val) list whose length lives on the device; then
  // d == nullptr, mode == SUM, B == 1 and nnz is the host upper bound (cap)
  const uint32_t* live_idx = nullptr;
  const float* live_val = nullptr;
  const uint64_t* d_nnz = nullptr;
};
uint64_t replay_ws_bytes(uint64_t len, const RecInfo* recs, uint32_t nrec);
lowdiff_status replay_run(lowdiff_state* st, const lowdiff_opt* o, const RecInfo* recs,
                          uint32_t nrec, void* ws, cudaStream_t s);
lowdiff_status replay_check(const void* ws, cudaStream_t s);
uint64_t replay_parallel_ws_bytes(uint32_t nrec, uint64_t entries, uint64_t lo, uint64_t hi);
lowdiff_status replay_parallel_run(lowdiff_state* st, const RecInfo* recs, uint32_t nrec, void* ws,
                                   cudaStream_t s);

// ---- LowDiff+ dense updates (plus.cu, host_update.cpp) ----------------------------------------
void dense_update_scalars(lowdiff_state* st, const lowdiff_opt* o, float lr, DenseStep* d);
lowdiff_status dense_update_run(lowdiff_state* st, const lowdiff_opt* o, const void* grad, int gdt, float lr,
                                cudaStream_t s);

}  // namespace lowdiff
