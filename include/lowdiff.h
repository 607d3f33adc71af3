/*
 * lowdiff.h — C ABI of the B200-native LowDiff hot path (liblowdiff.so).
 *
 * LowDiff (Yao et al., SC'25; /root/reference/PAPER.md, cited P:line) reuses each training
 * iteration's compressed, synchronized gradient G~_t as the differential checkpoint C^D_t
 * (Finding 1), batches B of them into one write (§4.2) and replays the chain
 * onto a full checkpoint on recovery (Alg.1 lines 16-24). The five calls below are
 * the data-parallel hot path BASELINE.json north_star names:
 *
 *   lowdiff_compress          Comp(G_{i,t})        Alg.1 line 4
 *   lowdiff_allgather_sparse  Sync(G~_{i,t})       Alg.1 line 5
 *   lowdiff_batch_merge       batched C^B_t        §4.2 Step 2
 *   lowdiff_stage_d2h         offload to CPU       §4.2 Step 1
 *   lowdiff_replay            Recovery             Alg.1 lines 16-24, Eq.1
 *
 * Conventions (all calls):
 *  - Pointers are DEVICE pointers unless the argument says "host". The caller owns every buffer
 *    (device memory, pinned host memory, workspaces); the library allocates nothing on the
 *    hot-path calls. Workspace sizes come from the *_workspace_size queries.
 *  - Every call is asynchronous on the given stream (a cudaStream_t; NULL = legacy default
 *    stream). Host-side argument validation is synchronous. Data-dependent counts (nnz, record
 *    bytes) are written to caller DEVICE memory; only lowdiff_record_bytes synchronizes.
 *  - Every call returns a lowdiff_status; nothing is thrown across the ABI. On failure,
 *    lowdiff_last_error() returns a thread-local description.
 *  - Device pointers to bulk arrays must be 16-byte aligned (EINVAL otherwise).
 *  - Index width is u32; n must be < 2^31 (EINVAL otherwise; every BASELINE config fits:
 *    GPT-2 XL has n = 1,557,611,200).
 *  - Floating point: IEEE binary32, round-to-nearest-even per operation, no FMA contraction,
 *    no flush-to-zero, fixed fold orders (rank-ascending, iteration-ascending), no float atomics:
 *    results are deterministic and equal the CPU oracle's bit for bit.
 */
#ifndef LOWDIFF_H
#define LOWDIFF_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct CUstream_st* lowdiff_stream_t; /* == cudaStream_t */

typedef int32_t lowdiff_status;
enum {
  LOWDIFF_OK = 0,
  LOWDIFF_EINVAL = 1,        /* bad argument (null/misaligned pointer, size, dtype, range)    */
  LOWDIFF_EWORKSPACE = 2,    /* workspace smaller than the *_workspace_size query returned   */
  LOWDIFF_ECAPACITY = 3,     /* an output (record, coalesced list) exceeds its capacity       */
  LOWDIFF_ECHAIN = 4,        /* replay records not contiguous in t, or shard/n/nranks differ */
  LOWDIFF_ECORRUPT = 5,      /* record bytes fail validation                                  */
  LOWDIFF_EUNSUPPORTED = 6,  /* e.g. SUM record with momentum/Adam without opt-in             */
  LOWDIFF_ECUDA = 7,         /* CUDA runtime error (message in lowdiff_last_error)            */
  LOWDIFF_ENCCL = 8,         /* NCCL error                                                    */
  LOWDIFF_ETIMEOUT = 9       /* a peer-memory wait expired (lowdiff_p2p_*)                    */
};

typedef enum { LOWDIFF_F32 = 0, LOWDIFF_BF16 = 1 } lowdiff_dtype;
typedef enum { LOWDIFF_MERGE_SUM = 0, LOWDIFF_MERGE_STACK = 1 } lowdiff_merge_mode;
typedef enum { LOWDIFF_OPT_SGD = 0, LOWDIFF_OPT_MOMENTUM = 1, LOWDIFF_OPT_ADAM = 2 } lowdiff_opt_kind;

const char* lowdiff_status_string(lowdiff_status s);
const char* lowdiff_last_error(void);      /* thread-local detail of the last failure       */
const char* lowdiff_version(void);

/* k = max(1, min(n, floor(rho * n))) evaluated in double — the number of pairs one rank emits
 * at compression ratio rho (reading #2). */
uint64_t lowdiff_k_for_density(uint64_t n, double rho);

/* Bytes of one rank's packed pairs: pad16(4k) + pad16(sizeof(vdt) * k). */
uint64_t lowdiff_pairs_bytes(uint64_t k, lowdiff_dtype vdt);

/* Contiguous parameter-index shard owned by `rank` of `nranks`:
 * [floor(rank n / nranks), floor((rank+1) n / nranks))   (reading #22). */
lowdiff_status lowdiff_shard_bounds(uint64_t n, int32_t nranks, int32_t rank, uint64_t* lo, uint64_t* hi);

/* ---------------------------------------------------------------------------------------------
 * (0) Plan — the paper's problem statement: a flat gradient of n elements compressed at ratio rho
 *     (P:130), differentials batched B per write (batching size b) and a
 *     full checkpoint every full_every iterations (f = 1/FCF), on rank `rank` of
 *     `nranks` data-parallel ranks.
 *   lowdiff_plan_init fills k = lowdiff_k_for_density(n, rho) and the rank's shard [lo, hi)
 *     (lowdiff_shard_bounds). Errors: EINVAL (n = 0 or n >= 2^31, rho not in (0, 1], B = 0 or
 *     B > 255, nranks < 1, rank out of range, unknown dtype).
 *   lowdiff_plan_record_due(t): the record-boundary policy for iteration t (0-based; DESIGN.md
 *     reading #25). A full checkpoint C^F_t (M_t, before G~_t is applied) is due before iteration
 *     t when t % full_every == 0 (full_every = 0: only at t = 0). A record never spans a full
 *     checkpoint: the open record closes after iteration t when it holds B iterations, or when the
 *     next iteration starts with a full checkpoint — then it is a SHORT record (B' < B iterations;
 *     legal, the header carries B'). Outputs (host, any may be NULL): *full_checkpoint_due,
 *     *close_record, *batch_len = iterations in the open record including t (= B' when it closes).
 *     What a failure loses: iterations after the last closed and persisted record.
 * ------------------------------------------------------------------------------------------- */
typedef struct {
  uint64_t n;
  double rho;
  uint64_t k;
  uint32_t B;
  uint32_t full_every;      /* FCF in iterations; 0 = only the initial full checkpoint */
  int32_t gdt, vdt;         /* lowdiff_dtype of the gradient and of the emitted values */
  int32_t nranks, rank;
  uint64_t lo, hi;
} lowdiff_plan;
lowdiff_status lowdiff_plan_init(lowdiff_plan* plan, uint64_t n, double rho, uint32_t B, uint32_t full_every,
                                 lowdiff_dtype gdt, lowdiff_dtype vdt, int32_t nranks, int32_t rank);
lowdiff_status lowdiff_plan_record_due(const lowdiff_plan* plan, uint64_t t, int32_t* close_record,
                                       uint32_t* batch_len, int32_t* full_checkpoint_due);

/* ---------------------------------------------------------------------------------------------
 * (1) Compress — Comp(G_{i,t}), Alg.1 line 4; "sparsification" at ratio rho.
 *     Exact top-k with error feedback (north_star; readings #1-#8):
 *       a = fp32(grad) + residual                         (one fp32 add; bf16 widening exact)
 *       S = the k largest a by |a| (u32 key = bits(a) & 0x7FFFFFFF; equal keys: lower index first)
 *       pairs = [ idx u32 x k ascending | zero pad to 16 B | val x k | zero pad to 16 B ]
 *         vdt F32 : val = a[S];             residual <- a off S, +0 on S
 *         vdt BF16: val = bf16_rne(a[S]);   residual <- a off S, a - fp32(val) on S (exact)
 *   grad      [n] gdt (F32 or BF16), read only.      residual [n] fp32, updated in place.
 *   pairs     lowdiff_pairs_bytes(k, vdt) bytes, written.   1 <= k <= n < 2^31.
 *   ws        lowdiff_compress_workspace_size(n, k) bytes, device, 16-byte aligned. Its first 256
 *             bytes carry a per-residual threshold STATE between calls (the previous call's exact
 *             k-th key, an adaptive margin, counters): pass the same ws for the same residual to
 *             keep it warm. The state is a hint only — a fresh, foreign or garbage workspace reads as
 *             "cold" (checked against n, k, the residual pointer and the dtypes) and the OUTPUT IS
 *             IDENTICAL either way; the rest of ws is scratch.
 * Execution: one streaming pass keeps every element whose key is >= T (T = the previous k-th key
 *   lowered by the margin) as a candidate; one cooperative select finds the exact k-th key among
 *   them and writes the pairs. If the candidates number < k (cold start, or the k-th key dropped
 *   by more than the margin) or exceed the capacity (8k + 65536), the select recovers on device
 *   with ONE rescan of the residual at a corrected threshold (from a stratified sample, resp. the
 *   exact first-digit histogram of the candidates); only if that also misses does an exact
 *   full-array select run. Paths and non-finite inputs are counted in the state:
 *   lowdiff_compress_counters.
 * Errors: EINVAL (k, n, dtype, alignment), EWORKSPACE. Non-finite a (Inf/NaN) are ordered by bit
 *   pattern above every finite key (reading #4) and counted, not rejected.
 * ------------------------------------------------------------------------------------------- */
lowdiff_status lowdiff_compress_workspace_size(uint64_t n, uint64_t k, uint64_t* bytes);
lowdiff_status lowdiff_compress(const void* grad, lowdiff_dtype gdt, float* residual, uint64_t n,
                                uint64_t k, void* pairs, lowdiff_dtype vdt, void* ws,
                                uint64_t ws_bytes, lowdiff_stream_t stream);

/* ---------------------------------------------------------------------------------------------
 * (2) Sparse all-gather + coalesce — Sync(G~_{i,t}), Alg.1 line 5; "Allgather".
 *     Every rank passes its k pairs (same k and vdt on all ranks); ncclAllGather moves the fixed-
 *     size packed buffers over NVLink; then the union of gathered indices within [lo, hi) is
 *     coalesced: val = (rank-ascending fp32 fold) / P if `average`, else the fold. Zero sums are
 *     kept (the index set is the union). Output: idx u32 ascending unique, val fp32, and the
 *     count in *d_out_nnz (device u64). out_cap must be >= min(P*k, hi-lo) (else EINVAL).
 *   comm == NULL means P = 1 (no collective; coalesce of the local list only).
 * lowdiff_coalesce is the same coalesce over P packed buffers already resident on this device
 * (laid out back to back, each lowdiff_pairs_bytes(k, vdt) long) — the post-gather half.
 * ------------------------------------------------------------------------------------------- */
typedef struct lowdiff_comm lowdiff_comm;
int32_t        lowdiff_comm_unique_id_bytes(void);                 /* 128 */
lowdiff_status lowdiff_comm_get_unique_id(uint8_t* id /* host, 128 bytes */);
lowdiff_status lowdiff_comm_init(lowdiff_comm** comm, const uint8_t* id /* host */, int32_t nranks,
                                 int32_t rank);  /* binds the calling thread's current device */
lowdiff_status lowdiff_comm_destroy(lowdiff_comm* comm);

lowdiff_status lowdiff_coalesce_workspace_size(int32_t nranks, uint64_t k, lowdiff_dtype vdt,
                                               uint64_t lo, uint64_t hi, uint64_t* bytes);
lowdiff_status lowdiff_coalesce(const void* gathered, int32_t nranks, uint64_t k, lowdiff_dtype vdt,
                                uint64_t lo, uint64_t hi, int32_t average, uint32_t* out_idx,
                                float* out_val, uint64_t out_cap, uint64_t* d_out_nnz, void* ws,
                                uint64_t ws_bytes, lowdiff_stream_t stream);
lowdiff_status lowdiff_allgather_sparse_workspace_size(int32_t nranks, uint64_t k, lowdiff_dtype vdt,
                                                       uint64_t lo, uint64_t hi, uint64_t* bytes);
lowdiff_status lowdiff_allgather_sparse(lowdiff_comm* comm, const void* pairs, uint64_t k,
                                        lowdiff_dtype vdt, uint64_t lo, uint64_t hi, int32_t average,
                                        uint32_t* out_idx, float* out_val, uint64_t out_cap,
                                        uint64_t* d_out_nnz, void* ws, uint64_t ws_bytes,
                                        lowdiff_stream_t stream);

/* ---------------------------------------------------------------------------------------------
 * (2') The same Sync (Alg.1 line 5; "Allgather") fused with the coalesce over peer
 *     memory (NVLink / NVSwitch P2P, CUDA IPC): no all-gather copy. Every rank owns an exchange
 *     WINDOW of lowdiff_p2p_window_bytes(nranks, k, vdt) bytes in its own HBM:
 *       [u64 ready[nranks] | u64 done[nranks] | u64 epoch | pad to 256 | slot 0 | slot 1]
 *     (each slot one packed pairs buffer, 256-byte aligned). The windows of all ranks are mapped
 *     into every rank. lowdiff_p2p_allgather_sparse, called by every rank in the same order
 *     (epoch e = 0, 1, ... counted on the device, so the calls may be captured in a CUDA graph
 *     as long as each replay makes an even number of them: the slot is picked on the host by the
 *     call's parity, checked against the device epoch), enqueues on `stream`:
 *       1. wait until every peer finished reading this rank's slot e&1 of epoch e-2 (done >= e-1)
 *       2. copy `pairs` into the local slot e&1. Zero-copy variant: lowdiff_p2p_slot(c, stream)
 *          enqueues wait 1 on `stream` and returns the slot; compress into it on that stream and
 *          pass it as `pairs` — steps 1-2 are then skipped
 *       3. release-store ready[rank] = e+1 into every window (after a system-scope fence)
 *       4. wait until every ready[p] >= e+1 in the local window (acquire)
 *       5. coalesce over [lo, hi) reading each rank's slot e&1 directly from its owner's HBM —
 *          the multiway merge of lowdiff_coalesce, bit-identical output (rank-ascending fold)
 *       6. release-store done[rank] = e+1 into every peer window
 *     Waits spin on device with a bounded time (LOWDIFF_P2P_TIMEOUT_MS, default 20000); a
 *     timeout sets a flag read by lowdiff_p2p_status (ETIMEOUT) instead of hanging the GPU, and
 *     the outputs of that call are then undefined.
 *   window     caller-owned device memory (cudaMalloc / torch), 256-byte aligned; zeroed by
 *              lowdiff_p2p_init (synchronously). Keep it alive until lowdiff_p2p_destroy.
 *   handle     LOWDIFF_P2P_HANDLE_BYTES bytes: CUDA IPC handle of the window's allocation plus
 *              the window's offset in it. Exchange them (e.g. torch.distributed all_gather),
 *              then every rank calls lowdiff_p2p_init with all of them in rank order (its own
 *              entry is not opened), then all ranks barrier before the first allgather call.
 *   lowdiff_p2p_init_local: every window lives in this process (`windows` holds the nranks
 *              device pointers), e.g. one process driving one device per rank. Several ranks on
 *              ONE device in one process are not supported: their streams may share a hardware
 *              queue, so a rank's spinning wait can block a peer's work until it times out.
 * Errors: EINVAL (sizes, alignment, P < 2; from lowdiff_p2p_status: slot parity mismatch), ECUDA
 * (IPC open failed: peers on devices without P2P access), ETIMEOUT (a wait expired: a rank did
 * not make the matching call).
 * ------------------------------------------------------------------------------------------- */
#define LOWDIFF_P2P_HANDLE_BYTES 80
typedef struct lowdiff_p2p lowdiff_p2p;
uint64_t       lowdiff_p2p_window_bytes(int32_t nranks, uint64_t k, lowdiff_dtype vdt);
lowdiff_status lowdiff_p2p_export_handle(const void* window, uint8_t* handle /* host, 80 B */);
lowdiff_status lowdiff_p2p_init(lowdiff_p2p** c, void* window, const uint8_t* handles /* host, nranks x 80 B */,
                                int32_t nranks, int32_t rank, uint64_t k, lowdiff_dtype vdt);
lowdiff_status lowdiff_p2p_init_local(lowdiff_p2p** c, void* const* windows /* host array */,
                                      int32_t nranks, int32_t rank, uint64_t k, lowdiff_dtype vdt);
lowdiff_status lowdiff_p2p_destroy(lowdiff_p2p* c);
void*          lowdiff_p2p_slot(lowdiff_p2p* c, lowdiff_stream_t stream); /* next call's slot; NULL on error */
lowdiff_status lowdiff_p2p_allgather_sparse(lowdiff_p2p* c, const void* pairs, uint64_t lo, uint64_t hi,
                                            int32_t average, uint32_t* out_idx, float* out_val,
                                            uint64_t out_cap, uint64_t* d_out_nnz, void* ws,
                                            uint64_t ws_bytes /* >= lowdiff_coalesce_workspace_size */,
                                            lowdiff_stream_t stream);
lowdiff_status lowdiff_p2p_status(const lowdiff_p2p* c);  /* ETIMEOUT once any wait expired; no sync */

/* ---------------------------------------------------------------------------------------------
 * (3) Batch merge — Step 2 of batched gradient writing: B consecutive differentials of
 *     one shard become one record C^B ("tensor addition or dictionary accumulation"):
 *       SUM   (tensor addition):       U = union; val = iteration-ascending fp32 fold
 *       STACK (dictionary accumulation): per u in U the (iteration, value) list, iteration order
 *     The record layout (little-endian, every section 16-byte aligned, zero padding):
 *       header (lowdiff_record_header, 80 B) | f32 lr[B] | u32 idx[nnz] |
 *       SUM: f32 val[nnz]      STACK: u32 off[nnz+1] | u8 it[nent] | f32 val[nent]
 *   diffs     HOST array of B views; idx/val/d_nnz are device pointers, `cap` bounds nnz (host).
 *   d_record  record_cap bytes; d_record_bytes (device u64) receives the record's size.
 *   1 <= B <= 255. The record never exceeds lowdiff_record_max_bytes(mode, B, sum of caps).
 * ------------------------------------------------------------------------------------------- */
typedef struct {
  const uint32_t* idx;     /* device, ascending unique, lo <= idx < hi */
  const float* val;        /* device */
  const uint64_t* d_nnz;   /* device u64: number of entries */
  uint64_t cap;            /* host: upper bound of *d_nnz */
  float lr;                /* learning rate of this iteration (stored in the record's lr[]) */
} lowdiff_diff_view;

typedef struct {           /* == the first 80 bytes of every record */
  uint8_t magic[8];        /* "LOWDIFF\x01" */
  uint32_t version, mode, B, nranks;
  uint64_t n, lo, hi, t_first, nnz, nent, total_bytes;
} lowdiff_record_header;

uint64_t       lowdiff_record_size(lowdiff_merge_mode mode, uint32_t B, uint64_t nnz, uint64_t nent);
uint64_t       lowdiff_record_max_bytes(lowdiff_merge_mode mode, uint32_t B, uint64_t max_entries);
/* The same bound for a record of the shard [lo, hi): its unique indices are at most hi - lo
 * (max_entries still bounds the STACK entries). At C5 (B = 32, 12.5 M entries per differential,
 * 194.7 M-index shard) 3.6 GB instead of 5.2 GB. */
uint64_t       lowdiff_record_max_bytes_shard(lowdiff_merge_mode mode, uint32_t B, uint64_t max_entries,
                                              uint64_t lo, uint64_t hi);
lowdiff_status lowdiff_batch_merge_workspace_size(uint32_t B, uint64_t max_entries, uint64_t lo,
                                                  uint64_t hi, uint64_t* bytes);
lowdiff_status lowdiff_batch_merge(const lowdiff_diff_view* diffs /* host [B] */, uint32_t B,
                                   lowdiff_merge_mode mode, uint64_t n, uint64_t lo, uint64_t hi,
                                   uint64_t t_first, uint32_t nranks, void* d_record,
                                   uint64_t record_cap, uint64_t* d_record_bytes, void* ws,
                                   uint64_t ws_bytes, lowdiff_stream_t stream);
/* Same, with the diffs' values in `vdt` (`val` then points to bf16 when vdt = BF16): each value is
 * widened to fp32 exactly, so the record equals the one built from the coalesced fp32 lists. This
 * lets a P = 1 ring slot be the compressed pairs buffer itself (zero-copy), bf16 too. */
lowdiff_status lowdiff_batch_merge_ex(const lowdiff_diff_view* diffs, uint32_t B, lowdiff_merge_mode mode,
                                      lowdiff_dtype vdt, uint64_t n, uint64_t lo, uint64_t hi, uint64_t t_first,
                                      uint32_t nranks, void* d_record, uint64_t record_cap,
                                      uint64_t* d_record_bytes, void* ws, uint64_t ws_bytes,
                                      lowdiff_stream_t stream);

/* ---------------------------------------------------------------------------------------------
 * (4) Stage — Step 1, `offload_to_cpu()` non-blocking.
 *   lowdiff_record_bytes: synchronizes `stream`, reads *d_record_bytes; ECAPACITY if the merge
 *     needed more than record_cap bytes (the record was not written).
 *   lowdiff_stage_d2h: async copy of `bytes` record bytes into caller-owned pinned host memory
 *     on copy_stream (a copy engine); byte-identical to the device record.
 * ------------------------------------------------------------------------------------------- */
lowdiff_status lowdiff_record_bytes(const uint64_t* d_record_bytes, uint64_t record_cap,
                                    lowdiff_stream_t stream, uint64_t* bytes /* host */);
lowdiff_status lowdiff_stage_d2h(const void* d_record, uint64_t bytes, void* h_pinned,
                                 uint64_t h_cap, lowdiff_stream_t copy_stream);

/* ---------------------------------------------------------------------------------------------
 * (5) Replay — Recovery, Alg.1 lines 16-24: from a full checkpoint at iteration t,
 *     apply the records of iterations t, t+1, ... in order. Each iteration is a DENSE optimizer
 *     step with gradient 0 at absent indices (Comp^{-1}): SGD (x -= lr*(g + wd x)),
 *     SGD-momentum (torch.optim.SGD conventions), Adam (Eq.1; bias-corrected, eps
 *     after the sqrt). STACK records: one step per iteration (lr = lr[j]). SUM records: one step
 *     with the summed gradient and lr[0] — exact trajectory only for plain SGD (weight decay 0),
 *     so momentum, Adam and SGD with weight decay need allow_accumulated_sum (else EUNSUPPORTED;
 *     reading #13); a SUM record's lr[] must be constant.
 *     Scalars are computed on the host in double and rounded once to fp32.
 *   recs[i].d_record: device record bytes; recs[i].h_head: HOST copy of (at least) its header
 *     and lr[] (e.g. the pinned staging buffer); h_head_len >= 80 + 4B.
 *   st: x (and m = momentum buffer or Adam m, v = Adam v) fp32 device arrays over [lo, hi),
 *     x_bf16 optional device bf16 copy of x written after the last step; st->t, st->adam_step and
 *     st->momentum_initialized are advanced on return (host fields).
 *     x0/m0/v0: optional full checkpoint C^F_t to load from (Alg.1 line 17, M_t <- Load(C^F_t)):
 *     when set, the replay reads the starting state from them and writes the result to x/m/v
 *     (same HBM traffic as in place; the checkpoint stays untouched). NULL = in place.
 * Errors: ECHAIN (t gap/overlap, n/lo/hi/nranks mismatch), ECORRUPT (header; the body through
 *   lowdiff_replay_check), EUNSUPPORTED.
 * ------------------------------------------------------------------------------------------- */
typedef struct {
  int32_t kind;                       /* lowdiff_opt_kind */
  double momentum, dampening, weight_decay, beta1, beta2, eps;
  int32_t nesterov;
  int32_t allow_accumulated_sum;
  int32_t approx_math;                /* Adam only. 0: every op correctly rounded, x/m/v bit-exact vs the
                                         oracle. 1: the step's sqrt and division through MUFU approximations
                                         (rsqrt and a short series for 1/(1 + eps/sqrt(v)); sqrt.approx and
                                         rcp.approx where the series does not apply): m, v as in 0, x within north_star's
                                         fp32 tolerance (1e-6 rel / 1e-7 abs) of the oracle, x_bf16 within
                                         2^-7 rel; no range gate (reading #33). Honoured for
                                         eps >= 2^-40; with a smaller eps the mode-0 kernel runs. */
} lowdiff_opt;

typedef struct {
  float* x; float* m; float* v; uint16_t* x_bf16;
  uint64_t n, lo, hi;
  uint64_t t;                         /* iteration whose G~ is applied next */
  uint64_t adam_step;                 /* Adam step count stored in the full checkpoint */
  int32_t momentum_initialized;
  const float* x0; const float* m0; const float* v0;   /* optional source checkpoint (see above) */
} lowdiff_state;

typedef struct {
  const void* d_record;               /* device */
  const void* h_head;                 /* host: header + lr[] (>= 80 + 4B bytes) */
  uint64_t h_head_len;
} lowdiff_record_view;

lowdiff_status lowdiff_record_parse(const void* h_bytes, uint64_t len, lowdiff_record_header* out);
/* Workspace: 256 B error word + a starts table (4 B per record per 256-parameter warp tile of
 * [lo, hi)) + 2 B per entry of every STACK record (its (it, position) repacked for the dense kernel); the
 * size query reads each record's host header (recs[i].h_head) for mode and entry count. */
lowdiff_status lowdiff_replay_workspace_size(const lowdiff_state* st, const lowdiff_record_view* recs,
                                             uint32_t nrec, uint64_t* bytes);
lowdiff_status lowdiff_replay(lowdiff_state* st, const lowdiff_opt* opt,
                              const lowdiff_record_view* recs, uint32_t nrec, void* ws,
                              uint64_t ws_bytes, lowdiff_stream_t stream);
/* Device validation of the record bodies (a record damaged in storage is what recovery reads):
 * before any replay kernel reads a body, one pass checks that the device header equals the host
 * copy the call was planned from, lo <= idx < hi strictly ascending, and for STACK off[0] = 0,
 * off strictly increasing to off[nnz] = nent, it[] < B strictly increasing within each index.
 * On failure every replay kernel of the call returns without writing (the state is unchanged, no
 * index is used out of bounds). lowdiff_replay_check(ws) synchronizes `stream` and returns
 * ECORRUPT if the last lowdiff_replay with this workspace failed validation (lowdiff_replay itself
 * does not synchronize). lowdiff_replay_parallel validates and checks synchronously itself. */
lowdiff_status lowdiff_replay_check(const void* ws, lowdiff_stream_t stream);

/* ---------------------------------------------------------------------------------------------
 * (5c) Live update — Alg.1 training process, "G_t <- Comp^{-1}(G~_t)" and "M_{t+1} <- M_t +
 *     Adam(o_t, G_t)": the synchronized G~_t of the current iteration, exactly as
 *     lowdiff_allgather_sparse / lowdiff_coalesce leave it in device memory (idx ascending unique in
 *     [lo, hi), val fp32, *d_nnz entries, g->cap >= *d_nnz host bound, g->lr this iteration's lr),
 *     applied to the live shard state in place as ONE dense optimizer step. The arithmetic is that of
 *     lowdiff_replay on a one-iteration record of G~_t, so a later recovery from the differentials
 *     reproduces the live trajectory bit for bit (Finding 1). Unlike lowdiff_replay it never
 *     reads a header on the host and never synchronizes (capturable in a CUDA graph).
 *   st: as lowdiff_replay; st->t, st->adam_step, st->momentum_initialized advance by one step.
 *   ws: lowdiff_update_workspace_size bytes, device, 16-byte aligned, caller-owned.
 * Errors: EINVAL (null pointers, cap > hi - lo, bad state), EWORKSPACE, EUNSUPPORTED (Adam + wd).
 * ------------------------------------------------------------------------------------------- */
lowdiff_status lowdiff_update_workspace_size(const lowdiff_state* st, uint64_t* bytes);
lowdiff_status lowdiff_update(lowdiff_state* st, const lowdiff_opt* opt, const lowdiff_diff_view* g,
                              void* ws, uint64_t ws_bytes, lowdiff_stream_t stream);

/* ---------------------------------------------------------------------------------------------
 * (6) LowDiff+ — training without gradient compression (§5, Algorithm 2; SURVEY
 *     §8(f) NEXT-4). The dense synchronized gradient G_t of the shard [lo, hi) updates
 *       lowdiff_dense_update: the GPU model in place, "M^G_{t+1} <- M^G_t + Adam(o_t, G_t)"
 *                             (Alg. 2 line 7), asynchronously on `stream`;
 *       lowdiff_host_update:  the CPU-resident replica in place, "M^C_{t+1} <- M^C_t + Adam(o_t,
 *                             G_t)" (line 12; the in-memory checkpoint), synchronously
 *                             on the calling thread plus `threads` - 1 workers (>= 1).
 *     Both run the same IEEE fp32 op sequence as lowdiff_replay / lowdiff_update (SGD with
 *     optional weight decay, SGD-momentum, Adam; readings #16, #18, #19), so after the
 *     same gradients the replica equals the GPU model bit for bit ("keep it synchronized").
 *   st: x (and m, v as the optimizer needs) over [lo, hi): DEVICE pointers for the GPU update,
 *       HOST pointers for the host update; x0/m0/v0/x_bf16 must be NULL (in place only);
 *       st->t, st->adam_step, st->momentum_initialized advance by one step.
 *   grad: hi - lo gradient values, fp32 or bf16 (gdt), device (16-byte aligned) resp. host.
 *   lr: this iteration's learning rate.
 * Errors: EINVAL (null/misaligned pointers, bad dtype, x0/m0/v0/x_bf16 set), EUNSUPPORTED (Adam
 *   with weight decay), ECUDA.
 * ------------------------------------------------------------------------------------------- */
lowdiff_status lowdiff_dense_update(lowdiff_state* st, const lowdiff_opt* opt, const void* grad,
                                    lowdiff_dtype gdt, float lr, lowdiff_stream_t stream);
lowdiff_status lowdiff_host_update(lowdiff_state* st, const lowdiff_opt* opt, const void* grad,
                                   lowdiff_dtype gdt, float lr, int32_t threads);

/* ---------------------------------------------------------------------------------------------
 * (5b) Parallel recovery — §4.4 "Parallel recovery module" on Eq. 2 (P:92,
 *     M_n = C^F + C^D_1 + ... + C^D_n): for plain SGD (weight_decay 0) over SUM records that share
 *     one constant lr, the chain's differentials are first merged among themselves — ONE multiway
 *     merge (the paper's pairwise tree in a single level): per index, the record-ascending fp32 sum
 *     of the records' values, absent terms skipped — and the merged differential is applied to the
 *     checkpoint once:  x[i] = x[i] - lr * (v_1[i] + ... + v_R[i]).  One merge touches C^F instead
 *     of R. Its rounding differs from lowdiff_replay's sequential
 *     x - lr v_1 - lr v_2 ...: the two agree within the fp32 tolerance, not bit for bit (the CPU
 *     oracle's parallel recovery is matched bit for bit).
 *   Arguments, chain checks and state updates as lowdiff_replay (m/v unused); at most 256 records.
 *   Errors: as lowdiff_replay; EUNSUPPORTED unless SGD with weight_decay 0, every record SUM and
 *   every lr[] entry equal.
 * ------------------------------------------------------------------------------------------- */
lowdiff_status lowdiff_replay_parallel_workspace_size(const lowdiff_state* st, const lowdiff_record_view* recs,
                                                      uint32_t nrec, uint64_t* bytes);
lowdiff_status lowdiff_replay_parallel(lowdiff_state* st, const lowdiff_opt* opt,
                                       const lowdiff_record_view* recs, uint32_t nrec, void* ws,
                                       uint64_t ws_bytes, lowdiff_stream_t stream);

/* ---------------------------------------------------------------------------------------------
 * Checkpointing configuration model (§3.5 "Optimizing Checkpointing Configuration", P:318-350;
 * SURVEY §8(f) NEXT-3). Host-only arithmetic (fp64), no stream, no device memory.
 *
 * Parameters, all > 0 and finite (EINVAL otherwise), in ONE consistent time unit — the paper's
 * model counts the wasted work of b batched iterations as b/2 time units, i.e. the unit
 * is one training iteration (reading #29):
 *   N   GPUs;  M  mean time between failures;  W  checkpoint write bandwidth (bytes per unit);
 *   S   full checkpoint size (bytes);  T  total run time;  R_F  time to load a full checkpoint;
 *   R_D time to merge (replay) one differential checkpoint onto the full one.
 * Variables: f = full checkpoints per unit of time (FCF = 1/f iterations between them), b =
 * batching size (differentials per batched write).
 *
 * lowdiff_wasted_time: Eq. 3
 *   T_wasted(f, b) = (N T / M) (b/2 + R_F + (R_D/2) (1/(f b) - 1)) + N T S f / W
 * lowdiff_optimal_config: Eq. 5, the stationary point of Eq. 4
 *   f* = cbrt(R_D W^2 / (4 S^2 M^2)),  b* = cbrt(2 S R_D M / W)
 *   and the integer configuration (fcf >= batch >= 1) minimising Eq. 3: batch is floor/ceil(b*),
 *   fcf is floor/ceil of sqrt(2 S M batch / (R_D W)) (the b = batch root of Eq. 4's first line),
 *   clamped to >= batch — exact because Eq. 3 is convex in fcf and its minimum over fcf is convex
 *   in b (ties: smaller fcf, then smaller batch). Outputs are host pointers; any may be NULL.
 * ------------------------------------------------------------------------------------------- */
typedef struct lowdiff_config_model {
  double N, M, W, S, T, R_F, R_D;
} lowdiff_config_model;

lowdiff_status lowdiff_wasted_time(const lowdiff_config_model* m, double f, double b, double* t_wasted);
lowdiff_status lowdiff_optimal_config(const lowdiff_config_model* m, double* f_star, double* b_star,
                                      uint32_t* fcf, uint32_t* batch);

/* ---------------------------------------------------------------------------------------------
 * Instrumentation (bench/tests only; not on the data path).
 *   lowdiff_launch_count: number of kernels this library has launched in the process.
 *   lowdiff_profile_enable(1): from now on, bracket every launch of the named kernel classes
 *     with CUDA events on the launching stream; lowdiff_profile_query sums the elapsed time
 *     (synchronizing the events) of launches whose class name equals `name`, then forgets them.
 *     Classes: "compress_stream", "compress_sample", "compress_select", "coalesce", "merge",
 *     "merge_pack", "replay_dense", "replay_sparse", "starts".
 * ------------------------------------------------------------------------------------------- */
uint64_t       lowdiff_launch_count(void);
/* After a lowdiff_compress on `stream` with workspace `ws` (syncs the stream): out10 = {first-pass
 * threshold key, first-pass candidates found, path (3 = first-pass candidates, fast select; 0 =
 * first-pass candidates, general select; 2 = rescan candidates; 1 = full-array select), k-th key,
 * ties kept, candidate capacity, fine-histogram shift, candidates in the k-th key's fine bin,
 * rescan threshold key, rescan candidates}. */
lowdiff_status lowdiff_compress_stats(const void* ws, uint64_t n, uint64_t k, lowdiff_stream_t stream,
                                      uint64_t* out10);
/* The threshold state of the residual `ws` was last used with (syncs `stream`): out9 =
 * {calls, rescans (path 2), full-array fallbacks (path 1), calls that saw non-finite a, non-finite
 * count of the last call, first-pass candidates of the last call, last k-th key, margin x 2^32,
 * fast-select calls (path 3)}.
 * All zero for a workspace never used by lowdiff_compress. Counters restart when the workspace
 * moves to another residual / n / k. */
lowdiff_status lowdiff_compress_counters(const void* ws, lowdiff_stream_t stream, uint64_t* out9);
/* Test hooks: while enabled, every later lowdiff_compress uses `key` as its first-pass candidate
 * threshold (lowdiff_debug_force_threshold: drives the rescan recovery) or as the rescan's
 * threshold (lowdiff_debug_force_rescan_threshold: drives the exact full-array path). */
lowdiff_status lowdiff_debug_force_threshold(int32_t enable, uint32_t key);
lowdiff_status lowdiff_debug_force_rescan_threshold(int32_t enable, uint32_t key);
lowdiff_status lowdiff_profile_enable(int32_t on);
lowdiff_status lowdiff_profile_query(const char* name, double* total_ms, uint64_t* launches);

#ifdef __cplusplus
}
#endif
#endif /* LOWDIFF_H */
