// C ABI of liblowdiff (include/lowdiff.h): argument validation, workspace sizing, record header
// parsing, NCCL bootstrap, the D2H stage, and instrumentation. All compute runs in the kernels of
// compress.cu / merge.cu / replay.cu.
#include <math.h>
#include <nccl.h>
#include <stdarg.h>
#include <stdio.h>
#include <string.h>

#include <atomic>
#include <mutex>
#include <string>
#include <vector>

#include "common.cuh"
#include "internal.h"

namespace lowdiff {

static thread_local std::string g_last_error;
static std::atomic<uint64_t> g_launches{0};

lowdiff_status fail(lowdiff_status s, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  g_last_error = buf;
  return s;
}

lowdiff_status cuda_status(cudaError_t e, const char* what) {
  if (e == cudaSuccess) return LOWDIFF_OK;
  return fail(LOWDIFF_ECUDA, "%s: %s", what, cudaGetErrorString(e));
}

void note_launch() { g_launches.fetch_add(1, std::memory_order_relaxed); }

// ---- profiling: CUDA events bracketing launches of named kernel classes ----------------------
namespace {
struct ProfRec {
  std::string cls;
  cudaEvent_t a, b;
};
std::mutex g_prof_mu;
bool g_prof_on = false;
std::vector<ProfRec> g_prof;
std::vector<cudaEvent_t> g_ev_pool;

cudaEvent_t get_event() {
  if (!g_ev_pool.empty()) {
    cudaEvent_t e = g_ev_pool.back();
    g_ev_pool.pop_back();
    return e;
  }
  cudaEvent_t e;
  cudaEventCreate(&e);
  return e;
}
}  // namespace

ProfScope::ProfScope(const char* c, cudaStream_t s) : cls(c), stream(s), slot(-1) {
  if (!g_prof_on) return;
  std::lock_guard<std::mutex> lk(g_prof_mu);
  ProfRec r{c, get_event(), get_event()};
  cudaEventRecord(r.a, s);
  g_prof.push_back(r);
  slot = (int)g_prof.size() - 1;
}
ProfScope::~ProfScope() {
  if (slot < 0) return;
  std::lock_guard<std::mutex> lk(g_prof_mu);
  cudaEventRecord(g_prof[slot].b, stream);
}

}  // namespace lowdiff

using namespace lowdiff;

namespace {

bool aligned16(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }

uint64_t psize(lowdiff_dtype d) { return d == LOWDIFF_BF16 ? 2 : 4; }

}  // namespace

struct lowdiff_comm {
  ncclComm_t comm;
  int nranks, rank;
};

extern "C" {

const char* lowdiff_status_string(lowdiff_status s) {
  switch (s) {
    case LOWDIFF_OK: return "ok";
    case LOWDIFF_EINVAL: return "invalid argument";
    case LOWDIFF_EWORKSPACE: return "workspace too small";
    case LOWDIFF_ECAPACITY: return "output capacity exceeded";
    case LOWDIFF_ECHAIN: return "records do not form a chain from the state";
    case LOWDIFF_ECORRUPT: return "corrupt record";
    case LOWDIFF_EUNSUPPORTED: return "unsupported combination";
    case LOWDIFF_ECUDA: return "CUDA error";
    case LOWDIFF_ENCCL: return "NCCL error";
    case LOWDIFF_ETIMEOUT: return "peer-memory wait timed out";
  }
  return "unknown status";
}

const char* lowdiff_last_error(void) { return g_last_error.c_str(); }
const char* lowdiff_version(void) { return "lowdiff-b200 0.1 (sm_100a)"; }

uint64_t lowdiff_k_for_density(uint64_t n, double rho) {
  double k = floor(rho * (double)n);
  if (k < 1.0) k = 1.0;
  if (k > (double)n) k = (double)n;
  return (uint64_t)k;
}

uint64_t lowdiff_pairs_bytes(uint64_t k, lowdiff_dtype vdt) { return pad16(4 * k) + pad16(psize(vdt) * k); }

lowdiff_status lowdiff_shard_bounds(uint64_t n, int32_t nranks, int32_t rank, uint64_t* lo, uint64_t* hi) {
  if (nranks < 1 || rank < 0 || rank >= nranks || !lo || !hi) return fail(LOWDIFF_EINVAL, "shard_bounds: bad rank");
  *lo = (uint64_t)((unsigned __int128)rank * n / (unsigned)nranks);
  *hi = (uint64_t)((unsigned __int128)(rank + 1) * n / (unsigned)nranks);
  return LOWDIFF_OK;
}

// ---- (0) plan: the problem statement and the record-boundary policy (reading #25) -------------
lowdiff_status lowdiff_plan_init(lowdiff_plan* p, uint64_t n, double rho, uint32_t B, uint32_t full_every,
                                 lowdiff_dtype gdt, lowdiff_dtype vdt, int32_t nranks, int32_t rank) {
  if (!p) return fail(LOWDIFF_EINVAL, "plan_init: null plan");
  if (n == 0 || n >= (1ull << 31)) return fail(LOWDIFF_EINVAL, "plan_init: need 1 <= n < 2^31");
  if (!(rho > 0.0 && rho <= 1.0)) return fail(LOWDIFF_EINVAL, "plan_init: rho must be in (0, 1]");
  if (B == 0 || B > 255) return fail(LOWDIFF_EINVAL, "plan_init: need 1 <= B <= 255");
  if ((gdt != LOWDIFF_F32 && gdt != LOWDIFF_BF16) || (vdt != LOWDIFF_F32 && vdt != LOWDIFF_BF16))
    return fail(LOWDIFF_EINVAL, "plan_init: bad dtype");
  uint64_t lo, hi;
  lowdiff_status s = lowdiff_shard_bounds(n, nranks, rank, &lo, &hi);
  if (s) return s;
  p->n = n; p->rho = rho; p->k = lowdiff_k_for_density(n, rho); p->B = B; p->full_every = full_every;
  p->gdt = gdt; p->vdt = vdt; p->nranks = nranks; p->rank = rank; p->lo = lo; p->hi = hi;
  return LOWDIFF_OK;
}

lowdiff_status lowdiff_plan_record_due(const lowdiff_plan* p, uint64_t t, int32_t* close_record,
                                       uint32_t* batch_len, int32_t* full_checkpoint_due) {
  if (!p || p->B == 0) return fail(LOWDIFF_EINVAL, "plan_record_due: bad plan");
  const uint64_t F = p->full_every;
  const uint64_t f = F ? t / F * F : 0;            // the full checkpoint the open chain starts from
  const uint64_t pos = (t - f) % p->B;             // t's place in its record
  const bool full_next = F && (t + 1) % F == 0;    // a full checkpoint is due before t + 1
  if (full_checkpoint_due) *full_checkpoint_due = (F ? t % F == 0 : t == 0) ? 1 : 0;
  if (close_record) *close_record = (pos + 1 == p->B || full_next) ? 1 : 0;
  if (batch_len) *batch_len = (uint32_t)(pos + 1);
  return LOWDIFF_OK;
}

// ---- (1) compress ---------------------------------------------------------------------------
lowdiff_status lowdiff_compress_workspace_size(uint64_t n, uint64_t k, uint64_t* bytes) {
  if (!bytes || n == 0 || n >= (1ull << 31) || k == 0 || k > n)
    return fail(LOWDIFF_EINVAL, "compress_workspace_size: need 1 <= k <= n < 2^31");
  *bytes = compress_ws_bytes(n, k);
  return LOWDIFF_OK;
}

lowdiff_status lowdiff_compress(const void* grad, lowdiff_dtype gdt, float* residual, uint64_t n,
                                uint64_t k, void* pairs, lowdiff_dtype vdt, void* ws, uint64_t ws_bytes,
                                lowdiff_stream_t stream) {
  if (n == 0 || n >= (1ull << 31) || k == 0 || k > n)
    return fail(LOWDIFF_EINVAL, "compress: need 1 <= k <= n < 2^31 (n=%llu k=%llu)",
                (unsigned long long)n, (unsigned long long)k);
  if ((gdt != LOWDIFF_F32 && gdt != LOWDIFF_BF16) || (vdt != LOWDIFF_F32 && vdt != LOWDIFF_BF16))
    return fail(LOWDIFF_EINVAL, "compress: bad dtype");
  if (!grad || !residual || !pairs || !ws || !aligned16(grad) || !aligned16(residual) ||
      !aligned16(pairs) || !aligned16(ws))
    return fail(LOWDIFF_EINVAL, "compress: null or non-16-byte-aligned pointer");
  if (ws_bytes < compress_ws_bytes(n, k))
    return fail(LOWDIFF_EWORKSPACE, "compress: workspace %llu < %llu", (unsigned long long)ws_bytes,
                (unsigned long long)compress_ws_bytes(n, k));
  return compress_run(grad, gdt, residual, n, k, pairs, vdt, ws, (cudaStream_t)stream);
}

// ---- (2) all-gather + coalesce ------------------------------------------------------------------
int32_t lowdiff_comm_unique_id_bytes(void) { return (int32_t)sizeof(ncclUniqueId); }

lowdiff_status lowdiff_comm_get_unique_id(uint8_t* id) {
  if (!id) return fail(LOWDIFF_EINVAL, "comm_get_unique_id: null");
  ncclUniqueId u;
  ncclResult_t r = ncclGetUniqueId(&u);
  if (r != ncclSuccess) return fail(LOWDIFF_ENCCL, "ncclGetUniqueId: %s", ncclGetErrorString(r));
  memcpy(id, &u, sizeof(u));
  return LOWDIFF_OK;
}

lowdiff_status lowdiff_comm_init(lowdiff_comm** comm, const uint8_t* id, int32_t nranks, int32_t rank) {
  if (!comm || !id || nranks < 1 || rank < 0 || rank >= nranks) return fail(LOWDIFF_EINVAL, "comm_init");
  ncclUniqueId u;
  memcpy(&u, id, sizeof(u));
  lowdiff_comm* c = new lowdiff_comm();
  ncclResult_t r = ncclCommInitRank(&c->comm, nranks, u, rank);
  if (r != ncclSuccess) {
    delete c;
    return fail(LOWDIFF_ENCCL, "ncclCommInitRank: %s", ncclGetErrorString(r));
  }
  c->nranks = nranks;
  c->rank = rank;
  *comm = c;
  return LOWDIFF_OK;
}

lowdiff_status lowdiff_comm_destroy(lowdiff_comm* comm) {
  if (!comm) return LOWDIFF_OK;
  ncclResult_t r = ncclCommDestroy(comm->comm);
  delete comm;
  if (r != ncclSuccess) return fail(LOWDIFF_ENCCL, "ncclCommDestroy: %s", ncclGetErrorString(r));
  return LOWDIFF_OK;
}

static lowdiff_status check_coalesce_args(int32_t P, uint64_t k, lowdiff_dtype vdt, uint64_t lo, uint64_t hi) {
  if (P < 1 || P > kMaxLists) return fail(LOWDIFF_EINVAL, "coalesce: 1 <= nranks <= %d", kMaxLists);
  if (k == 0 || lo >= hi || hi >= (1ull << 31) + 1 || (vdt != LOWDIFF_F32 && vdt != LOWDIFF_BF16))
    return fail(LOWDIFF_EINVAL, "coalesce: bad k/lo/hi/vdt");
  if ((uint64_t)P * k >= (1ull << 31)) return fail(LOWDIFF_EINVAL, "coalesce: P*k must be < 2^31");
  return LOWDIFF_OK;
}

lowdiff_status lowdiff_coalesce_workspace_size(int32_t nranks, uint64_t k, lowdiff_dtype vdt, uint64_t lo,
                                               uint64_t hi, uint64_t* bytes) {
  lowdiff_status s = check_coalesce_args(nranks, k, vdt, lo, hi);
  if (s) return s;
  if (!bytes) return fail(LOWDIFF_EINVAL, "null bytes");
  *bytes = merge_ws_bytes(nranks, (uint64_t)nranks * k, lo, hi);
  return LOWDIFF_OK;
}

lowdiff_status lowdiff_coalesce(const void* gathered, int32_t nranks, uint64_t k, lowdiff_dtype vdt,
                                uint64_t lo, uint64_t hi, int32_t average, uint32_t* out_idx, float* out_val,
                                uint64_t out_cap, uint64_t* d_out_nnz, void* ws, uint64_t ws_bytes,
                                lowdiff_stream_t stream) {
  lowdiff_status s = check_coalesce_args(nranks, k, vdt, lo, hi);
  if (s) return s;
  if (!gathered || !out_idx || !out_val || !d_out_nnz || !ws || !aligned16(gathered) || !aligned16(ws) ||
      !aligned16(out_idx) || !aligned16(out_val))
    return fail(LOWDIFF_EINVAL, "coalesce: null or misaligned pointer");
  const uint64_t need = (uint64_t)nranks * k < hi - lo ? (uint64_t)nranks * k : hi - lo;
  if (out_cap < need) return fail(LOWDIFF_EINVAL, "coalesce: out_cap %llu < min(P*k, hi-lo) = %llu",
                                  (unsigned long long)out_cap, (unsigned long long)need);
  const uint64_t wsz = merge_ws_bytes(nranks, (uint64_t)nranks * k, lo, hi);
  if (ws_bytes < wsz) return fail(LOWDIFF_EWORKSPACE, "coalesce: workspace too small");
  ListSet* ls = new ListSet();
  ls->L = nranks;
  ls->bf16 = vdt == LOWDIFF_BF16;
  const uint64_t pb = lowdiff_pairs_bytes(k, vdt);
  for (int p = 0; p < nranks; ++p) {
    const uint8_t* base = static_cast<const uint8_t*>(gathered) + (uint64_t)p * pb;
    ls->list[p].idx = reinterpret_cast<const uint32_t*>(base);
    ls->list[p].val = base + pad16(4 * k);
    ls->list[p].d_len = nullptr;
    ls->list[p].len = k;
  }
  s = merge_run(*ls, kCoalesce, lo, hi, average, (uint64_t)nranks * k, out_idx, out_val, out_cap,
                d_out_nnz, nullptr, 0, 0, 0, nullptr, 0, nullptr, ws, (cudaStream_t)stream);
  delete ls;
  return s;
}

lowdiff_status lowdiff_allgather_sparse_workspace_size(int32_t nranks, uint64_t k, lowdiff_dtype vdt,
                                                       uint64_t lo, uint64_t hi, uint64_t* bytes) {
  uint64_t cws = 0;
  lowdiff_status s = lowdiff_coalesce_workspace_size(nranks, k, vdt, lo, hi, &cws);
  if (s) return s;
  *bytes = align256(cws) + (nranks > 1 ? align256((uint64_t)nranks * lowdiff_pairs_bytes(k, vdt)) : 0);
  return LOWDIFF_OK;
}

lowdiff_status lowdiff_allgather_sparse(lowdiff_comm* comm, const void* pairs, uint64_t k, lowdiff_dtype vdt,
                                        uint64_t lo, uint64_t hi, int32_t average, uint32_t* out_idx,
                                        float* out_val, uint64_t out_cap, uint64_t* d_out_nnz, void* ws,
                                        uint64_t ws_bytes, lowdiff_stream_t stream) {
  const int P = comm ? comm->nranks : 1;
  uint64_t need = 0;
  lowdiff_status s = lowdiff_allgather_sparse_workspace_size(P, k, vdt, lo, hi, &need);
  if (s) return s;
  if (!pairs || !ws || !aligned16(pairs) || !aligned16(ws) || !aligned16(out_idx) || !aligned16(out_val))
    return fail(LOWDIFF_EINVAL, "allgather_sparse: pointer");
  if (ws_bytes < need) return fail(LOWDIFF_EWORKSPACE, "allgather_sparse: workspace too small");
  uint64_t cws = 0;
  lowdiff_coalesce_workspace_size(P, k, vdt, lo, hi, &cws);
  const void* gathered = pairs;
  if (P > 1) {
    uint8_t* gbuf = static_cast<uint8_t*>(ws) + align256(cws);
    const uint64_t pb = lowdiff_pairs_bytes(k, vdt);
    ncclResult_t r = ncclAllGather(pairs, gbuf, pb, ncclUint8, comm->comm, (cudaStream_t)stream);
    if (r != ncclSuccess) return fail(LOWDIFF_ENCCL, "ncclAllGather: %s", ncclGetErrorString(r));
    gathered = gbuf;
  }
  return lowdiff_coalesce(gathered, P, k, vdt, lo, hi, average, out_idx, out_val, out_cap, d_out_nnz, ws,
                          align256(cws), stream);
}

// ---- (3) batch merge -------------------------------------------------------------------------
uint64_t lowdiff_record_size(lowdiff_merge_mode mode, uint32_t B, uint64_t nnz, uint64_t nent) {
  uint64_t s = 80 + pad16(4ull * B) + pad16(4 * nnz);
  if (mode == LOWDIFF_MERGE_SUM) return s + pad16(4 * nnz);
  return s + pad16(4 * (nnz + 1)) + pad16(nent) + pad16(4 * nent);
}

uint64_t lowdiff_record_max_bytes(lowdiff_merge_mode mode, uint32_t B, uint64_t max_entries) {
  return lowdiff_record_size(mode, B, max_entries, max_entries);
}

uint64_t lowdiff_record_max_bytes_shard(lowdiff_merge_mode mode, uint32_t B, uint64_t max_entries, uint64_t lo,
                                        uint64_t hi) {
  const uint64_t u = hi > lo && hi - lo < max_entries ? hi - lo : max_entries;   // unique indices <= shard
  return lowdiff_record_size(mode, B, u, max_entries);
}

lowdiff_status lowdiff_batch_merge_workspace_size(uint32_t B, uint64_t max_entries, uint64_t lo, uint64_t hi,
                                                  uint64_t* bytes) {
  if (!bytes || B == 0 || B > 255 || lo >= hi || hi > (1ull << 31) || max_entries >= (1ull << 31))
    return fail(LOWDIFF_EINVAL, "batch_merge_workspace_size: bad arguments");
  *bytes = merge_ws_bytes((int)B, max_entries ? max_entries : 1, lo, hi);
  return LOWDIFF_OK;
}

lowdiff_status lowdiff_batch_merge(const lowdiff_diff_view* diffs, uint32_t B, lowdiff_merge_mode mode,
                                   uint64_t n, uint64_t lo, uint64_t hi, uint64_t t_first, uint32_t nranks,
                                   void* d_record, uint64_t record_cap, uint64_t* d_record_bytes, void* ws,
                                   uint64_t ws_bytes, lowdiff_stream_t stream) {
  return lowdiff_batch_merge_ex(diffs, B, mode, LOWDIFF_F32, n, lo, hi, t_first, nranks, d_record, record_cap,
                                d_record_bytes, ws, ws_bytes, stream);
}

lowdiff_status lowdiff_batch_merge_ex(const lowdiff_diff_view* diffs, uint32_t B, lowdiff_merge_mode mode,
                                      lowdiff_dtype vdt, uint64_t n, uint64_t lo, uint64_t hi, uint64_t t_first,
                                      uint32_t nranks, void* d_record, uint64_t record_cap,
                                      uint64_t* d_record_bytes, void* ws, uint64_t ws_bytes,
                                      lowdiff_stream_t stream) {
  if (vdt != LOWDIFF_F32 && vdt != LOWDIFF_BF16) return fail(LOWDIFF_EINVAL, "batch_merge: bad value dtype");
  if (!diffs || B == 0 || B > 255 || lo >= hi || hi > n || n >= (1ull << 31) ||
      (mode != LOWDIFF_MERGE_SUM && mode != LOWDIFF_MERGE_STACK))
    return fail(LOWDIFF_EINVAL, "batch_merge: bad B/mode/range");
  if (!d_record || !d_record_bytes || !ws || !aligned16(d_record) || !aligned16(ws))
    return fail(LOWDIFF_EINVAL, "batch_merge: null or misaligned pointer");
  uint64_t max_entries = 0;
  for (uint32_t j = 0; j < B; ++j) {
    if (!diffs[j].idx || !diffs[j].val || !diffs[j].d_nnz) return fail(LOWDIFF_EINVAL, "batch_merge: diff %u", j);
    max_entries += diffs[j].cap;
  }
  if (max_entries == 0) max_entries = 1;
  if (max_entries >= (1ull << 31)) return fail(LOWDIFF_EINVAL, "batch_merge: too many entries");
  const uint64_t wsz = merge_ws_bytes((int)B, max_entries, lo, hi);
  if (ws_bytes < wsz) return fail(LOWDIFF_EWORKSPACE, "batch_merge: workspace too small");
  ListSet* ls = new ListSet();
  ls->L = (int)B;
  ls->bf16 = vdt == LOWDIFF_BF16;
  float lr[256];
  for (uint32_t j = 0; j < B; ++j) {
    ls->list[j].idx = diffs[j].idx;
    ls->list[j].val = diffs[j].val;
    ls->list[j].d_len = diffs[j].d_nnz;
    ls->list[j].len = diffs[j].cap;
    lr[j] = diffs[j].lr;
  }
  lowdiff_status s = merge_run(*ls, mode == LOWDIFF_MERGE_SUM ? kMergeSum : kMergeStack, lo, hi, 0, max_entries,
                               nullptr, nullptr, 0, nullptr, lr, n, t_first, nranks, d_record, record_cap,
                               d_record_bytes, ws, (cudaStream_t)stream);
  delete ls;
  return s;
}

// ---- (4) stage -----------------------------------------------------------------------------------
lowdiff_status lowdiff_record_bytes(const uint64_t* d_record_bytes, uint64_t record_cap, lowdiff_stream_t stream,
                                    uint64_t* bytes) {
  if (!d_record_bytes || !bytes) return fail(LOWDIFF_EINVAL, "record_bytes: null");
  uint64_t v = 0;
  LD_CUDA(cudaMemcpyAsync(&v, d_record_bytes, 8, cudaMemcpyDeviceToHost, (cudaStream_t)stream), "record_bytes copy");
  LD_CUDA(cudaStreamSynchronize((cudaStream_t)stream), "record_bytes sync");
  *bytes = v;
  if (v > record_cap) return fail(LOWDIFF_ECAPACITY, "record needs %llu bytes > capacity %llu",
                                  (unsigned long long)v, (unsigned long long)record_cap);
  return LOWDIFF_OK;
}

lowdiff_status lowdiff_stage_d2h(const void* d_record, uint64_t bytes, void* h_pinned, uint64_t h_cap,
                                 lowdiff_stream_t copy_stream) {
  if (!d_record || !h_pinned) return fail(LOWDIFF_EINVAL, "stage_d2h: null");
  if (bytes > h_cap) return fail(LOWDIFF_ECAPACITY, "stage_d2h: %llu bytes > host capacity %llu",
                                 (unsigned long long)bytes, (unsigned long long)h_cap);
  LD_CUDA(cudaMemcpyAsync(h_pinned, d_record, bytes, cudaMemcpyDeviceToHost, (cudaStream_t)copy_stream),
          "stage_d2h");
  return LOWDIFF_OK;
}

// ---- (5) replay ------------------------------------------------------------------------------------
lowdiff_status lowdiff_record_parse(const void* h_bytes, uint64_t len, lowdiff_record_header* out) {
  if (!h_bytes || !out || len < 80) return fail(LOWDIFF_ECORRUPT, "record_parse: short");
  lowdiff_record_header h;
  memcpy(&h, h_bytes, 80);
  static const uint8_t magic[8] = {'L', 'O', 'W', 'D', 'I', 'F', 'F', 1};
  if (memcmp(h.magic, magic, 8) != 0 || h.version != 1 || h.mode > 1 || h.B == 0 || h.B > 255 ||
      h.lo >= h.hi || h.hi > h.n || (h.mode == LOWDIFF_MERGE_SUM && h.nent != h.nnz) ||
      h.nnz > h.hi - h.lo || h.total_bytes != lowdiff_record_size((lowdiff_merge_mode)h.mode, h.B, h.nnz, h.nent))
    return fail(LOWDIFF_ECORRUPT, "record_parse: bad header");
  *out = h;
  return LOWDIFF_OK;
}

static lowdiff_status build_recinfo(const lowdiff_state* st, const lowdiff_opt* o, const lowdiff_record_view* recs,
                                    uint32_t nrec, std::vector<RecInfo>& R) {
  R.resize(nrec);
  uint64_t t = st->t;
  uint32_t nranks0 = 0;
  for (uint32_t q = 0; q < nrec; ++q) {
    lowdiff_record_header h;
    if (!recs[q].d_record || !recs[q].h_head || !aligned16(recs[q].d_record))
      return fail(LOWDIFF_EINVAL, "replay: record %u pointers", q);
    lowdiff_status s = lowdiff_record_parse(recs[q].h_head, recs[q].h_head_len, &h);
    if (s) return s;
    if (recs[q].h_head_len < 80 + 4ull * h.B) return fail(LOWDIFF_EINVAL, "replay: h_head shorter than header+lr");
    if (q == 0) nranks0 = h.nranks;
    if (h.n != st->n || h.lo != st->lo || h.hi != st->hi || h.nranks != nranks0)
      return fail(LOWDIFF_ECHAIN, "replay: record %u is for another shard/model", q);
    if (h.t_first != t) return fail(LOWDIFF_ECHAIN, "replay: record %u starts at t=%llu, expected %llu", q,
                                    (unsigned long long)h.t_first, (unsigned long long)t);
    t += h.B;
    const float* lr = reinterpret_cast<const float*>(static_cast<const uint8_t*>(recs[q].h_head) + 80);
    if (h.mode == LOWDIFF_MERGE_SUM) {
      if ((o->kind != LOWDIFF_OPT_SGD || o->weight_decay != 0.0) && !o->allow_accumulated_sum)   // reading #13
        return fail(LOWDIFF_EUNSUPPORTED,
                    "replay: SUM record with momentum, Adam or weight decay needs allow_accumulated_sum");
      for (uint32_t j = 1; j < h.B; ++j)
        if (memcmp(&lr[j], &lr[0], 4) != 0) return fail(LOWDIFF_EUNSUPPORTED, "replay: SUM record with varying lr");
    }
    RecInfo& r = R[q];
    r.d = static_cast<const uint8_t*>(recs[q].d_record);
    r.mode = h.mode;
    r.B = h.B;
    r.nnz = h.nnz;
    r.nent = h.nent;
    r.off_lr = 80;
    r.off_idx = 80 + pad16(4ull * h.B);
    if (h.mode == LOWDIFF_MERGE_SUM) {
      r.off_val = r.off_idx + pad16(4 * h.nnz);
      r.off_off = r.off_it = 0;
    } else {
      r.off_off = r.off_idx + pad16(4 * h.nnz);
      r.off_it = r.off_off + pad16(4 * (h.nnz + 1));
      r.off_val = r.off_it + pad16(h.nent);
    }
    r.h_lr = lr;
    r.h_head_bytes = recs[q].h_head;
  }
  return LOWDIFF_OK;
}

static lowdiff_status check_state(const lowdiff_state* st, const lowdiff_opt* o) {
  if (!st || !o || !st->x || st->lo >= st->hi || st->hi > st->n || st->n >= (1ull << 31))
    return fail(LOWDIFF_EINVAL, "replay: bad state");
  if (o->kind < 0 || o->kind > 2) return fail(LOWDIFF_EINVAL, "replay: bad optimizer kind");
  if (o->kind == LOWDIFF_OPT_ADAM && o->weight_decay != 0.0)
    return fail(LOWDIFF_EUNSUPPORTED, "replay: Adam with weight decay");
  if (o->kind != LOWDIFF_OPT_SGD && !st->m) return fail(LOWDIFF_EINVAL, "replay: m required");
  if (o->kind == LOWDIFF_OPT_ADAM && !st->v) return fail(LOWDIFF_EINVAL, "replay: v required");
  if (!aligned16(st->x) || (st->m && !aligned16(st->m)) || (st->v && !aligned16(st->v)) ||
      (st->x_bf16 && (reinterpret_cast<uintptr_t>(st->x_bf16) & 7u)) ||
      (st->x0 && !aligned16(st->x0)) || (st->m0 && !aligned16(st->m0)) || (st->v0 && !aligned16(st->v0)))
    return fail(LOWDIFF_EINVAL, "replay: misaligned state");
  return LOWDIFF_OK;
}

lowdiff_status lowdiff_replay_workspace_size(const lowdiff_state* st, const lowdiff_record_view* recs, uint32_t nrec,
                                             uint64_t* bytes) {
  if (!st || !bytes || st->lo >= st->hi) return fail(LOWDIFF_EINVAL, "replay_workspace_size");
  if (nrec && !recs) return fail(LOWDIFF_EINVAL, "replay_workspace_size: null records");
  std::vector<RecInfo> R(nrec);                    // only mode and nent size the workspace
  for (uint32_t q = 0; q < nrec; ++q) {
    lowdiff_record_header h;
    if (!recs[q].h_head) return fail(LOWDIFF_EINVAL, "replay_workspace_size: record %u has no host header", q);
    const lowdiff_status s = lowdiff_record_parse(recs[q].h_head, recs[q].h_head_len, &h);
    if (s) return s;
    R[q].mode = h.mode;
    R[q].nent = h.nent;
  }
  *bytes = replay_ws_bytes(st->hi - st->lo, R.data(), nrec) + 256;
  return LOWDIFF_OK;
}

lowdiff_status lowdiff_replay(lowdiff_state* st, const lowdiff_opt* opt, const lowdiff_record_view* recs,
                              uint32_t nrec, void* ws, uint64_t ws_bytes, lowdiff_stream_t stream) {
  lowdiff_status s = check_state(st, opt);
  if (s) return s;
  if (nrec && !recs) return fail(LOWDIFF_EINVAL, "replay: null records");
  std::vector<RecInfo> R;
  s = build_recinfo(st, opt, recs, nrec, R);
  if (s) return s;
  if (nrec == 0) return LOWDIFF_OK;
  if (!ws || !aligned16(ws) || ws_bytes < replay_ws_bytes(st->hi - st->lo, R.data(), nrec))
    return fail(LOWDIFF_EWORKSPACE, "replay: workspace too small");
  return replay_run(st, opt, R.data(), nrec, ws, (cudaStream_t)stream);
}

lowdiff_status lowdiff_replay_check(const void* ws, lowdiff_stream_t stream) {
  if (!ws) return fail(LOWDIFF_EINVAL, "replay_check: null workspace");
  return replay_check(ws, (cudaStream_t)stream);
}

lowdiff_status lowdiff_update_workspace_size(const lowdiff_state* st, uint64_t* bytes) {
  if (!st || !bytes || st->lo >= st->hi) return fail(LOWDIFF_EINVAL, "update_workspace_size");
  *bytes = replay_ws_bytes(st->hi - st->lo, nullptr, 1) + 256;
  return LOWDIFF_OK;
}

lowdiff_status lowdiff_update(lowdiff_state* st, const lowdiff_opt* opt, const lowdiff_diff_view* g, void* ws,
                              uint64_t ws_bytes, lowdiff_stream_t stream) {
  lowdiff_status s = check_state(st, opt);
  if (s) return s;
  if (!g || !g->idx || !g->val || !g->d_nnz) return fail(LOWDIFF_EINVAL, "update: null gradient view");
  if (g->cap > st->hi - st->lo) return fail(LOWDIFF_EINVAL, "update: cap exceeds the shard length");
  RecInfo r;                                       // G~_t as a one-iteration SUM list (count on device)
  r.d = nullptr;
  r.mode = LOWDIFF_MERGE_SUM;
  r.B = 1;
  r.nnz = r.nent = g->cap;
  r.off_lr = r.off_idx = r.off_val = r.off_off = r.off_it = 0;
  r.h_lr = &g->lr;
  r.live_idx = g->idx;
  r.live_val = g->val;
  r.d_nnz = g->d_nnz;
  if (!ws || !aligned16(ws) || ws_bytes < replay_ws_bytes(st->hi - st->lo, &r, 1))
    return fail(LOWDIFF_EWORKSPACE, "update: workspace too small");
  return replay_run(st, opt, &r, 1, ws, (cudaStream_t)stream);
}

static lowdiff_status check_dense(const lowdiff_state* st, const lowdiff_opt* opt, const void* grad, int gdt) {
  lowdiff_status s = check_state(st, opt);
  if (s) return s;
  if (!grad) return fail(LOWDIFF_EINVAL, "dense update: null gradient");
  if (gdt != LOWDIFF_F32 && gdt != LOWDIFF_BF16) return fail(LOWDIFF_EINVAL, "dense update: gradient dtype");
  if (st->x0 || st->m0 || st->v0 || st->x_bf16)
    return fail(LOWDIFF_EINVAL, "dense update: in place only (x0/m0/v0/x_bf16 must be NULL)");
  return LOWDIFF_OK;
}

lowdiff_status lowdiff_dense_update(lowdiff_state* st, const lowdiff_opt* opt, const void* grad, lowdiff_dtype gdt,
                                    float lr, lowdiff_stream_t stream) {
  lowdiff_status s = check_dense(st, opt, grad, gdt);
  if (s) return s;
  if (!aligned16(grad)) return fail(LOWDIFF_EINVAL, "dense_update: misaligned gradient");
  return dense_update_run(st, opt, grad, gdt, lr, (cudaStream_t)stream);
}

lowdiff_status lowdiff_host_update(lowdiff_state* st, const lowdiff_opt* opt, const void* grad, lowdiff_dtype gdt,
                                   float lr, int32_t threads) {
  lowdiff_status s = check_dense(st, opt, grad, gdt);
  if (s) return s;
  DenseStep d;
  dense_update_scalars(st, opt, lr, &d);
  host_update_run(d, st->x, st->m, st->v, grad, gdt == LOWDIFF_BF16, st->hi - st->lo, threads);
  return LOWDIFF_OK;
}

static lowdiff_status parallel_supported(const lowdiff_opt* o, const std::vector<RecInfo>& R) {
  if (o->kind != LOWDIFF_OPT_SGD || o->weight_decay != 0.0)
    return fail(LOWDIFF_EUNSUPPORTED, "replay_parallel: plain SGD (weight_decay 0) only");
  if (R.size() > (size_t)kMaxLists) return fail(LOWDIFF_EUNSUPPORTED, "replay_parallel: more than %d records", kMaxLists);
  for (const RecInfo& r : R) {
    if (r.mode != LOWDIFF_MERGE_SUM) return fail(LOWDIFF_EUNSUPPORTED, "replay_parallel: SUM records only");
    for (uint32_t j = 0; j < r.B; ++j)
      if (r.h_lr[j] != R[0].h_lr[0]) return fail(LOWDIFF_EUNSUPPORTED, "replay_parallel: lr must be one constant");
  }
  return LOWDIFF_OK;
}

lowdiff_status lowdiff_replay_parallel_workspace_size(const lowdiff_state* st, const lowdiff_record_view* recs,
                                                      uint32_t nrec, uint64_t* bytes) {
  if (!st || !bytes || st->lo >= st->hi || (nrec && !recs)) return fail(LOWDIFF_EINVAL, "replay_parallel_workspace_size");
  uint64_t entries = 0;
  for (uint32_t q = 0; q < nrec; ++q) {
    lowdiff_record_header h;
    lowdiff_status s = lowdiff_record_parse(recs[q].h_head, recs[q].h_head_len, &h);
    if (s) return s;
    entries += h.nnz;
  }
  *bytes = replay_parallel_ws_bytes(nrec ? nrec : 1, entries, st->lo, st->hi);
  return LOWDIFF_OK;
}

lowdiff_status lowdiff_replay_parallel(lowdiff_state* st, const lowdiff_opt* opt, const lowdiff_record_view* recs,
                                       uint32_t nrec, void* ws, uint64_t ws_bytes, lowdiff_stream_t stream) {
  lowdiff_status s = check_state(st, opt);
  if (s) return s;
  if (nrec && !recs) return fail(LOWDIFF_EINVAL, "replay_parallel: null records");
  std::vector<RecInfo> R;
  s = build_recinfo(st, opt, recs, nrec, R);
  if (s) return s;
  if (nrec == 0) return LOWDIFF_OK;
  s = parallel_supported(opt, R);
  if (s) return s;
  uint64_t entries = 0;
  for (const RecInfo& r : R) entries += r.nnz;
  if (!ws || !aligned16(ws) || ws_bytes < replay_parallel_ws_bytes(nrec, entries, st->lo, st->hi))
    return fail(LOWDIFF_EWORKSPACE, "replay_parallel: workspace too small");
  return replay_parallel_run(st, R.data(), nrec, ws, (cudaStream_t)stream);
}

// ---- instrumentation ------------------------------------------------------------------------------
uint64_t lowdiff_launch_count(void) { return g_launches.load(); }

lowdiff_status lowdiff_debug_force_threshold(int32_t enable, uint32_t key) {
  compress_force_threshold(0, enable, key);
  return LOWDIFF_OK;
}

lowdiff_status lowdiff_debug_force_rescan_threshold(int32_t enable, uint32_t key) {
  compress_force_threshold(1, enable, key);
  return LOWDIFF_OK;
}

lowdiff_status lowdiff_compress_counters(const void* ws, lowdiff_stream_t stream, uint64_t* out9) {
  if (!ws || !out9) return fail(LOWDIFF_EINVAL, "compress_counters: null");
  return compress_counters(ws, (cudaStream_t)stream, out9);
}

lowdiff_status lowdiff_compress_stats(const void* ws, uint64_t n, uint64_t k, lowdiff_stream_t stream,
                                      uint64_t* out10) {
  if (!ws || !out10) return fail(LOWDIFF_EINVAL, "compress_stats: null");
  return compress_stats(ws, n, k, out10, (cudaStream_t)stream);
}

lowdiff_status lowdiff_profile_enable(int32_t on) {
  std::lock_guard<std::mutex> lk(g_prof_mu);
  g_prof_on = on != 0;
  return LOWDIFF_OK;
}

lowdiff_status lowdiff_profile_query(const char* name, double* total_ms, uint64_t* launches) {
  if (!name || !total_ms || !launches) return fail(LOWDIFF_EINVAL, "profile_query: null");
  std::lock_guard<std::mutex> lk(g_prof_mu);
  double tot = 0;
  uint64_t cnt = 0;
  std::vector<ProfRec> keep;
  for (auto& r : g_prof) {
    if (r.cls == name) {
      cudaError_t e = cudaEventSynchronize(r.b);
      if (e != cudaSuccess) return cuda_status(e, "profile_query");
      float ms = 0;
      cudaEventElapsedTime(&ms, r.a, r.b);
      tot += ms;
      ++cnt;
      g_ev_pool.push_back(r.a);
      g_ev_pool.push_back(r.b);
    } else {
      keep.push_back(r);
    }
  }
  g_prof.swap(keep);
  *total_ms = tot;
  *launches = cnt;
  return LOWDIFF_OK;
}

}  // extern "C"
