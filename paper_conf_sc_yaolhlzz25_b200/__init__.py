"""paper_conf_sc_yaolhlzz25_b200 — Python binding of liblowdiff (include/lowdiff.h).

LowDiff's data-parallel hot path (Yao et al., SC'25; Alg.1, §4.1-4.2) on B200: every
step runs in the sm_100a kernels of ``csrc/`` behind the C ABI; this module only marshals
arguments (torch tensors -> device pointers, the current CUDA stream, host structs). PyTorch is
used for device memory, pinned host memory, streams and process groups — nothing else.

There is NO CPU fallback: if the shared library is missing or no CUDA device is present, every
call raises. (The CPU oracle in ``oracle/`` is test infrastructure and is never imported here.)

Names follow the ABI: compress, coalesce, allgather_sparse (via Comm), batch_merge,
record_bytes, stage_d2h, replay.
"""
from __future__ import annotations

import ctypes as C
import os

import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
SO_PATH = os.environ.get("LOWDIFF_SO") or os.path.join(_HERE, "liblowdiff.so")   # (override: variant experiments)

F32, BF16 = 0, 1
SUM, STACK = 0, 1
SGD, MOMENTUM, ADAM = 0, 1, 2
_DT = {"f32": F32, "bf16": BF16, F32: F32, BF16: BF16}
_MODE = {"sum": SUM, "stack": STACK, SUM: SUM, STACK: STACK}
_KIND = {"sgd": SGD, "momentum": MOMENTUM, "adam": ADAM}
STATUS = {0: "OK", 1: "EINVAL", 2: "EWORKSPACE", 3: "ECAPACITY", 4: "ECHAIN", 5: "ECORRUPT",
          6: "EUNSUPPORTED", 7: "ECUDA", 8: "ENCCL", 9: "ETIMEOUT"}


class LowDiffError(RuntimeError):
    def __init__(self, code: int, what: str, detail: str):
        super().__init__(f"{what}: {STATUS.get(code, code)} ({detail})")
        self.code = code
        self.status = STATUS.get(code, str(code))


class DiffView(C.Structure):
    _fields_ = [("idx", C.c_void_p), ("val", C.c_void_p), ("d_nnz", C.c_void_p), ("cap", C.c_uint64),
                ("lr", C.c_float)]


class RecordHeader(C.Structure):
    _fields_ = [("magic", C.c_uint8 * 8), ("version", C.c_uint32), ("mode", C.c_uint32),
                ("B", C.c_uint32), ("nranks", C.c_uint32), ("n", C.c_uint64), ("lo", C.c_uint64),
                ("hi", C.c_uint64), ("t_first", C.c_uint64), ("nnz", C.c_uint64), ("nent", C.c_uint64),
                ("total_bytes", C.c_uint64)]


class Opt(C.Structure):
    _fields_ = [("kind", C.c_int32), ("momentum", C.c_double), ("dampening", C.c_double),
                ("weight_decay", C.c_double), ("beta1", C.c_double), ("beta2", C.c_double),
                ("eps", C.c_double), ("nesterov", C.c_int32), ("allow_accumulated_sum", C.c_int32),
                ("approx_math", C.c_int32)]


class State(C.Structure):
    _fields_ = [("x", C.c_void_p), ("m", C.c_void_p), ("v", C.c_void_p), ("x_bf16", C.c_void_p),
                ("n", C.c_uint64), ("lo", C.c_uint64), ("hi", C.c_uint64), ("t", C.c_uint64),
                ("adam_step", C.c_uint64), ("momentum_initialized", C.c_int32),
                ("x0", C.c_void_p), ("m0", C.c_void_p), ("v0", C.c_void_p)]


class Plan(C.Structure):
    """lowdiff_plan: the problem statement (n, rho -> k, B, FCF, dtypes, rank -> shard)."""
    _fields_ = [("n", C.c_uint64), ("rho", C.c_double), ("k", C.c_uint64), ("B", C.c_uint32),
                ("full_every", C.c_uint32), ("gdt", C.c_int32), ("vdt", C.c_int32), ("nranks", C.c_int32),
                ("rank", C.c_int32), ("lo", C.c_uint64), ("hi", C.c_uint64)]


class RecordView(C.Structure):
    _fields_ = [("d_record", C.c_void_p), ("h_head", C.c_void_p), ("h_head_len", C.c_uint64)]


EXPORTS = [
    "lowdiff_status_string", "lowdiff_last_error", "lowdiff_version", "lowdiff_k_for_density",
    "lowdiff_pairs_bytes", "lowdiff_shard_bounds", "lowdiff_compress_workspace_size",
    "lowdiff_compress", "lowdiff_comm_unique_id_bytes", "lowdiff_comm_get_unique_id",
    "lowdiff_comm_init", "lowdiff_comm_destroy", "lowdiff_coalesce_workspace_size",
    "lowdiff_coalesce", "lowdiff_allgather_sparse_workspace_size", "lowdiff_allgather_sparse",
    "lowdiff_record_size", "lowdiff_record_max_bytes", "lowdiff_batch_merge_workspace_size",
    "lowdiff_batch_merge", "lowdiff_record_bytes", "lowdiff_stage_d2h", "lowdiff_record_parse",
    "lowdiff_replay_workspace_size", "lowdiff_replay", "lowdiff_launch_count",
    "lowdiff_profile_enable", "lowdiff_profile_query", "lowdiff_compress_stats",
    "lowdiff_debug_force_threshold", "lowdiff_debug_force_rescan_threshold", "lowdiff_compress_counters",
    "lowdiff_wasted_time", "lowdiff_optimal_config",
    "lowdiff_replay_parallel_workspace_size", "lowdiff_replay_parallel",
    "lowdiff_update_workspace_size", "lowdiff_update", "lowdiff_dense_update", "lowdiff_host_update",
    "lowdiff_p2p_window_bytes", "lowdiff_p2p_export_handle", "lowdiff_p2p_init", "lowdiff_p2p_init_local",
    "lowdiff_p2p_destroy", "lowdiff_p2p_slot", "lowdiff_p2p_allgather_sparse", "lowdiff_p2p_status",
    "lowdiff_batch_merge_ex", "lowdiff_plan_init", "lowdiff_plan_record_due", "lowdiff_replay_check",
    "lowdiff_record_max_bytes_shard",
]

_lib = None


def lib() -> C.CDLL:
    """Load liblowdiff.so (built in-tree by build.py). Raises if it is missing."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(SO_PATH):
        raise RuntimeError(f"liblowdiff.so not built ({SO_PATH}); run "
                           "`python -m paper_conf_sc_yaolhlzz25_b200.build` — there is no fallback")
    L = C.CDLL(SO_PATH)
    u64, i32, vp, f64 = C.c_uint64, C.c_int32, C.c_void_p, C.c_double
    sig = {
        "lowdiff_status_string": ([i32], C.c_char_p),
        "lowdiff_last_error": ([], C.c_char_p),
        "lowdiff_version": ([], C.c_char_p),
        "lowdiff_k_for_density": ([u64, f64], u64),
        "lowdiff_pairs_bytes": ([u64, i32], u64),
        "lowdiff_shard_bounds": ([u64, i32, i32, vp, vp], i32),
        "lowdiff_compress_workspace_size": ([u64, u64, vp], i32),
        "lowdiff_compress": ([vp, i32, vp, u64, u64, vp, i32, vp, u64, vp], i32),
        "lowdiff_comm_unique_id_bytes": ([], i32),
        "lowdiff_comm_get_unique_id": ([vp], i32),
        "lowdiff_comm_init": ([vp, vp, i32, i32], i32),
        "lowdiff_comm_destroy": ([vp], i32),
        "lowdiff_coalesce_workspace_size": ([i32, u64, i32, u64, u64, vp], i32),
        "lowdiff_coalesce": ([vp, i32, u64, i32, u64, u64, i32, vp, vp, u64, vp, vp, u64, vp], i32),
        "lowdiff_allgather_sparse_workspace_size": ([i32, u64, i32, u64, u64, vp], i32),
        "lowdiff_allgather_sparse": ([vp, vp, u64, i32, u64, u64, i32, vp, vp, u64, vp, vp, u64, vp], i32),
        "lowdiff_record_size": ([i32, C.c_uint32, u64, u64], u64),
        "lowdiff_record_max_bytes": ([i32, C.c_uint32, u64], u64),
        "lowdiff_batch_merge_workspace_size": ([C.c_uint32, u64, u64, u64, vp], i32),
        "lowdiff_batch_merge_ex": ([vp, C.c_uint32, i32, i32, u64, u64, u64, u64, C.c_uint32, vp, u64, vp, vp,
                                    u64, vp], i32),
        "lowdiff_batch_merge": ([vp, C.c_uint32, i32, u64, u64, u64, u64, C.c_uint32, vp, u64, vp, vp,
                                 u64, vp], i32),
        "lowdiff_record_bytes": ([vp, u64, vp, vp], i32),
        "lowdiff_stage_d2h": ([vp, u64, vp, u64, vp], i32),
        "lowdiff_record_parse": ([vp, u64, vp], i32),
        "lowdiff_replay_workspace_size": ([vp, vp, C.c_uint32, vp], i32),
        "lowdiff_replay": ([vp, vp, vp, C.c_uint32, vp, u64, vp], i32),
        "lowdiff_launch_count": ([], u64),
        "lowdiff_profile_enable": ([i32], i32),
        "lowdiff_profile_query": ([C.c_char_p, vp, vp], i32),
        "lowdiff_compress_stats": ([vp, u64, u64, vp, vp], i32),
        "lowdiff_debug_force_threshold": ([i32, C.c_uint32], i32),
        "lowdiff_debug_force_rescan_threshold": ([i32, C.c_uint32], i32),
        "lowdiff_compress_counters": ([vp, vp, vp], i32),
        "lowdiff_wasted_time": ([vp, f64, f64, vp], i32),
        "lowdiff_replay_parallel_workspace_size": ([vp, vp, C.c_uint32, vp], i32),
        "lowdiff_replay_parallel": ([vp, vp, vp, C.c_uint32, vp, u64, vp], i32),
        "lowdiff_optimal_config": ([vp, vp, vp, vp, vp], i32),
        "lowdiff_update_workspace_size": ([vp, vp], i32),
        "lowdiff_update": ([vp, vp, vp, vp, u64, vp], i32),
        "lowdiff_dense_update": ([vp, vp, vp, i32, C.c_float, vp], i32),
        "lowdiff_host_update": ([vp, vp, vp, i32, C.c_float, i32], i32),
        "lowdiff_p2p_window_bytes": ([i32, u64, i32], u64),
        "lowdiff_p2p_export_handle": ([vp, vp], i32),
        "lowdiff_p2p_init": ([vp, vp, vp, i32, i32, u64, i32], i32),
        "lowdiff_p2p_init_local": ([vp, vp, i32, i32, u64, i32], i32),
        "lowdiff_p2p_destroy": ([vp], i32),
        "lowdiff_p2p_slot": ([vp, vp], vp),
        "lowdiff_p2p_allgather_sparse": ([vp, vp, u64, u64, i32, vp, vp, u64, vp, vp, u64, vp], i32),
        "lowdiff_p2p_status": ([vp], i32),
        "lowdiff_plan_init": ([vp, u64, f64, C.c_uint32, C.c_uint32, i32, i32, i32, i32], i32),
        "lowdiff_plan_record_due": ([vp, u64, vp, vp, vp], i32),
        "lowdiff_replay_check": ([vp, vp], i32),
        "lowdiff_record_max_bytes_shard": ([i32, C.c_uint32, u64, u64, u64], u64),
    }
    for name, (args, res) in sig.items():
        f = getattr(L, name)
        f.argtypes, f.restype = args, res
    _lib = L
    return L


def _check(code: int, what: str):
    if code != 0:
        raise LowDiffError(code, what, lib().lowdiff_last_error().decode(errors="replace"))


def _cuda(t: torch.Tensor, name: str) -> int:
    if not t.is_cuda:
        raise ValueError(f"{name} must be a CUDA tensor (no CPU path exists)")
    if not t.is_contiguous():
        raise ValueError(f"{name} must be contiguous")
    return t.data_ptr()


def _stream(stream) -> int:
    s = stream if stream is not None else torch.cuda.current_stream()
    return s.cuda_stream if hasattr(s, "cuda_stream") else int(s)


# ---- workspaces (caller-owned device memory, cached per device and purpose) -------------------
_ws_cache: dict = {}


def workspace(nbytes: int, device, tag: str = "ws") -> torch.Tensor:
    d = torch.device(device)
    if d.type == "cuda" and d.index is None:
        d = torch.device("cuda", torch.cuda.current_device())
    key = (str(d), tag)
    buf = _ws_cache.get(key)
    if buf is None or buf.numel() < nbytes:
        # zeroed once (the compress threshold state reads a fresh workspace as cold either way;
        # zeroing keeps compute-sanitizer initcheck quiet about that intended read)
        buf = torch.zeros(max(nbytes, 256), dtype=torch.uint8, device=device)
        _ws_cache[key] = buf
    return buf


def release_workspaces():
    _ws_cache.clear()


# ---- sizes ----------------------------------------------------------------------------------------
def k_for_density(n: int, rho: float) -> int:
    return int(lib().lowdiff_k_for_density(n, rho))


def pairs_bytes(k: int, vdt="f32") -> int:
    return int(lib().lowdiff_pairs_bytes(k, _DT[vdt]))


def shard_bounds(n: int, nranks: int, rank: int) -> tuple[int, int]:
    lo, hi = C.c_uint64(), C.c_uint64()
    _check(lib().lowdiff_shard_bounds(n, nranks, rank, C.byref(lo), C.byref(hi)), "shard_bounds")
    return lo.value, hi.value


def plan_init(n: int, rho: float, B: int, full_every: int, gdt="f32", vdt="f32", nranks: int = 1,
              rank: int = 0) -> Plan:
    """lowdiff_plan_init: k, the rank's shard [lo, hi) and the batching / full-checkpoint policy."""
    p = Plan()
    _check(lib().lowdiff_plan_init(C.byref(p), n, float(rho), B, full_every, _DT[gdt], _DT[vdt], nranks, rank),
           "plan_init")
    return p


def plan_record_due(plan: Plan, t: int) -> tuple[bool, int, bool]:
    """lowdiff_plan_record_due for iteration t: (close the open record after t, its length so far
    including t, a full checkpoint is due before t) — DESIGN.md reading #25."""
    close, blen, full = C.c_int32(), C.c_uint32(), C.c_int32()
    _check(lib().lowdiff_plan_record_due(C.byref(plan), t, C.byref(close), C.byref(blen), C.byref(full)),
           "plan_record_due")
    return bool(close.value), int(blen.value), bool(full.value)


class ConfigModel(C.Structure):
    """lowdiff_config_model (§3.5): time in units of one training iteration."""
    _fields_ = [(k, C.c_double) for k in ("N", "M", "W", "S", "T", "R_F", "R_D")]


def _model(m: dict) -> ConfigModel:
    return ConfigModel(*(float(m[k]) for k in ("N", "M", "W", "S", "T", "R_F", "R_D")))


def wasted_time(model: dict, f: float, b: float) -> float:
    """Eq. 3 for full-checkpoint frequency f and batching size b."""
    out = C.c_double()
    cm = _model(model)
    _check(lib().lowdiff_wasted_time(C.byref(cm), float(f), float(b), C.byref(out)), "wasted_time")
    return out.value


def optimal_config(model: dict) -> dict:
    """Eq. 5 and the best integer (FCF, B) around it: {"f_star", "b_star", "fcf", "B"}."""
    fs, bs = C.c_double(), C.c_double()
    fcf, b = C.c_uint32(), C.c_uint32()
    cm = _model(model)
    _check(lib().lowdiff_optimal_config(C.byref(cm), C.byref(fs), C.byref(bs), C.byref(fcf), C.byref(b)),
           "optimal_config")
    return {"f_star": fs.value, "b_star": bs.value, "fcf": fcf.value, "B": b.value}


def record_size(mode, B: int, nnz: int, nent: int) -> int:
    return int(lib().lowdiff_record_size(_MODE[mode], B, nnz, nent))


def record_max_bytes(mode, B: int, max_entries: int, lo: int | None = None, hi: int | None = None) -> int:
    """Upper bound of a record's bytes; with the shard [lo, hi) its unique indices are bounded too."""
    if lo is not None and hi is not None:
        return int(lib().lowdiff_record_max_bytes_shard(_MODE[mode], B, max_entries, lo, hi))
    return int(lib().lowdiff_record_max_bytes(_MODE[mode], B, max_entries))


def pairs_views(pairs: torch.Tensor, k: int, vdt="f32"):
    """(idx int32[k], val float32|bfloat16[k]) views into a packed pairs buffer."""
    off = ((4 * k + 15) // 16) * 16
    idx = pairs[:4 * k].view(torch.int32)
    esz = 2 if _DT[vdt] == BF16 else 4
    val = pairs[off:off + esz * k].view(torch.bfloat16 if esz == 2 else torch.float32)
    return idx, val


# ---- (1) compress ---------------------------------------------------------------------------------
def compress_workspace_size(n: int, k: int) -> int:
    b = C.c_uint64()
    _check(lib().lowdiff_compress_workspace_size(n, k, C.byref(b)), "compress_workspace_size")
    return b.value


def compress(grad: torch.Tensor, residual: torch.Tensor, k: int, vdt="f32", pairs=None, ws=None,
             stream=None) -> torch.Tensor:
    """Comp(G_{i,t}) (Alg.1 line 4): exact top-k of |grad + residual| with error feedback.
    residual is updated in place; returns the packed pairs buffer (uint8)."""
    n = grad.numel()
    if grad.dtype not in (torch.float32, torch.bfloat16) or residual.dtype != torch.float32:
        raise ValueError("grad must be fp32/bf16 and residual fp32")
    if residual.numel() != n:
        raise ValueError("residual size mismatch")
    gdt = BF16 if grad.dtype == torch.bfloat16 else F32
    nb = pairs_bytes(k, vdt)
    if pairs is None:
        pairs = torch.empty(nb, dtype=torch.uint8, device=grad.device)
    assert pairs.numel() >= nb
    wsb = compress_workspace_size(n, k)
    if ws is None:
        ws = workspace(wsb, grad.device, "compress")
    _check(lib().lowdiff_compress(_cuda(grad, "grad"), gdt, _cuda(residual, "residual"), n, k,
                                  _cuda(pairs, "pairs"), _DT[vdt], _cuda(ws, "ws"), ws.numel(),
                                  _stream(stream)), "compress")
    return pairs


# ---- (2) coalesce / sparse all-gather ------------------------------------------------------------
def coalesce_workspace_size(nranks: int, k: int, vdt, lo: int, hi: int) -> int:
    b = C.c_uint64()
    _check(lib().lowdiff_coalesce_workspace_size(nranks, k, _DT[vdt], lo, hi, C.byref(b)),
           "coalesce_workspace_size")
    return b.value


def _coalesce_outputs(device, P, k, lo, hi, out_idx, out_val, d_nnz):
    cap = min(P * k, hi - lo)
    if out_idx is None:
        out_idx = torch.empty(max(cap, 1), dtype=torch.int32, device=device)
    if out_val is None:
        out_val = torch.empty(max(cap, 1), dtype=torch.float32, device=device)
    if d_nnz is None:
        d_nnz = torch.zeros(1, dtype=torch.int64, device=device)
    assert out_idx.numel() >= cap and out_val.numel() >= cap
    return out_idx, out_val, d_nnz


def coalesce(gathered: torch.Tensor, nranks: int, k: int, vdt="f32", lo: int = 0, hi: int | None = None,
             average: bool = True, out_idx=None, out_val=None, d_nnz=None, ws=None, stream=None, n=None):
    """Coalesce P packed pair buffers already on this device (the post-gather half of Sync)."""
    assert hi is not None
    out_idx, out_val, d_nnz = _coalesce_outputs(gathered.device, nranks, k, lo, hi, out_idx, out_val, d_nnz)
    wsb = coalesce_workspace_size(nranks, k, vdt, lo, hi)
    if ws is None:
        ws = workspace(wsb, gathered.device, "coalesce")
    _check(lib().lowdiff_coalesce(_cuda(gathered, "gathered"), nranks, k, _DT[vdt], lo, hi, int(average),
                                  _cuda(out_idx, "out_idx"), _cuda(out_val, "out_val"), out_idx.numel(),
                                  _cuda(d_nnz, "d_nnz"), _cuda(ws, "ws"), ws.numel(), _stream(stream)),
           "coalesce")
    return out_idx, out_val, d_nnz


def broadcast_bytes(data: bytes | None, nbytes: int, group=None) -> bytes:
    """Rank 0's `data` (nbytes long) on every rank of the torch.distributed group (host plumbing for
    the NCCL unique id; works on the nccl and gloo backends)."""
    import torch.distributed as dist
    t = torch.zeros(nbytes, dtype=torch.uint8)
    if data is not None:
        t.copy_(torch.frombuffer(bytearray(data), dtype=torch.uint8))
    if dist.is_initialized() and dist.get_world_size(group) > 1:
        dev = "cuda" if dist.get_backend(group) == "nccl" else "cpu"
        td = t.to(dev)
        dist.broadcast(td, src=0, group=group)
        t = td.cpu()
    return bytes(t.tolist())


class Comm:
    """NCCL communicator of liblowdiff, bootstrapped through torch.distributed (the unique id is
    broadcast from rank 0 over the default process group)."""

    def __init__(self, nranks: int, rank: int, group=None):
        self.nranks, self.rank = nranks, rank
        nid = int(lib().lowdiff_comm_unique_id_bytes())
        data = None
        if rank == 0:
            buf = (C.c_uint8 * nid)()
            _check(lib().lowdiff_comm_get_unique_id(buf), "comm_get_unique_id")
            data = bytes(buf)
        raw = (C.c_uint8 * nid)(*broadcast_bytes(data, nid, group))
        self._h = C.c_void_p()
        _check(lib().lowdiff_comm_init(C.byref(self._h), raw, nranks, rank), "comm_init")

    @property
    def handle(self):
        return self._h

    def destroy(self):
        if self._h:
            _check(lib().lowdiff_comm_destroy(self._h), "comm_destroy")
            self._h = C.c_void_p()


def allgather_sparse_workspace_size(nranks: int, k: int, vdt, lo: int, hi: int) -> int:
    b = C.c_uint64()
    _check(lib().lowdiff_allgather_sparse_workspace_size(nranks, k, _DT[vdt], lo, hi, C.byref(b)),
           "allgather_sparse_workspace_size")
    return b.value


def allgather_sparse(comm: Comm | None, pairs: torch.Tensor, k: int, vdt="f32", lo: int = 0,
                     hi: int | None = None, average: bool = True, out_idx=None, out_val=None,
                     d_nnz=None, ws=None, stream=None):
    """Sync(G~_{i,t}) (Alg.1 line 5): NCCL all-gather of every rank's pairs + coalesce of [lo, hi)."""
    P = comm.nranks if comm is not None else 1
    out_idx, out_val, d_nnz = _coalesce_outputs(pairs.device, P, k, lo, hi, out_idx, out_val, d_nnz)
    wsb = allgather_sparse_workspace_size(P, k, vdt, lo, hi)
    if ws is None:
        ws = workspace(wsb, pairs.device, "allgather")
    _check(lib().lowdiff_allgather_sparse(comm.handle if comm is not None else None,
                                          _cuda(pairs, "pairs"), k, _DT[vdt], lo, hi, int(average),
                                          _cuda(out_idx, "out_idx"), _cuda(out_val, "out_val"),
                                          out_idx.numel(), _cuda(d_nnz, "d_nnz"), _cuda(ws, "ws"),
                                          ws.numel(), _stream(stream)), "allgather_sparse")
    return out_idx, out_val, d_nnz


# ---- (2') all-gather fused with coalesce over peer memory (NVLink P2P, CUDA IPC) -------------------
P2P_HANDLE_BYTES = 80


def p2p_window_bytes(nranks: int, k: int, vdt="f32") -> int:
    return int(lib().lowdiff_p2p_window_bytes(nranks, k, _DT[vdt]))


class P2P:
    """lowdiff_p2p_*: Sync(G~_{i,t}) (Alg.1 line 5) with the coalesce reading every rank's
    pairs straight out of its owner's exchange window over NVLink (no all-gather copy).

    Multi-process: P2P(nranks, rank, k, vdt, group=...) allocates this rank's window, exchanges the
    CUDA IPC handles with torch.distributed.all_gather_object (any backend) and barriers.
    Single process: P2P.local(nranks, k, vdt, device) returns one handle per simulated rank, all
    windows on one device (each rank must then be driven on its own stream)."""

    def __init__(self, nranks: int, rank: int, k: int, vdt="f32", device=None, group=None, _windows=None):
        self.nranks, self.rank, self.k, self.vdt = nranks, rank, k, vdt
        nb = p2p_window_bytes(nranks, k, vdt)
        self._h = C.c_void_p()
        if _windows is not None:                    # single-process: every window given
            self.window = _windows[rank]
            ptrs = (C.c_void_p * nranks)(*[w.data_ptr() for w in _windows])
            _check(lib().lowdiff_p2p_init_local(C.byref(self._h), ptrs, nranks, rank, k, _DT[vdt]),
                   "p2p_init_local")
            return
        import torch.distributed as dist
        device = torch.device(device if device is not None else "cuda")
        self.window = _aligned_window(nb, device)
        h = (C.c_uint8 * P2P_HANDLE_BYTES)()
        _check(lib().lowdiff_p2p_export_handle(C.c_void_p(self.window.data_ptr()), h), "p2p_export_handle")
        allh = [None] * nranks
        dist.all_gather_object(allh, bytes(h), group=group)
        raw = (C.c_uint8 * (P2P_HANDLE_BYTES * nranks))(*b"".join(allh))
        _check(lib().lowdiff_p2p_init(C.byref(self._h), C.c_void_p(self.window.data_ptr()), raw, nranks, rank,
                                      k, _DT[vdt]), "p2p_init")
        dist.barrier(group=group)

    @classmethod
    def local(cls, nranks: int, k: int, vdt="f32", device="cuda"):
        nb = p2p_window_bytes(nranks, k, vdt)
        wins = [_aligned_window(nb, torch.device(device)) for _ in range(nranks)]
        return [cls(nranks, r, k, vdt, _windows=wins) for r in range(nranks)]

    def slot(self, stream=None) -> torch.Tensor:
        """The local slot the next allgather_sparse publishes (after enqueuing, on `stream`, the wait
        that makes it writable): compress into it to skip the copy."""
        p = lib().lowdiff_p2p_slot(self._h, _stream(stream))
        if not p:
            _check(7, "p2p_slot")
        off = p - self.window.data_ptr()
        return self.window[off:off + pairs_bytes(self.k, self.vdt)]

    def allgather_sparse(self, pairs: torch.Tensor, lo: int, hi: int, average: bool = True, out_idx=None,
                         out_val=None, d_nnz=None, ws=None, stream=None):
        out_idx, out_val, d_nnz = _coalesce_outputs(pairs.device, self.nranks, self.k, lo, hi, out_idx, out_val,
                                                     d_nnz)
        wsb = coalesce_workspace_size(self.nranks, self.k, self.vdt, lo, hi)
        if ws is None:
            ws = workspace(wsb, pairs.device, f"p2p{self.rank}")
        _check(lib().lowdiff_p2p_allgather_sparse(self._h, _cuda(pairs, "pairs"), lo, hi, int(average),
                                                  _cuda(out_idx, "out_idx"), _cuda(out_val, "out_val"),
                                                  out_idx.numel(), _cuda(d_nnz, "d_nnz"), _cuda(ws, "ws"),
                                                  ws.numel(), _stream(stream)), "p2p_allgather_sparse")
        return out_idx, out_val, d_nnz

    def status(self):
        """Raises LowDiffError(ETIMEOUT) once any peer wait of this handle expired (no sync)."""
        _check(lib().lowdiff_p2p_status(self._h), "p2p_status")

    def destroy(self):
        if self._h:
            _check(lib().lowdiff_p2p_destroy(self._h), "p2p_destroy")
            self._h = C.c_void_p()


def _aligned_window(nbytes: int, device) -> torch.Tensor:
    buf = torch.empty(nbytes + 256, dtype=torch.uint8, device=device)
    off = (-buf.data_ptr()) % 256
    return buf[off:off + nbytes]


# ---- (3) batch merge --------------------------------------------------------------------------------
def batch_merge_workspace_size(B: int, max_entries: int, lo: int, hi: int) -> int:
    b = C.c_uint64()
    _check(lib().lowdiff_batch_merge_workspace_size(B, max_entries, lo, hi, C.byref(b)),
           "batch_merge_workspace_size")
    return b.value


def batch_merge(diffs, mode, n: int, lo: int, hi: int, t_first: int, nranks: int, record=None,
                d_record_bytes=None, ws=None, stream=None):
    """Merge B differentials [(idx int32, val fp32, d_nnz int64[1], cap, lr), ...] (iteration order)
    into one record (§4.2 Step 2). Returns (record uint8 tensor, d_record_bytes int64[1]).
    bf16 `val` tensors (a P = 1 ring of compressed pairs buffers) go through lowdiff_batch_merge_ex."""
    B = len(diffs)
    views = (DiffView * B)()
    dev = diffs[0][0].device
    max_entries = 0
    for j, (idx, val, d_nnz, cap, lr) in enumerate(diffs):
        views[j] = DiffView(_cuda(idx, "idx"), _cuda(val, "val"), _cuda(d_nnz, "d_nnz"), int(cap), float(lr))
        max_entries += int(cap)
    max_entries = max(max_entries, 1)
    cap_bytes = record_max_bytes(mode, B, max_entries)
    if record is None:
        record = torch.empty(cap_bytes, dtype=torch.uint8, device=dev)
    if d_record_bytes is None:
        d_record_bytes = torch.zeros(1, dtype=torch.int64, device=dev)
    wsb = batch_merge_workspace_size(B, max_entries, lo, hi)
    if ws is None:
        ws = workspace(wsb, dev, "merge")
    vdts = {d[1].dtype for d in diffs}
    if vdts not in ({torch.float32}, {torch.bfloat16}):
        raise ValueError("diff values must all be float32 or all bfloat16")
    vdt = BF16 if vdts == {torch.bfloat16} else F32
    _check(lib().lowdiff_batch_merge_ex(views, B, _MODE[mode], vdt, n, lo, hi, t_first, nranks,
                                        _cuda(record, "record"), record.numel(),
                                        _cuda(d_record_bytes, "d_record_bytes"), _cuda(ws, "ws"), ws.numel(),
                                        _stream(stream)), "batch_merge")
    return record, d_record_bytes


# ---- (4) stage -----------------------------------------------------------------------------------------
def record_bytes(d_record_bytes: torch.Tensor, record_cap: int, stream=None) -> int:
    out = C.c_uint64()
    _check(lib().lowdiff_record_bytes(_cuda(d_record_bytes, "d_record_bytes"), record_cap, _stream(stream),
                                      C.byref(out)), "record_bytes")
    return out.value


def stage_d2h(record: torch.Tensor, nbytes: int, pinned: torch.Tensor, copy_stream=None):
    """Async D2H of the record into caller-owned pinned host memory (Step 1)."""
    if not pinned.is_pinned():
        raise ValueError("stage target must be pinned host memory")
    _check(lib().lowdiff_stage_d2h(_cuda(record, "record"), nbytes, pinned.data_ptr(), pinned.numel(),
                                   _stream(copy_stream)), "stage_d2h")


def record_parse(h_bytes) -> dict:
    """Header of a host record (numpy array, bytes, or CPU tensor)."""
    import numpy as np
    if isinstance(h_bytes, torch.Tensor):
        arr = h_bytes.numpy()
    else:
        arr = np.frombuffer(bytes(h_bytes), dtype=np.uint8) if not isinstance(h_bytes, np.ndarray) else h_bytes
    arr = np.ascontiguousarray(arr, dtype=np.uint8)
    h = RecordHeader()
    _check(lib().lowdiff_record_parse(arr.ctypes.data, arr.size, C.byref(h)), "record_parse")
    return {f: getattr(h, f) for f, _ in RecordHeader._fields_ if f != "magic"}


# ---- (5) replay ----------------------------------------------------------------------------------------
def _replay_args(state: dict, opt: dict, records):
    import numpy as np
    o = Opt(_KIND[opt["kind"]], opt.get("momentum", 0.0), opt.get("dampening", 0.0),
            opt.get("weight_decay", 0.0), opt.get("beta1", 0.9), opt.get("beta2", 0.999),
            opt.get("eps", 1e-8), int(opt.get("nesterov", 0)), int(opt.get("allow_accumulated_sum", 0)),
            int(opt.get("approx_math", 0)))
    ptr = lambda key: _cuda(state[key], key) if state.get(key) is not None else None
    st = State(ptr("x"), ptr("m"), ptr("v"), ptr("x_bf16"), state["n"], state["lo"], state["hi"],
               state["t"], state["adam_step"], state["momentum_initialized"],
               ptr("x0"), ptr("m0"), ptr("v0"))
    R = len(records)
    views = (RecordView * max(R, 1))()
    keep = []
    for q, (drec, head) in enumerate(records):
        if isinstance(head, torch.Tensor):
            h = head if head.device.type == "cpu" else head.cpu()
            hp, hl = h.data_ptr(), h.numel()
            keep.append(h)
        else:
            a = np.ascontiguousarray(np.frombuffer(bytes(head), np.uint8) if not isinstance(head, np.ndarray)
                                     else head, dtype=np.uint8)
            keep.append(a)
            hp, hl = a.ctypes.data, a.size
        views[q] = RecordView(_cuda(drec, "d_record"), hp, hl)
    return o, st, views, R, keep


def replay(state: dict, opt: dict, records, ws=None, stream=None, check: bool = True) -> dict:
    """Recovery (Alg.1 lines 16-24): replay records [(d_record uint8 CUDA tensor, h_head host bytes)]
    onto the state {x, m, v (fp32 CUDA), x_bf16 (optional), n, lo, hi, t, adam_step,
    momentum_initialized}; device arrays are updated in place, counters in the dict.
    check: synchronize and raise ECORRUPT if a record body failed the device validation (the state
    is then untouched); False leaves that to a later replay_check(ws)."""
    o, st, views, R, keep = _replay_args(state, opt, records)
    b = C.c_uint64()
    _check(lib().lowdiff_replay_workspace_size(C.byref(st), views, R, C.byref(b)), "replay_workspace_size")
    if ws is None:
        ws = workspace(b.value, state["x"].device, "replay")
    _check(lib().lowdiff_replay(C.byref(st), C.byref(o), views, R, _cuda(ws, "ws"), ws.numel(),
                                _stream(stream)), "replay")
    state["t"], state["adam_step"] = st.t, st.adam_step
    state["momentum_initialized"] = st.momentum_initialized
    if check and R:
        replay_check(ws, stream)
    return state


def replay_check(ws=None, stream=None):
    """lowdiff_replay_check: ECORRUPT if the last replay with this workspace rejected a record body."""
    if ws is None:
        ws = _ws_cache.get((f"cuda:{torch.cuda.current_device()}", "replay"))
        if ws is None:
            return
    _check(lib().lowdiff_replay_check(_cuda(ws, "ws"), _stream(stream)), "replay_check")


def update(state: dict, opt: dict, g_t, ws=None, stream=None) -> dict:
    """Live update (Alg.1 training process): apply this iteration's synchronized G~_t =
    (idx int32, val fp32, d_nnz int64[1], cap, lr) — as allgather_sparse/coalesce return it — to the
    state as one dense optimizer step, in place, without a host synchronization. Bit-identical to
    replay() of a one-iteration record of G~_t."""
    o, st, _, _, _ = _replay_args(state, opt, [])
    idx, val, d_nnz, cap, lr = g_t
    view = DiffView(_cuda(idx, "idx"), _cuda(val, "val"), _cuda(d_nnz, "d_nnz"), int(cap), float(lr))
    b = C.c_uint64()
    _check(lib().lowdiff_update_workspace_size(C.byref(st), C.byref(b)), "update_workspace_size")
    if ws is None:
        ws = workspace(b.value, state["x"].device, "update")
    _check(lib().lowdiff_update(C.byref(st), C.byref(o), C.byref(view), _cuda(ws, "ws"), ws.numel(),
                                _stream(stream)), "update")
    state["t"], state["adam_step"] = st.t, st.adam_step
    state["momentum_initialized"] = st.momentum_initialized
    return state


def _dense_args(state: dict, opt: dict, grad: torch.Tensor, device: bool):
    o = Opt(_KIND[opt["kind"]], opt.get("momentum", 0.0), opt.get("dampening", 0.0),
            opt.get("weight_decay", 0.0), opt.get("beta1", 0.9), opt.get("beta2", 0.999),
            opt.get("eps", 1e-8), int(opt.get("nesterov", 0)), 0)
    if grad.dtype not in (torch.float32, torch.bfloat16) or not grad.is_contiguous():
        raise ValueError("grad must be a contiguous fp32/bf16 tensor")
    L = state["hi"] - state["lo"]
    for key in ("x", "m", "v"):
        t = state.get(key)
        if t is not None and (t.is_cuda != device or t.dtype != torch.float32 or t.numel() != L
                              or not t.is_contiguous()):
            raise ValueError(f"state[{key!r}] must be a contiguous fp32 {'CUDA' if device else 'CPU'} tensor of {L}")
    if grad.is_cuda != device or grad.numel() != L:
        raise ValueError(f"grad must be a {'CUDA' if device else 'CPU'} tensor of {L} values")
    ptr = lambda key: state[key].data_ptr() if state.get(key) is not None else None
    st = State(ptr("x"), ptr("m"), ptr("v"), None, state["n"], state["lo"], state["hi"], state["t"],
               state["adam_step"], state["momentum_initialized"], None, None, None)
    return o, st, BF16 if grad.dtype == torch.bfloat16 else F32


def dense_update(state: dict, opt: dict, grad: torch.Tensor, lr: float, stream=None) -> dict:
    """LowDiff+ GPU model update (Alg. 2 line 7): one dense optimizer step of the shard state from
    the dense gradient (CUDA fp32/bf16), in place, asynchronous on the stream."""
    o, st, gdt = _dense_args(state, opt, grad, True)
    _check(lib().lowdiff_dense_update(C.byref(st), C.byref(o), grad.data_ptr(), gdt, float(lr), _stream(stream)),
           "dense_update")
    state["t"], state["adam_step"] = st.t, st.adam_step
    state["momentum_initialized"] = st.momentum_initialized
    return state


def host_update(state: dict, opt: dict, grad: torch.Tensor, lr: float, threads: int = 0) -> dict:
    """LowDiff+ CPU replica update (Alg. 2 line 12): the same step on host tensors, `threads`
    workers (0 = all cores). Blocks the calling thread (ctypes releases the GIL meanwhile)."""
    o, st, gdt = _dense_args(state, opt, grad, False)
    threads = threads or os.cpu_count() or 1
    _check(lib().lowdiff_host_update(C.byref(st), C.byref(o), grad.data_ptr(), gdt, float(lr), int(threads)),
           "host_update")
    state["t"], state["adam_step"] = st.t, st.adam_step
    state["momentum_initialized"] = st.momentum_initialized
    return state


def replay_parallel(state: dict, opt: dict, records, ws=None, stream=None) -> dict:
    """Parallel recovery (Eq. 2): merge the chain's SUM differentials once, apply them to the
    checkpoint once (plain SGD, constant lr). Same arguments as replay()."""
    o, st, views, R, keep = _replay_args(state, opt, records)
    b = C.c_uint64()
    _check(lib().lowdiff_replay_parallel_workspace_size(C.byref(st), views, R, C.byref(b)),
           "replay_parallel_workspace_size")
    if ws is None:
        ws = workspace(b.value, state["x"].device, "replay_parallel")
    _check(lib().lowdiff_replay_parallel(C.byref(st), C.byref(o), views, R, _cuda(ws, "ws"), ws.numel(),
                                         _stream(stream)), "replay_parallel")
    state["t"] = st.t
    return state


# ---- instrumentation --------------------------------------------------------------------------------
def compress_stats(n: int, k: int, device="cuda", stream=None, ws=None) -> dict:
    """Diagnostics of the last compress that used `ws` (default: the cached workspace; syncs).
    path: 3 = first-pass candidates with the fast select, 0 = first-pass candidates with the general
    select, 2 = rescan recovery, 1 = exact full-array select."""
    if ws is None:
        ws = workspace(compress_workspace_size(n, k), device, "compress")
    out = (C.c_uint64 * 10)()
    _check(lib().lowdiff_compress_stats(_cuda(ws, "ws"), n, k, _stream(stream), out), "compress_stats")
    d = dict(zip(("t_est", "candidates", "path", "kstar", "ties_kept", "capacity", "fine_shift", "inbin",
                  "t2", "candidates2"), list(out)))
    d["fallback"] = int(d["path"] == 1)
    d["rescan"] = int(d["path"] == 2)
    d["first_pass"] = int(d["path"] in (0, 3))
    return d


def compress_counters(n: int = 0, k: int = 0, device="cuda", stream=None, ws=None) -> dict:
    """The persistent threshold state of a compress workspace (syncs): calls, rescans, full-array
    fallbacks, non-finite calls/count, last candidates, last k-th key, margin."""
    if ws is None:
        ws = workspace(compress_workspace_size(n, k), device, "compress")
    out = (C.c_uint64 * 9)()
    _check(lib().lowdiff_compress_counters(_cuda(ws, "ws"), _stream(stream), out), "compress_counters")
    v = list(out)
    return {"calls": v[0], "rescans": v[1], "fallbacks": v[2], "nonfinite_calls": v[3],
            "last_nonfinite": v[4], "last_candidates": v[5], "kstar": v[6], "delta": v[7] / 2.0 ** 32,
            "fast_calls": v[8]}


def debug_force_threshold(key: int | None):
    """Test hook: force the compress first-pass candidate threshold (None restores the default)."""
    _check(lib().lowdiff_debug_force_threshold(0 if key is None else 1, 0 if key is None else key),
           "debug_force_threshold")


def debug_force_rescan_threshold(key: int | None):
    """Test hook: force the threshold of the compress rescan recovery (None restores the default)."""
    _check(lib().lowdiff_debug_force_rescan_threshold(0 if key is None else 1, 0 if key is None else key),
           "debug_force_rescan_threshold")


def launch_count() -> int:
    return int(lib().lowdiff_launch_count())


def profile_enable(on: bool = True):
    _check(lib().lowdiff_profile_enable(int(on)), "profile_enable")


def profile_query(name: str) -> tuple[float, int]:
    ms, cnt = C.c_double(), C.c_uint64()
    _check(lib().lowdiff_profile_query(name.encode(), C.byref(ms), C.byref(cnt)), "profile_query")
    return ms.value, cnt.value
