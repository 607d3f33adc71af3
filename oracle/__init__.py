"""LowDiff CPU oracle — TEST INFRASTRUCTURE ONLY.

A ctypes view of ``lowdiff_oracle.cpp``: the plain, slow, single-threaded CPU
implementation of what the hot path computes, written from the paper
(/root/reference/PAPER.md, cited P:line) and the readings listed in DESIGN.md.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` leg may import this package. The product path
(``paper_conf_sc_yaolhlzz25_b200``) never imports it, and the two share no code: only
the seeded input generators in ``workloads/`` serve both.

Functions (numpy in, numpy out) and the passage each follows:
  compress      O1  Comp(G_{i,t}), Alg.1 line 4; top-k + EF per BASELINE north_star
  pairs_pack        the packed (idx | val) wire layout of one rank's G~_{i,t}
  coalesce      O2  Sync, Alg.1 line 5, P:213
  batch_merge   O3+O4  batched C^B_t, §4.2 Step 2; serialized record bytes
  record_size       record byte-size formula (DESIGN.md §Record layout)
  replay        O5  Recovery, Alg.1 lines 16-24; Adam Eq.1
  config_model  O6  (module oracle.config_model, plain fp64 Python) Eq. 3 / Eq. 5 of §3.5
                    (P:318-350): wasted time, (f*, b*), the best integer (FCF, B)

Parity pins for every function are in tests/test_oracle_*.py (none is "parity unpinned").
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "lowdiff_oracle.cpp")
_SO = os.path.join(_HERE, "liblowdiff_oracle.so")

F32, BF16 = 0, 1
SUM, STACK = 0, 1
SGD, MOMENTUM, ADAM = 0, 1, 2
OK, EINVAL, ECAPACITY, ECHAIN, ECORRUPT, EUNSUPPORTED = 0, 1, 3, 4, 5, 6


def build(force: bool = False) -> str:
    """Compile the oracle with g++ (-O2 -ffp-contract=off, no fast-math). Returns the .so path."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        tmp = _SO + f".tmp{os.getpid()}"
        subprocess.check_call(["g++", "-O2", "-ffp-contract=off", "-fno-fast-math", "-std=c++17",
                               "-shared", "-fPIC", "-o", tmp, _SRC])
        os.replace(tmp, _SO)
    return _SO


class _Opt(C.Structure):
    _fields_ = [("kind", C.c_int), ("momentum", C.c_double), ("dampening", C.c_double),
                ("weight_decay", C.c_double), ("beta1", C.c_double), ("beta2", C.c_double),
                ("eps", C.c_double), ("nesterov", C.c_int), ("allow_accumulated_sum", C.c_int)]


class _State(C.Structure):
    _fields_ = [("x", C.c_void_p), ("m", C.c_void_p), ("v", C.c_void_p), ("x_bf16", C.c_void_p),
                ("n", C.c_uint64), ("lo", C.c_uint64), ("hi", C.c_uint64), ("t", C.c_uint64),
                ("adam_step", C.c_uint64), ("momentum_initialized", C.c_int)]


_lib = None


def lib():
    global _lib
    if _lib is None:
        L = C.CDLL(build())
        u64, vp, i32 = C.c_uint64, C.c_void_p, C.c_int
        L.oracle_bf16_rne.argtypes = [C.c_float]; L.oracle_bf16_rne.restype = C.c_uint16
        L.oracle_pairs_bytes.argtypes = [u64, i32]; L.oracle_pairs_bytes.restype = u64
        L.oracle_pairs_pack.argtypes = [vp, vp, u64, i32, vp]; L.oracle_pairs_pack.restype = i32
        L.oracle_compress.argtypes = [vp, i32, vp, u64, u64, i32, vp, vp]
        L.oracle_compress.restype = i32
        L.oracle_coalesce.argtypes = [i32, vp, u64, i32, u64, u64, i32, vp, vp, u64, vp]
        L.oracle_coalesce.restype = i32
        L.oracle_record_size.argtypes = [i32, C.c_uint32, u64, u64]; L.oracle_record_size.restype = u64
        L.oracle_batch_merge.argtypes = [C.c_uint32, vp, vp, vp, vp, i32, u64, u64, u64, u64,
                                         C.c_uint32, vp, u64, vp]
        L.oracle_batch_merge.restype = i32
        L.oracle_replay.argtypes = [C.POINTER(_Opt), C.POINTER(_State), vp, vp, C.c_uint32]
        L.oracle_replay.restype = i32
        _lib = L
    return _lib


class OracleError(RuntimeError):
    def __init__(self, code: int, what: str):
        super().__init__(f"oracle {what} returned status {code}")
        self.code = code


def _ptr(a: np.ndarray) -> int:
    assert a.flags["C_CONTIGUOUS"]
    return a.ctypes.data


def _check(code: int, what: str):
    if code != OK:
        raise OracleError(code, what)


def bf16_rne(x: np.ndarray) -> np.ndarray:
    """fp32 -> bf16 bits (uint16), round to nearest even (oracle's own conversion)."""
    L = lib()
    x = np.ascontiguousarray(x, dtype=np.float32).ravel()
    return np.array([L.oracle_bf16_rne(float(v)) for v in x], dtype=np.uint16)


def bf16_bits_to_f32(h: np.ndarray) -> np.ndarray:
    return (np.asarray(h, dtype=np.uint16).astype(np.uint32) << 16).view(np.float32)


def pairs_bytes(k: int, vdt: int) -> int:
    return int(lib().oracle_pairs_bytes(k, vdt))


def compress(g: np.ndarray, r: np.ndarray, k: int, vdt: int = F32):
    """O1. g: float32, or uint16 bf16 bits; r: float32 residual (NOT modified).

    Returns (idx uint32[k] ascending, val float32[k] or uint16[k] bf16 bits, r_new float32[n]).
    """
    gdt = BF16 if g.dtype == np.uint16 else F32
    g = np.ascontiguousarray(g)
    r_new = np.array(r, dtype=np.float32, copy=True)
    n = r_new.size
    idx = np.empty(k, dtype=np.uint32)
    val = np.empty(k, dtype=np.uint16 if vdt == BF16 else np.float32)
    _check(lib().oracle_compress(_ptr(g), gdt, _ptr(r_new), n, k, vdt, _ptr(idx), _ptr(val)),
           "compress")
    return idx, val, r_new


def pairs_pack(idx: np.ndarray, val: np.ndarray, vdt: int = F32) -> np.ndarray:
    idx = np.ascontiguousarray(idx, dtype=np.uint32)
    val = np.ascontiguousarray(val, dtype=np.uint16 if vdt == BF16 else np.float32)
    k = idx.size
    out = np.empty(pairs_bytes(k, vdt), dtype=np.uint8)
    _check(lib().oracle_pairs_pack(_ptr(idx), _ptr(val), k, vdt, _ptr(out)), "pairs_pack")
    return out


def coalesce(pairs: list[np.ndarray], k: int, vdt: int, lo: int, hi: int, average: bool = True):
    """O2. pairs: per-rank packed byte buffers (rank order). Returns (idx uint32, val float32)."""
    P = len(pairs)
    bufs = [np.ascontiguousarray(p, dtype=np.uint8) for p in pairs]
    ptrs = (C.c_void_p * P)(*[_ptr(b) for b in bufs])
    cap = min(P * k, hi - lo)
    idx = np.empty(max(cap, 1), dtype=np.uint32)
    val = np.empty(max(cap, 1), dtype=np.float32)
    nnz = C.c_uint64(0)
    _check(lib().oracle_coalesce(P, C.cast(ptrs, C.c_void_p), k, vdt, lo, hi, int(average),
                                 _ptr(idx), _ptr(val), cap, C.addressof(nnz)), "coalesce")
    return idx[:nnz.value].copy(), val[:nnz.value].copy()


def record_size(mode: int, B: int, nnz: int, nent: int) -> int:
    return int(lib().oracle_record_size(mode, B, nnz, nent))


def batch_merge(diffs: list[tuple[np.ndarray, np.ndarray]], lr, mode: int, n: int, lo: int,
                hi: int, t_first: int, nranks: int) -> np.ndarray:
    """O3+O4. diffs: B (idx uint32 ascending, val float32) in iteration order. Returns record bytes."""
    B = len(diffs)
    idxs = [np.ascontiguousarray(d[0], dtype=np.uint32) for d in diffs]
    vals = [np.ascontiguousarray(d[1], dtype=np.float32) for d in diffs]
    nnz = np.array([i.size for i in idxs], dtype=np.uint64)
    lr = np.ascontiguousarray(np.broadcast_to(np.asarray(lr, dtype=np.float32), (B,)))
    ip = (C.c_void_p * B)(*[_ptr(i) if i.size else 0 for i in idxs])
    vp = (C.c_void_p * B)(*[_ptr(v) if v.size else 0 for v in vals])
    total = record_size(mode, B, int(nnz.sum()), int(nnz.sum()))
    out = np.empty(total, dtype=np.uint8)
    nbytes = C.c_uint64(0)
    _check(lib().oracle_batch_merge(B, C.cast(ip, C.c_void_p), C.cast(vp, C.c_void_p), _ptr(nnz),
                                    _ptr(lr), mode, n, lo, hi, t_first, nranks, _ptr(out), total,
                                    C.addressof(nbytes)), "batch_merge")
    return out[:nbytes.value].copy()


def replay(opt: dict, state: dict, records: list[np.ndarray]) -> dict:
    """O5. state: {"x","m","v" float32 arrays (modified in place; m/v may be None), "n","lo","hi",
    "t","adam_step","momentum_initialized", optional "x_bf16" uint16 array}. Returns state."""
    kinds = {"sgd": SGD, "momentum": MOMENTUM, "adam": ADAM}
    o = _Opt(kinds[opt["kind"]], opt.get("momentum", 0.0), opt.get("dampening", 0.0),
             opt.get("weight_decay", 0.0), opt.get("beta1", 0.9), opt.get("beta2", 0.999),
             opt.get("eps", 1e-8), int(opt.get("nesterov", 0)),
             int(opt.get("allow_accumulated_sum", 0)))
    arrs = {}
    for key in ("x", "m", "v", "x_bf16"):
        a = state.get(key)
        if a is not None:
            assert a.flags["C_CONTIGUOUS"]
        arrs[key] = _ptr(a) if a is not None else None
    st = _State(arrs["x"], arrs["m"], arrs["v"], arrs["x_bf16"], state["n"], state["lo"],
                state["hi"], state["t"], state["adam_step"], state["momentum_initialized"])
    recs = [np.ascontiguousarray(r, dtype=np.uint8) for r in records]
    R = len(recs)
    rp = (C.c_void_p * max(R, 1))(*[_ptr(r) for r in recs])
    rl = np.array([r.size for r in recs] or [0], dtype=np.uint64)
    _check(lib().oracle_replay(C.byref(o), C.byref(st), C.cast(rp, C.c_void_p), _ptr(rl), R),
           "replay")
    state["t"], state["adam_step"] = st.t, st.adam_step
    state["momentum_initialized"] = st.momentum_initialized
    return state


def parse_record(rec: np.ndarray) -> dict:
    """Read a record's header and sections (little-endian) — a reader for tests."""
    b = np.ascontiguousarray(rec, dtype=np.uint8)
    h = {}
    assert bytes(b[:8]) == b"LOWDIFF\x01"
    u32 = lambda o: int(b[o:o + 4].view(np.uint32)[0])
    u64 = lambda o: int(b[o:o + 8].view(np.uint64)[0])
    h.update(version=u32(8), mode=u32(12), B=u32(16), nranks=u32(20), n=u64(24), lo=u64(32),
             hi=u64(40), t_first=u64(48), nnz=u64(56), nent=u64(64), total_bytes=u64(72))
    p16 = lambda x: (x + 15) // 16 * 16
    pos = 80
    B, nnz, nent = h["B"], h["nnz"], h["nent"]
    h["lr"] = b[pos:pos + 4 * B].view(np.float32).copy(); pos += p16(4 * B)
    h["idx"] = b[pos:pos + 4 * nnz].view(np.uint32).copy(); pos += p16(4 * nnz)
    if h["mode"] == SUM:
        h["val"] = b[pos:pos + 4 * nnz].view(np.float32).copy()
    else:
        h["off"] = b[pos:pos + 4 * (nnz + 1)].view(np.uint32).copy(); pos += p16(4 * (nnz + 1))
        h["it"] = b[pos:pos + nent].copy(); pos += p16(nent)
        h["val"] = b[pos:pos + 4 * nent].view(np.float32).copy()
    return h
