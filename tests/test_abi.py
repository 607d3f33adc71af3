"""The C ABI library loads and exports every symbol include/lowdiff.h declares; host-only calls
(sizes, shard bounds, header parsing, argument validation) behave as documented. No GPU needed:
no call here reaches a kernel."""
import ctypes as C
import os
import re

import numpy as np
import pytest

import oracle
import paper_conf_sc_yaolhlzz25_b200 as ld

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module", autouse=True)
def built():
    from paper_conf_sc_yaolhlzz25_b200 import build
    build.build()


def header_functions():
    src = open(os.path.join(ROOT, "include", "lowdiff.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(lowdiff_[a-z0-9_]+)\s*\(", src)))


def test_every_declared_symbol_is_exported():
    names = header_functions()
    assert len(names) >= 25
    L = ld.lib()
    for name in names:
        assert hasattr(L, name), name
    assert sorted(ld.EXPORTS) == names


def test_host_helpers_match_definitions():
    assert ld.k_for_density(269_722, 0.01) == 2697
    assert ld.k_for_density(138_357_544, 0.001) == 138_357
    assert ld.k_for_density(1_557_611_200, 0.001) == 1_557_611
    assert ld.k_for_density(10, 1e-9) == 1 and ld.k_for_density(10, 5.0) == 10
    for k in (1, 3, 4, 5, 2697):
        for vdt, o in (("f32", oracle.F32), ("bf16", oracle.BF16)):
            assert ld.pairs_bytes(k, vdt) == oracle.pairs_bytes(k, o)
    n = 1_557_611_200
    bounds = [ld.shard_bounds(n, 8, p) for p in range(8)]
    assert bounds[0][0] == 0 and bounds[-1][1] == n
    assert all(bounds[p][1] == bounds[p + 1][0] for p in range(7))
    assert bounds[1] == (n // 8, 2 * n // 8)
    for mode, om in (("sum", oracle.SUM), ("stack", oracle.STACK)):
        for B, nnz, nent in ((1, 0, 0), (2, 6, 8), (16, 1000, 3000), (255, 7, 7)):
            if mode == "sum":
                nent = nnz
            assert ld.record_size(mode, B, nnz, nent) == oracle.record_size(om, B, nnz, nent)


def test_record_max_bytes_shard_bound():
    """A shard's record has at most hi - lo unique indices (bound the record buffers by
    min(B cap, hi - lo)); the entries stay bounded by max_entries."""
    for mode in ("sum", "stack"):
        for B, me, lo, hi in ((32, 400_000_000, 0, 194_701_400), (8, 1000, 10, 5000), (4, 10, 0, 1_000_000)):
            u = min(me, hi - lo)
            assert ld.record_max_bytes(mode, B, me, lo, hi) == ld.record_size(mode, B, u, me if mode == "stack" else u)
            assert ld.record_max_bytes(mode, B, me, lo, hi) <= ld.record_max_bytes(mode, B, me)
    # C5 shard, STACK, B = 32 differentials of ~12.5 M entries
    assert ld.record_max_bytes("stack", 32, 32 * 12_460_888, 0, 194_701_400) < 3.7e9 < \
        ld.record_max_bytes("stack", 32, 32 * 12_460_888)


def test_p2p_window_layout():
    """Exchange window of the fused Sync (include/lowdiff.h (2')): u64 ready[P] | u64 done[P] |
    u64 epoch, padded to 256 B, then two 256-B aligned slots of one packed pairs buffer each."""
    a256 = lambda x: (x + 255) // 256 * 256
    for P in (2, 3, 8, 64):
        for k, vdt in ((1, "f32"), (2697, "f32"), (3_351_418, "bf16")):
            assert ld.p2p_window_bytes(P, k, vdt) == a256(16 * P + 8) + 2 * a256(ld.pairs_bytes(k, vdt))
    assert ld.p2p_window_bytes(65, 100) == 0 and ld.p2p_window_bytes(2, 0) == 0   # out of range


def test_record_parse_reads_oracle_records():
    rng = np.random.default_rng(3)
    diffs = []
    for j in range(3):
        idx = np.sort(rng.choice(np.arange(100, 900), 50, replace=False)).astype(np.uint32)
        diffs.append((idx, rng.standard_normal(50).astype(np.float32)))
    for om, mode in ((oracle.SUM, 0), (oracle.STACK, 1)):
        rec = oracle.batch_merge(diffs, 0.5, om, 1000, 100, 900, 42, 4)
        h = ld.record_parse(rec)
        ref = oracle.parse_record(rec)
        for key in ("version", "mode", "B", "nranks", "n", "lo", "hi", "t_first", "nnz", "nent",
                    "total_bytes"):
            assert h[key] == ref[key], key
        bad = rec.copy()
        bad[72] ^= 1                                        # total_bytes
        with pytest.raises(ld.LowDiffError) as e:
            ld.record_parse(bad)
        assert e.value.status == "ECORRUPT"


def test_argument_validation_is_host_side():
    L = ld.lib()
    assert L.lowdiff_compress(None, 0, None, 10, 0, None, 0, None, 0, None) == 1       # k = 0
    assert L.lowdiff_compress(None, 0, None, 10, 11, None, 0, None, 0, None) == 1      # k > n
    assert L.lowdiff_compress(None, 0, None, 1 << 31, 5, None, 0, None, 0, None) == 1  # n >= 2^31
    assert L.lowdiff_compress(None, 7, None, 10, 5, None, 0, None, 0, None) == 1       # dtype
    assert L.lowdiff_compress(C.c_void_p(16), 0, C.c_void_p(16), 10, 5, C.c_void_p(16), 0,
                              C.c_void_p(16), 0, None) == 2                            # workspace
    assert L.lowdiff_compress(C.c_void_p(8), 0, C.c_void_p(16), 10, 5, C.c_void_p(16), 0,
                              C.c_void_p(16), 1 << 30, None) == 1                      # alignment
    b = C.c_uint64()
    assert L.lowdiff_batch_merge_workspace_size(0, 10, 0, 10, C.byref(b)) == 1          # B = 0
    assert L.lowdiff_batch_merge_workspace_size(256, 10, 0, 10, C.byref(b)) == 1        # B > 255
    assert L.lowdiff_batch_merge_workspace_size(4, 10, 5, 5, C.byref(b)) == 1           # lo >= hi
    assert L.lowdiff_coalesce_workspace_size(0, 10, 0, 0, 10, C.byref(b)) == 1          # P = 0
    assert L.lowdiff_coalesce_workspace_size(2, 10, 0, 0, 10, C.byref(b)) == 0 and b.value > 0
    assert ld.lib().lowdiff_status_string(4) == b"records do not form a chain from the state"
    assert L.lowdiff_launch_count() == 0


def test_product_path_has_no_cpu_fallback():
    import torch
    g = torch.zeros(16)
    r = torch.zeros(16)
    with pytest.raises(ValueError, match="CUDA"):
        ld.compress(g, r, 4)
    src = open(os.path.join(ROOT, "paper_conf_sc_yaolhlzz25_b200", "__init__.py")).read()
    assert "import oracle" not in src and "from oracle" not in src
