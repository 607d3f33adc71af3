"""Pins of oracle O2 (coalesce after the sparse all-gather) and O3/O4 (batch merge + record).

O2 follows Sync (Alg.1 line 5; "Allgather or Allreduce"); O3 follows Step 2 of
batched gradient writing with "tensor addition or dictionary accumulation".
Record layout: DESIGN.md §Record layout.

Pins: Python set union; dense numpy decompress-and-add (a different computation from the
oracle's ordered map); torch.sparse_coo_tensor(...).coalesce() (library); P = 1 / B = 1
identities; STACK unstacking reproduces every input differential bit-for-bit; the
hand-derived worked example and header bytes (tests/golden/worked_example.json); the paper's
Table 4 storage sizes as a bytes-per-pair pin.
"""
import json
import os

import numpy as np
import pytest
import torch

import oracle

HERE = os.path.dirname(__file__)
GOLD = json.load(open(os.path.join(HERE, "golden", "worked_example.json")))
TABLE4 = json.load(open(os.path.join(HERE, "golden", "table4_storage.json")))


def rand_lists(rng, P, n, k, clustered=False):
    out = []
    for _ in range(P):
        if clustered:
            base = rng.integers(0, max(1, n - 4 * k))
            idx = np.sort(rng.choice(np.arange(base, min(n, base + 4 * k)), k, replace=False))
        else:
            idx = np.sort(rng.choice(n, k, replace=False))
        val = rng.standard_normal(k).astype(np.float32)
        val[rng.random(k) < 0.05] = 0.0
        out.append((idx.astype(np.uint32), val))
    return out


def test_worked_example_coalesce():
    ex0, ex1 = GOLD["rank0"], GOLD["rank1"]
    p0 = oracle.pairs_pack(np.array(ex0["idx"], np.uint32), np.array(ex0["val"], np.float32))
    p1 = oracle.pairs_pack(np.array(ex1["idx"], np.uint32), np.array(ex1["val"], np.float32))
    idx, val = oracle.coalesce([p0, p1], 3, oracle.F32, 0, 8, True)
    assert idx.tolist() == GOLD["coalesce_P2_average"]["idx"]
    assert val.tolist() == GOLD["coalesce_P2_average"]["val"]


@pytest.mark.parametrize("P", [1, 2, 3, 8])
@pytest.mark.parametrize("clustered", [False, True])
def test_coalesce_dense_and_union(rng, P, clustered):
    n, k = 20_000, 700
    lists = rand_lists(rng, P, n, k, clustered)
    pairs = [oracle.pairs_pack(i, v) for i, v in lists]
    for lo, hi in [(0, n), (0, n // 3), (n // 3, n), (5000, 5001)]:
        for average in (True, False):
            idx, val = oracle.coalesce(pairs, k, oracle.F32, lo, hi, average)
            union = set()
            for i, _ in lists:
                union |= set(int(x) for x in i if lo <= x < hi)
            assert idx.tolist() == sorted(union)
            dense = np.zeros(n, np.float32)
            for i, v in lists:
                d = np.zeros(n, np.float32); d[i] = v
                dense = dense + d
            if average:
                dense = dense / np.float32(P)
            assert np.all(val == dense[idx])                    # == : +0 and -0 compare equal
            # library cross-check within tolerance
            I = np.concatenate([i for i, _ in lists]).astype(np.int64)
            V = np.concatenate([v for _, v in lists])
            sp = torch.sparse_coo_tensor(torch.from_numpy(I)[None], torch.from_numpy(V), (n,)).coalesce()
            si, sv = sp.indices()[0].numpy(), sp.values().numpy()
            sel = (si >= lo) & (si < hi)
            assert np.array_equal(si[sel], idx.astype(np.int64))
            ref = sv[sel] / (P if average else 1)
            assert np.all(np.abs(val - ref) <= 1e-7 + 1e-6 * np.abs(ref))


def test_coalesce_p1_identity(rng):
    (i, v), = rand_lists(rng, 1, 1000, 100)
    idx, val = oracle.coalesce([oracle.pairs_pack(i, v)], 100, oracle.F32, 0, 1000, True)
    assert np.array_equal(idx, i) and np.array_equal(val.view(np.uint32), v.view(np.uint32))


def test_coalesce_bf16_values(rng):
    lists = rand_lists(rng, 4, 5000, 300)
    pairs, ref = [], []
    for i, v in lists:
        h = torch.from_numpy(v).to(torch.bfloat16)
        pairs.append(oracle.pairs_pack(i, h.view(torch.int16).numpy().view(np.uint16), oracle.BF16))
        ref.append((i, h.to(torch.float32).numpy()))
    idx, val = oracle.coalesce(pairs, 300, oracle.BF16, 0, 5000, True)
    dense = np.zeros(5000, np.float32)
    for i, v in ref:
        d = np.zeros(5000, np.float32); d[i] = v; dense = dense + d
    assert np.all(val == dense[idx] / np.float32(4))


def test_worked_example_merge_bytes():
    D0 = (np.array(GOLD["coalesce_P2_average"]["idx"], np.uint32),
          np.array(GOLD["coalesce_P2_average"]["val"], np.float32))
    D1 = (np.array(GOLD["D1"]["idx"], np.uint32), np.array(GOLD["D1"]["val"], np.float32))
    rec = oracle.batch_merge([D0, D1], GOLD["lr"], oracle.SUM, 8, 0, 8, 0, 2)
    assert rec.size == GOLD["merge_sum"]["bytes"]
    assert rec[:80].tobytes().hex() == GOLD["merge_sum"]["header_hex"]
    h = oracle.parse_record(rec)
    assert h["idx"].tolist() == GOLD["merge_sum"]["idx"]
    assert h["val"].tolist() == GOLD["merge_sum"]["val"]
    rec = oracle.batch_merge([D0, D1], GOLD["lr"], oracle.STACK, 8, 0, 8, 0, 2)
    assert rec.size == GOLD["merge_stack"]["bytes"]
    h = oracle.parse_record(rec)
    for key in ("off", "it", "val"):
        assert h[key].tolist() == GOLD["merge_stack"][key]
    assert h["nent"] == GOLD["merge_stack"]["nent"]


@pytest.mark.parametrize("B", [1, 2, 5, 16])
def test_merge_sum_dense_and_stack_unstack(rng, B):
    n = 30_000
    lo, hi = 1000, 25_000
    diffs = []
    for j in range(B):
        nn = int(rng.integers(0, 900))
        idx = np.sort(rng.choice(np.arange(lo, hi), nn, replace=False)).astype(np.uint32)
        diffs.append((idx, rng.standard_normal(nn).astype(np.float32)))
    lr = (np.arange(B, dtype=np.float32) + 1) * np.float32(0.01)
    rs = oracle.batch_merge(diffs, lr, oracle.SUM, n, lo, hi, 77, 4)
    hs = oracle.parse_record(rs)
    assert hs["total_bytes"] == rs.size == oracle.record_size(oracle.SUM, B, hs["nnz"], hs["nnz"])
    assert (hs["n"], hs["lo"], hs["hi"], hs["t_first"], hs["B"], hs["nranks"]) == (n, lo, hi, 77, B, 4)
    assert np.array_equal(hs["lr"], lr)
    union = sorted(set().union(*[set(d[0].tolist()) for d in diffs]))
    assert hs["idx"].tolist() == union
    dense = np.zeros(n, np.float32)
    for i, v in diffs:
        d = np.zeros(n, np.float32); d[i] = v; dense = dense + d
    assert np.all(hs["val"] == dense[hs["idx"]])
    # STACK: unstacking reproduces each differential bit-for-bit
    rk = oracle.batch_merge(diffs, lr, oracle.STACK, n, lo, hi, 77, 4)
    hk = oracle.parse_record(rk)
    assert hk["nent"] == sum(d[0].size for d in diffs)
    assert rk.size == oracle.record_size(oracle.STACK, B, hk["nnz"], hk["nent"])
    for j, (i, v) in enumerate(diffs):
        sel_u, sel_v = [], []
        for u in range(hk["nnz"]):
            for e in range(hk["off"][u], hk["off"][u + 1]):
                if hk["it"][e] == j:
                    sel_u.append(hk["idx"][u]); sel_v.append(hk["val"][e])
        assert np.array_equal(np.array(sel_u, np.uint32), i)
        assert np.array_equal(np.array(sel_v, np.float32).view(np.uint32), v.view(np.uint32))
    # section padding bytes are zero
    assert rk.size % 16 == 0 and rs.size % 16 == 0
    if B == 1:
        assert np.array_equal(hs["idx"], diffs[0][0])
        assert np.array_equal(hs["val"].view(np.uint32), diffs[0][1].view(np.uint32))


def test_table4_bytes_per_pair():
    """PAPER.md Table 4: LowDiff's differential storage vs the full checkpoint.
    A full checkpoint is x, m, v in fp32 (3Ψ values, Finding 2) = 12Ψ bytes; the
    table's LowDiff column equals 0.1Ψ stored pairs at 8 bytes per pair (u32 index + fp32
    value) to within ±7% for all six models. The oracle's SUM record must cost 8 bytes per
    coalesced pair (+ a constant header), so its ratio to 12Ψ matches the table."""
    for row in TABLE4["rows"]:
        psi = row["params"]
        nnz = int(0.1 * psi)
        rec = oracle.record_size(oracle.SUM, 1, nnz, nnz)
        model_ratio = rec / (12.0 * psi)
        paper_ratio = row["lowdiff"] / row["full"]
        assert abs(model_ratio / paper_ratio - 1.0) < 0.075, row


def test_merge_rejects_bad_arguments():
    d = (np.array([5], np.uint32), np.array([1.0], np.float32))
    with pytest.raises(oracle.OracleError):
        oracle.batch_merge([d], 0.1, oracle.SUM, 10, 6, 10, 0, 1)     # idx outside [lo, hi)
    with pytest.raises(oracle.OracleError):
        oracle.batch_merge([d] * 256, 0.1, oracle.SUM, 10, 0, 10, 0, 1)  # B > 255
