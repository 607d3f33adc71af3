"""lowdiff_plan_init / lowdiff_plan_record_due (include/lowdiff.h (0)): the paper's problem
statement — n, rho, batching size B, full-checkpoint frequency FCF
 — and the record-boundary policy of DESIGN.md reading #25 (a record closes every B
iterations and before every full checkpoint, so a chain never spans one; P:326 bounds what a
failure loses). Host-only calls: no GPU."""
import math

import pytest

import paper_conf_sc_yaolhlzz25_b200 as ld


@pytest.fixture(scope="module", autouse=True)
def built():
    from paper_conf_sc_yaolhlzz25_b200 import build
    build.build()


def expected_schedule(B, F, T):
    """Independent enumeration of reading #25: full checkpoints at multiples of F (only t = 0 when
    F = 0); between two of them, records [f, f+B), [f+B, f+2B), ... the last one cut short at the
    next full checkpoint. Returns (set of full-checkpoint iterations, list of (t_first, length))."""
    fulls = {0} if F == 0 else {t for t in range(T) if t % F == 0}
    starts = sorted(fulls) + [T if F == 0 else math.ceil(T / F) * F]
    records = []
    for f, g in zip(starts[:-1], starts[1:]):
        end = g if F else T
        for a in range(f, end, B):
            records.append((a, min(B, end - a)))
    return fulls, [(a, min(b, T - a)) for a, b in records if a < T]   # the last one may still be open


@pytest.mark.parametrize("B,F", [(4, 8), (4, 10), (8, 8), (5, 12), (16, 7), (1, 3), (3, 0), (7, 1), (255, 1000)])
def test_record_due_matches_reading_25(B, F):
    T = 3 * max(F, B) + 5
    plan = ld.plan_init(1000, 0.01, B, F)
    fulls, records = expected_schedule(B, F, T)
    got_fulls, got_records, open_first = set(), [], 0
    for t in range(T):
        close, blen, full = ld.plan_record_due(plan, t)
        if full:
            got_fulls.add(t)
            assert blen == 1                           # a full checkpoint always opens a record
        assert blen == t - open_first + 1
        if close:
            got_records.append((open_first, blen))
            open_first = t + 1
    if open_first < T:
        got_records.append((open_first, T - open_first))   # the open (unflushed) record
    assert got_fulls == fulls
    assert got_records == records
    assert all(1 <= b <= B for _, b in got_records)
    # a chain never spans a full checkpoint
    for a, b in got_records:
        assert not any(a < f < a + b for f in got_fulls)


def test_plan_init_problem_statement():
    cases = [(269_722, 0.01, 4, 8, 1, 0), (25_557_032, 0.01, 8, 16, 8, 3), (138_357_544, 0.001, 16, 16, 8, 7),
             (335_141_888, 0.01, 8, 32, 8, 5), (1_557_611_200, 0.001, 32, 32, 8, 6)]
    for n, rho, B, F, P, p in cases:
        plan = ld.plan_init(n, rho, B, F, "f32", "f32", P, p)
        assert plan.k == max(1, min(n, math.floor(rho * n)))
        assert (plan.lo, plan.hi) == (p * n // P, (p + 1) * n // P)
        assert (plan.n, plan.B, plan.full_every, plan.nranks, plan.rank) == (n, B, F, P, p)
    plan = ld.plan_init(100, 0.5, 2, 4, "bf16", "bf16")
    assert (plan.gdt, plan.vdt) == (ld.BF16, ld.BF16)


@pytest.mark.parametrize("args", [(0, 0.01, 4, 8), (1 << 31, 0.01, 4, 8), (100, 0.0, 4, 8), (100, 1.5, 4, 8),
                                  (100, 0.01, 0, 8), (100, 0.01, 256, 8)])
def test_plan_init_rejects(args):
    with pytest.raises(ld.LowDiffError) as e:
        ld.plan_init(*args)
    assert e.value.status == "EINVAL"
    with pytest.raises(ld.LowDiffError):
        ld.plan_init(100, 0.01, 4, 8, "f32", "f32", 2, 2)       # rank out of range
