"""LowDiff+ (§5, Algorithm 2): the dense GPU update (Alg. 2 line 7)
and the host replica update (line 12) against the CPU oracle's optimizer step, bit for bit, and
the LowDiffPlus driver: after T real training iterations the CPU replica equals the GPU model
bitwise, and recovery restores it.

The oracle reference for T dense steps is its replay of T one-iteration records that carry every
index of [lo, hi) (absent entries and explicit zeros agree, reading #12/#14)."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_sc_yaolhlzz25_b200 as ld

CASES = [("sgd", 0.0, 0), ("sgd", 0.01, 0), ("momentum", 0.0, 0), ("momentum", 1e-4, 1), ("adam", 0.0, 0)]


def dense_chain(L, T, seed, bf16):
    rng = np.random.default_rng(seed)
    grads = []
    for t in range(T):
        g = (rng.standard_normal(L) * 10.0 ** rng.uniform(-4, -1)).astype(np.float32)
        g[rng.random(L) < 0.01] = 0.0
        g[rng.random(L) < 0.01] = -0.0
        if bf16:
            g = oracle.bf16_bits_to_f32(oracle.bf16_rne(g))
        grads.append(g)
    lrs = [np.float32(1e-3 * (1 + 0.5 * (t % 3))) for t in range(T)]
    return grads, lrs


def oracle_dense(kind, wd, nesterov, L, grads, lrs, x, m, v, adam_step):
    n, lo, hi = L + 7, 3, 3 + L
    idx = np.arange(lo, hi, dtype=np.uint32)
    recs = [oracle.batch_merge([(idx, g)], np.array([lr], np.float32), oracle.STACK, n, lo, hi, t, 1)
            for t, (g, lr) in enumerate(zip(grads, lrs))]
    opt = {"kind": kind, "weight_decay": wd, "momentum": 0.9, "nesterov": nesterov}
    st = {"x": x.copy(), "m": None if m is None else m.copy(), "v": None if v is None else v.copy(),
          "n": n, "lo": lo, "hi": hi, "t": 0, "adam_step": adam_step, "momentum_initialized": 0}
    oracle.replay(opt, st, recs)
    return opt, st


def init(kind, L, seed):
    rng = np.random.default_rng(seed)
    x = (rng.standard_normal(L) * 0.02).astype(np.float32)
    m = None if kind == "sgd" else (np.zeros(L, np.float32) if kind == "momentum" else
                                    (rng.standard_normal(L) * 1e-4).astype(np.float32))
    v = None if kind != "adam" else (m * m + np.float32(1e-10)).astype(np.float32)
    return x, m, v


def to_t(a, dev="cpu"):
    return None if a is None else torch.from_numpy(a.copy()).to(dev)


@pytest.mark.parametrize("bf16", [False, True])
@pytest.mark.parametrize("kind,wd,nesterov", CASES)
def test_host_update_matches_oracle(kind, wd, nesterov, bf16):
    """The CPU replica update (native C++, several threads, ragged length) == the oracle."""
    L, T = 10_007, 5
    grads, lrs = dense_chain(L, T, 31, bf16)
    x, m, v = init(kind, L, 32)
    opt, ref = oracle_dense(kind, wd, nesterov, L, grads, lrs, x, m, v, 9)
    st = {"x": to_t(x), "m": to_t(m), "v": to_t(v), "n": L + 7, "lo": 3, "hi": 3 + L, "t": 0, "adam_step": 9,
          "momentum_initialized": 0}
    for t, (g, lr) in enumerate(zip(grads, lrs)):
        gt = torch.from_numpy(g).to(torch.bfloat16) if bf16 else torch.from_numpy(g)
        ld.host_update(st, opt, gt, float(lr), threads=1 + t % 3)
    assert (st["t"], st["adam_step"], st["momentum_initialized"]) == \
        (ref["t"], ref["adam_step"], ref["momentum_initialized"])
    for key in ("x", "m", "v"):
        if ref[key] is not None:
            assert np.array_equal(st[key].numpy().view(np.uint32), ref[key].view(np.uint32)), key


def test_host_update_errors():
    L = 64
    st = {"x": torch.zeros(L), "m": None, "v": None, "n": L, "lo": 0, "hi": L, "t": 0, "adam_step": 0,
          "momentum_initialized": 0}
    with pytest.raises(ValueError):
        ld.host_update(st, {"kind": "sgd"}, torch.zeros(L + 1), 0.1)
    with pytest.raises(ld.LowDiffError):
        ld.host_update(st, {"kind": "adam"}, torch.zeros(L), 0.1)          # Adam needs m, v


@pytest.mark.gpu
@pytest.mark.parametrize("bf16", [False, True])
@pytest.mark.parametrize("kind,wd,nesterov", CASES)
def test_dense_update_matches_oracle(kind, wd, nesterov, bf16):
    """The GPU model update (Alg. 2 line 7) == the oracle, ragged length, fp32 and bf16 grads."""
    L, T = 1_000_003, 4
    grads, lrs = dense_chain(L, T, 41, bf16)
    x, m, v = init(kind, L, 42)
    opt, ref = oracle_dense(kind, wd, nesterov, L, grads, lrs, x, m, v, 5)
    st = {"x": to_t(x, "cuda"), "m": to_t(m, "cuda"), "v": to_t(v, "cuda"), "n": L + 7, "lo": 3, "hi": 3 + L,
          "t": 0, "adam_step": 5, "momentum_initialized": 0}
    before = ld.launch_count()
    for g, lr in zip(grads, lrs):
        gt = torch.from_numpy(g).cuda()
        ld.dense_update(st, opt, gt.to(torch.bfloat16) if bf16 else gt, float(lr))
    assert ld.launch_count() - before == T
    torch.cuda.synchronize()
    for key in ("x", "m", "v"):
        if ref[key] is not None:
            assert np.array_equal(st[key].cpu().numpy().view(np.uint32), ref[key].view(np.uint32)), key


@pytest.mark.gpu
@pytest.mark.parametrize("kind", ["sgd", "momentum", "adam"])
def test_lowdiff_plus_replica_equals_gpu_model(kind):
    """A small MLP trained T iterations with LowDiff+: the gradients the hooks snapshot are the
    ones autograd produced, the CPU replica equals the GPU model (and optimizer state) bit for bit
    after every iteration, the model trains, and recovery after a simulated software failure
    restores the replica."""
    from paper_conf_sc_yaolhlzz25_b200.plus import LowDiffPlus
    torch.manual_seed(0)
    model = torch.nn.Sequential(torch.nn.Linear(64, 256), torch.nn.ReLU(), torch.nn.Linear(256, 257),
                                torch.nn.ReLU(), torch.nn.Linear(257, 10)).cuda()
    lr = {"sgd": 0.05, "momentum": 0.02, "adam": 1e-3}[kind]
    plus = LowDiffPlus(model, {"kind": kind, "momentum": 0.9}, lr=lr, threads=4)
    xs, ys = torch.randn(512, 64, device="cuda"), torch.randint(0, 10, (512,), device="cuda")
    loss_fn = torch.nn.CrossEntropyLoss()
    losses = []
    for t in range(12):
        plus.zero_grad()
        loss = loss_fn(model(xs), ys)
        loss.backward()
        if t == 0:                                   # the flat gradient buffer holds autograd's grads
            ref = torch.autograd.grad(loss_fn(model(xs), ys), list(model.parameters()))
            assert torch.equal(torch.cat([r.reshape(-1) for r in ref]), plus.gflat)
        plus.step()
        losses.append(float(loss))
        plus.flush()
        for key in ("x", "m", "v"):
            if plus.state[key] is not None:
                assert torch.equal(plus.state[key].cpu().view(torch.int32), plus.replica[key].view(torch.int32)), (t, key)
    assert losses[-1] < losses[0]
    good = plus.state["x"].clone()
    plus.state["x"].fill_(float("nan"))              # the GPU copy is lost
    plus.recover()
    assert torch.equal(plus.state["x"].view(torch.int32), good.view(torch.int32))
    assert plus.state["t"] == 12 and plus.t == 12
    plus.close()
