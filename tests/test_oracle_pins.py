"""Pins of the fp64 oracle against things other than itself (no GPU).

Each test names what fixes the expected value: a hand-computed worked example,
a closed form, an invariant, a library routine (torch.autograd / torch.optim on
CPU in fp64 — an independent implementation), finite differences or brute-force
loops.  Together they make a dropped term, wrong sign/index or transposed
operand anywhere in oracle/ fail at least one test.
"""
import json
import math
import os
from fractions import Fraction

import numpy as np
import pytest

import oracle
from oracle import layers as L
from synth import (LayerDesc, LAYER_MLP, LAYER_TRANSFORMER, ACT_NONE, ACT_RELU, ACT_GELU, pack, unpack,
                   gen_params, gen_batch, mlp_stack, transformer_stack)

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def rel(a, b):
    a = np.asarray(a, np.float64); b = np.asarray(b, np.float64)
    nb = np.linalg.norm(b)
    return np.linalg.norm(a - b) / (nb if nb > 1e-30 else 1.0)


# --------------------------------------------------------------------------- (iv) Appendix A
def appendix_a():
    with open(os.path.join(GOLD, "appendix_a_mlp_step.json")) as f:
        return json.load(f)


def test_appendix_a_exact_loss_grads_and_adam():
    """loss, grads exact (dyadic rationals); W' to 1e-15 relative."""
    g = appendix_a()
    descs = [LayerDesc(LAYER_MLP, 2, 2, act=ACT_RELU), LayerDesc(LAYER_MLP, 2, 2, act=ACT_NONE)]
    params = [pack(descs[0], {"w": g["W1"], "b": g["b1"]}), pack(descs[1], {"w": g["W2"], "b": g["b2"]})]
    X = np.array(g["x"], np.float64); T = np.array(g["t"], np.float64)
    loss, grads, new_p, st = oracle.train_step(descs, params, oracle.AdamState.zeros(params), X, T,
                                              lr=1e-3, beta1=0.9, beta2=0.999, eps=1e-8)
    assert Fraction(loss) == Fraction(g["loss_num"], g["loss_den"])
    g1 = unpack(descs[0], grads[0]); g2 = unpack(descs[1], grads[1])
    assert np.array_equal(g1["w"], np.array(g["dW1"])) and np.array_equal(g1["b"], np.array(g["db1"]))
    assert np.array_equal(g2["w"], np.array(g["dW2"])) and np.array_equal(g2["b"], np.array(g["db2"]))
    p1 = unpack(descs[0], new_p[0]); p2 = unpack(descs[1], new_p[1])
    for got, key in ((p1["w"], "W1_new"), (p1["b"], "b1_new"), (p2["w"], "W2_new"), (p2["b"], "b2_new")):
        exp = np.array(g[key])
        assert np.max(np.abs(got - exp) / np.abs(exp)) < 1e-15, key
    assert np.allclose(unpack(descs[0], st.m[0])["w"], np.array(g["mW1"]), rtol=1e-15, atol=0)
    # intermediate values of the worked example
    Y, caches = oracle.stack_forward(descs, params, X)
    assert np.array_equal(Y, np.array(g["y"]))
    assert np.array_equal(caches[0][1]["Z"], np.array(g["z"]))


# --------------------------------------------------------------------------- (iii) finite differences
def _loss_of(descs, params, X, T):
    Y, _ = oracle.stack_forward(descs, params, X)
    return oracle.mse_loss(Y, T, X.shape[0])[0]


def _fd_check(descs, params, X, T, n_probe=None, seed=0, tol=1e-6):
    loss, grads, _ = oracle.stack_loss_and_grads(descs, params, X, T)
    rng = np.random.default_rng(seed)
    worst = 0.0
    for li, flat in enumerate(params):
        idx = np.arange(flat.size) if n_probe is None else rng.choice(flat.size, min(n_probe, flat.size), replace=False)
        num = np.empty(len(idx))
        for j, k in enumerate(idx):
            h = 1e-6 * max(1.0, abs(flat[k]))
            pp = [p.copy() for p in params]; pp[li][k] += h
            pm = [p.copy() for p in params]; pm[li][k] -= h
            num[j] = (_loss_of(descs, pp, X, T) - _loss_of(descs, pm, X, T)) / (2 * h)
        worst = max(worst, rel(grads[li][idx], num))
    assert worst < tol, worst


@pytest.mark.parametrize("act", [ACT_GELU, ACT_RELU, ACT_NONE])
def test_fd_mlp(act):
    descs = [LayerDesc(LAYER_MLP, 4, 4, act=act), LayerDesc(LAYER_MLP, 4, 3, act=act), LayerDesc(LAYER_MLP, 3, 4)]
    params = [p.astype(np.float64) for p in gen_params(descs)]
    rng = np.random.default_rng(3)
    X = rng.standard_normal((5, 4)); T = rng.standard_normal((5, 4))
    if act == ACT_RELU:  # stay away from ReLU kinks
        for li in range(2):
            Y, c = oracle.stack_forward(descs[:li + 1], params[:li + 1], X)
            assert np.min(np.abs(c[li][1]["Z"])) > 1e-3
    _fd_check(descs, params, X, T)


@pytest.mark.parametrize("causal", [False, True])
def test_fd_transformer(causal):
    descs = transformer_stack(2, 8, 2, 4, causal)
    params = [p.astype(np.float64) * 5.0 for p in gen_params(descs)]  # larger weights: non-trivial attention
    for p, d in zip(params, descs):  # restore LN gammas near 1 but not equal
        u = unpack(d, p); u["ln1_g"][:] = 1.0 + 0.1 * np.arange(8) / 8; u["ln2_g"][:] = 1.0 - 0.05 * np.arange(8) / 8
    rng = np.random.default_rng(5)
    X = rng.standard_normal((2, 4, 8)); T = rng.standard_normal((2, 4, 8))
    _fd_check(descs, params, X, T, n_probe=120)


# --------------------------------------------------------------------------- library routine: torch fp64
def _torch_block(X, p, B, S, h, causal):
    import torch
    import torch.nn.functional as F
    d = X.shape[-1]
    U = F.layer_norm(X, (d,), p["ln1_g"], p["ln1_b"], eps=1e-5)
    qkv = U @ p["w_qkv"] + p["b_qkv"]
    q, k, v = qkv.split(d, dim=-1)
    sh = lambda t: t.reshape(B, S, h, d // h).transpose(1, 2)
    c = F.scaled_dot_product_attention(sh(q), sh(k), sh(v), is_causal=causal)
    c = c.transpose(1, 2).reshape(B * S, d)
    X2 = X + c @ p["w_o"] + p["b_o"]
    U2 = F.layer_norm(X2, (d,), p["ln2_g"], p["ln2_b"], eps=1e-5)
    H = U2 @ p["w_fc1"] + p["b_fc1"]
    return X2 + F.gelu(H, approximate="tanh") @ p["w_fc2"] + p["b_fc2"]


@pytest.mark.parametrize("causal", [False, True])
def test_transformer_step_matches_torch_autograd_and_adam(causal):
    import torch
    B, S, d, h, nl = 3, 6, 16, 4, 2
    descs = transformer_stack(nl, d, h, S, causal)
    params = [p.astype(np.float64) * 8.0 for p in gen_params(descs)]
    for p, dd in zip(params, descs):
        u = unpack(dd, p); u["ln1_g"][:] = 1.0 + 0.3 * np.sin(np.arange(d)); u["ln2_g"][:] = 1.0 + 0.2 * np.cos(np.arange(d))
    X, T = gen_batch(descs, B, 1)
    X = X.astype(np.float64); T = T.astype(np.float64)
    state = oracle.AdamState.zeros(params)
    loss, grads, new_p, st = oracle.train_step(descs, params, state, X, T, lr=1e-2)

    tp = [torch.tensor(p, dtype=torch.float64, requires_grad=True) for p in params]
    A = torch.tensor(X.reshape(B * S, d))
    for dd, flat in zip(descs, tp):
        parts, off = {}, 0
        for name, shape in __import__("synth").segments(dd):
            n = int(np.prod(shape)); parts[name] = flat[off:off + n].reshape(shape); off += n
        A = _torch_block(A, parts, B, S, h, causal)
    tl = 0.5 * ((A - torch.tensor(T.reshape(B * S, d))) ** 2).sum() / B
    tl.backward()
    assert abs(tl.item() - loss) <= 1e-13 * abs(loss)
    for g, t in zip(grads, tp):
        assert rel(g, t.grad.numpy()) < 1e-11
    # Adam vs torch.optim.Adam fed the oracle's own gradients (gradients such as d b_k are
    # mathematically 0 and numerically noise; Adam's g/(|g|+eps) would amplify that noise)
    for g, t in zip(grads, tp):
        t.grad = torch.tensor(g)
    opt = torch.optim.Adam(tp, lr=1e-2, betas=(0.9, 0.999), eps=1e-8)
    opt.step()
    for w, t in zip(new_p, tp):
        assert rel(w, t.detach().numpy()) < 1e-13
    for m, t in zip(st.m, tp):
        assert rel(m, opt.state[t]["exp_avg"].numpy()) < 1e-13
    for v, t in zip(st.v, tp):
        assert rel(v, opt.state[t]["exp_avg_sq"].numpy()) < 1e-13


def test_mlp_step_matches_torch_autograd():
    import torch
    descs = mlp_stack(4, 32)
    params = [p.astype(np.float64) for p in gen_params(descs)]
    X, T = gen_batch(descs, 8, 2)
    loss, grads, _ = oracle.stack_loss_and_grads(descs, params, X.astype(np.float64), T.astype(np.float64))
    tp = [torch.tensor(p, requires_grad=True) for p in params]
    A = torch.tensor(X, dtype=torch.float64)
    for i, (dd, flat) in enumerate(zip(descs, tp)):
        W = flat[:32 * 32].reshape(32, 32); b = flat[32 * 32:]
        A = A @ W + b
        if i < 3:
            A = torch.nn.functional.gelu(A, approximate="tanh")
    tl = 0.5 * ((A - torch.tensor(T, dtype=torch.float64)) ** 2).sum() / 8
    tl.backward()
    assert abs(tl.item() - loss) < 1e-13 * loss
    for g, t in zip(grads, tp):
        assert rel(g, t.grad.numpy()) < 1e-12


# --------------------------------------------------------------------------- (i) microbatch linearity
@pytest.mark.parametrize("kind", ["mlp", "transformer"])
def test_microbatch_sum_equals_full_batch(kind):
    if kind == "mlp":
        descs = mlp_stack(3, 16); B, m = 12, 4
    else:
        descs = transformer_stack(2, 16, 2, 5, True); B, m = 4, 2
    params = [p.astype(np.float64) for p in gen_params(descs)]
    X, T = gen_batch(descs, B, 1)
    full_loss, full_g, _ = oracle.stack_loss_and_grads(descs, params, X, T)
    acc = [np.zeros_like(g) for g in full_g]; acc_loss = 0.0
    b = B // m
    for i in range(m):
        l, g, _ = oracle.stack_loss_and_grads(descs, params, X[i * b:(i + 1) * b], T[i * b:(i + 1) * b], loss_batch=B)
        acc_loss += l
        acc = [a + gi for a, gi in zip(acc, g)]
    assert abs(acc_loss - full_loss) <= 1e-12 * full_loss
    for a, g in zip(acc, full_g):
        assert rel(a, g) <= 1e-12


# --------------------------------------------------------------------------- (ii) decomposed matmul
@pytest.mark.parametrize("splits", [(1, 1, 1), (4, 1, 1), (3, 2, 5), (7, 3, 2)])
def test_split_gemm_equals_plain(splits):
    rng = np.random.default_rng(11)
    M, N, K = 37, 29, 53
    X = rng.standard_normal((M, K)); W = rng.standard_normal((K, N)); dY = rng.standard_normal((M, N))
    ref = (X @ W, dY @ W.T, X.T @ dY)  # block-matrix identity: the decomposition equals the definition
    got = oracle.split_gemm_fwd_bwd(X, W, dY, *splits)
    for a, b in zip(got, ref):
        assert rel(a, b) <= 1e-13
    rows = rng.integers(0, M, 20); cols = rng.integers(0, N, 20)
    assert np.allclose(oracle.sampled_gemm_entries(X, W, dY, rows, cols, "Y"), ref[0][rows, cols], rtol=1e-13)
    r2 = rng.integers(0, K, 20)
    assert np.allclose(oracle.sampled_gemm_entries(X, W, dY, rows, r2, "dX"), ref[1][rows, r2], rtol=1e-13)
    assert np.allclose(oracle.sampled_gemm_entries(X, W, dY, r2, cols, "dW"), ref[2][r2, cols], rtol=1e-13)


def test_gemm_brute_force_loops():
    rng = np.random.default_rng(2)
    X = rng.standard_normal((3, 4)); W = rng.standard_normal((4, 2)); dY = rng.standard_normal((3, 2))
    Y, dX, dW = oracle.gemm_fwd_bwd(X, W, dY)
    for i in range(3):
        for j in range(2):
            assert math.isclose(Y[i, j], sum(X[i, k] * W[k, j] for k in range(4)), rel_tol=1e-14)
    for i in range(3):
        for k in range(4):
            assert math.isclose(dX[i, k], sum(dY[i, j] * W[k, j] for j in range(2)), rel_tol=1e-13, abs_tol=1e-15)
    for k in range(4):
        for j in range(2):
            assert math.isclose(dW[k, j], sum(X[i, k] * dY[i, j] for i in range(3)), rel_tol=1e-13, abs_tol=1e-15)


# --------------------------------------------------------------------------- Adam closed forms
def test_adam_step1_and_step2_closed_forms():
    rng = np.random.default_rng(4)
    W = rng.standard_normal(50); g1 = rng.standard_normal(50); g2 = rng.standard_normal(50)
    lr, b1, b2, eps = 1e-3, 0.9, 0.999, 1e-8
    W1, m1, v1 = oracle.adam_update(W, g1, 0 * W, 0 * W, 1, lr, b1, b2, eps)
    assert np.allclose(W1, W - lr * g1 / (np.abs(g1) + eps), rtol=1e-14, atol=1e-16)
    W2, m2, v2 = oracle.adam_update(W1, g2, m1, v1, 2, lr, b1, b2, eps)
    m_ref = 0.09 * g1 + 0.1 * g2
    v_ref = 0.000999 * g1 ** 2 + 0.001 * g2 ** 2
    assert np.allclose(m2, m_ref, rtol=1e-13) and np.allclose(v2, v_ref, rtol=1e-13)
    assert np.allclose(W2, W1 - lr * (m_ref / 0.19) / (np.sqrt(v_ref / 0.001999) + eps), rtol=1e-13)
    # constant gradient: the same update every step
    g = rng.standard_normal(10); Wc = np.zeros(10); m = 0 * g; v = 0 * g; steps = []
    for t in range(1, 5):
        Wn, m, v = oracle.adam_update(Wc, g, m, v, t, lr, b1, b2, eps)
        steps.append(Wn - Wc); Wc = Wn
    for s in steps[1:]:
        assert np.allclose(s, steps[0], rtol=1e-12)


def test_linear_regression_closed_form():
    """One Linear + MSE is linear regression: grad_W = X^T (X W + b - T)/B, grad_b = sum(XW+b-T)/B."""
    rng = np.random.default_rng(6)
    B, di, do = 7, 5, 3
    X = rng.standard_normal((B, di)); T = rng.standard_normal((B, do))
    Wm = rng.standard_normal((di, do)); b = rng.standard_normal(do)
    descs = [LayerDesc(LAYER_MLP, di, do)]
    loss, grads, _ = oracle.stack_loss_and_grads(descs, [pack(descs[0], {"w": Wm, "b": b})], X, T)
    R = X @ Wm + b - T
    g = unpack(descs[0], grads[0])
    assert np.allclose(g["w"], X.T @ R / B, rtol=1e-13) and np.allclose(g["b"], R.sum(0) / B, rtol=1e-13)
    assert math.isclose(loss, 0.5 * np.sum(R * R) / B, rel_tol=1e-14)


# --------------------------------------------------------------------------- invariants and special cases
def test_layernorm_invariants():
    rng = np.random.default_rng(8)
    x = rng.standard_normal((6, 32)) * 3 + 1
    y, cache = L.layernorm_fwd(x, np.ones(32), np.zeros(32))
    assert np.allclose(y.mean(-1), 0, atol=1e-14)
    assert np.allclose(y.var(-1), 1 - 1e-5 / (x.var(-1) + 1e-5), rtol=1e-12)  # biased var, eps inside sqrt
    dy = rng.standard_normal((6, 32))
    g = rng.standard_normal(32)
    _, c2 = L.layernorm_fwd(x, g, rng.standard_normal(32))
    dx, dg, db = L.layernorm_bwd(dy, c2)
    assert np.allclose(dx.sum(-1), 0, atol=1e-12)  # sum_k dX = 0 (LN is invariant to shifting x)
    # near-invariance to scaling x - mu: sum_k xhat dx = rstd sum(xhat dxhat)(1 - mean(xhat^2)), O(eps/var)
    xhat, rstd = c2[0], c2[1][:, 0]
    lhs = (dx * xhat).sum(-1)
    rhs = rstd * (xhat * dy * g).sum(-1) * (1 - (xhat ** 2).mean(-1))
    assert np.allclose(lhs, rhs, rtol=1e-6, atol=1e-13) and np.all(np.abs(lhs) < 1e-4)
    # zero-variance row: xhat = 0 -> output = beta, no NaN (reading c24)
    yc, _ = L.layernorm_fwd(np.full((1, 8), 2.5), np.full(8, 3.0), np.arange(8.0))
    assert np.array_equal(yc[0], np.arange(8.0))


def test_softmax_invariants():
    rng = np.random.default_rng(9)
    z = rng.standard_normal((5, 11)) * 4
    p = L.softmax_fwd(z)
    assert np.allclose(p.sum(-1), 1, atol=1e-15) and np.all(p > 0)
    dz = L.softmax_bwd(rng.standard_normal((5, 11)), p)
    assert np.allclose(dz.sum(-1), 0, atol=1e-14)
    # shift invariance
    assert np.allclose(L.softmax_fwd(z + 100.0), p, rtol=1e-12)


def test_identity_block():
    """W_o = W_fc2 = 0 and b_o = b_fc2 = 0 => the block is the identity (Y == X exactly)."""
    d = 16
    desc = transformer_stack(1, d, 4, 5, False)[0]
    p = unpack(desc, gen_params([desc])[0].astype(np.float64).copy())
    for k in ("w_o", "b_o", "w_fc2", "b_fc2"):
        p[k][...] = 0
    X = np.random.default_rng(1).standard_normal((10, d))
    Y, _ = L.transformer_block_fwd(X, p, 2, 5, 4, False)
    assert np.array_equal(Y, X)


@pytest.mark.parametrize("causal", [False, True])
def test_uniform_attention_when_q_is_zero(causal):
    """Q = 0 => uniform P: C = mean of V over keys (or prefix mean 0..i when causal); causal row 0 = V[0]."""
    B, S, h, d = 2, 6, 2, 8
    rng = np.random.default_rng(10)
    qkv = rng.standard_normal((B * S, 3 * d)); qkv[:, :d] = 0
    C, (Q, K, V, P, _) = L.attention_fwd(qkv, B, S, h, causal)
    Vm = qkv[:, 2 * d:].reshape(B, S, d)
    Cm = C.reshape(B, S, d)
    for b in range(B):
        for i in range(S):
            exp = Vm[b, :i + 1].mean(0) if causal else Vm[b].mean(0)
            assert np.allclose(Cm[b, i], exp, rtol=1e-13, atol=1e-15)
    if causal:
        assert np.array_equal(Cm[:, 0], Vm[:, 0])


def test_block_forward_brute_force_loops():
    """Pure-Python loops (no NumPy matmul/einsum) for one tiny causal block."""
    B, S, d, h = 1, 3, 4, 2
    dh = d // h
    desc = transformer_stack(1, d, h, S, True)[0]
    flat = gen_params([desc])[0].astype(np.float64) * 10
    p = unpack(desc, flat)
    X = np.random.default_rng(12).standard_normal((S, d))
    Y, _ = L.transformer_block_fwd(X, p, B, S, h, True)

    def ln(row, g, b):
        mu = sum(row) / len(row); var = sum((r - mu) ** 2 for r in row) / len(row)
        return [(r - mu) / math.sqrt(var + 1e-5) * g[i] + b[i] for i, r in enumerate(row)]

    def mm(row, W, b):
        return [sum(row[k] * W[k][j] for k in range(len(row))) + b[j] for j in range(len(W[0]))]

    Xl = X.tolist(); P = {k: v.tolist() for k, v in p.items()}
    qkv = [mm(ln(Xl[s], P["ln1_g"], P["ln1_b"]), P["w_qkv"], P["b_qkv"]) for s in range(S)]
    C = [[0.0] * d for _ in range(S)]
    for hh in range(h):
        for i in range(S):
            sc = [sum(qkv[i][hh * dh + e] * qkv[j][d + hh * dh + e] for e in range(dh)) / math.sqrt(dh) for j in range(i + 1)]
            mx = max(sc); ex = [math.exp(s - mx) for s in sc]; tot = sum(ex)
            for e in range(dh):
                C[i][hh * dh + e] = sum(ex[j] / tot * qkv[j][2 * d + hh * dh + e] for j in range(i + 1))
    X2 = [[Xl[s][k] + v for k, v in enumerate(mm(C[s], P["w_o"], P["b_o"]))] for s in range(S)]
    gel = lambda x: 0.5 * x * (1 + math.tanh(math.sqrt(2 / math.pi) * (x + 0.044715 * x ** 3)))
    for s in range(S):
        Hs = mm(ln(X2[s], P["ln2_g"], P["ln2_b"]), P["w_fc1"], P["b_fc1"])
        out = [X2[s][k] + v for k, v in enumerate(mm([gel(x) for x in Hs], P["w_fc2"], P["b_fc2"]))]
        assert np.allclose(Y[s], out, rtol=1e-12, atol=1e-13)


def test_gelu_grad_matches_fd_and_known_values():
    x = np.linspace(-4, 4, 41)
    h = 1e-6
    assert np.allclose(L.gelu_tanh_grad(x), (L.gelu_tanh(x + h) - L.gelu_tanh(x - h)) / (2 * h), rtol=1e-7, atol=1e-9)
    assert L.gelu_tanh(np.array([0.0]))[0] == 0.0 and L.gelu_tanh_grad(np.array([0.0]))[0] == 0.5


def test_swap_model_paper_formulas():
    """P:726-735, 772-775 on cfg1's |W| (1,052,672 B fp32, m = 4)."""
    W = 4 * 4 * (256 * 256 + 256)
    assert W == 1052672
    assert oracle.weight_swap_baseline_dp(W, 4, 1) == 18 * W
    assert oracle.weight_swap_harmony_dp(W, 4, 1) == 3 * W
    assert oracle.weight_swap_baseline_dp(W, 4, 8) == 8 * 18 * W
    assert oracle.weight_swap_harmony_pp(W, 4, 8) == 3 * W
