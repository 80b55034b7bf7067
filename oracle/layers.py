"""Per-layer forward/backward of the registered layer kinds, fp64 NumPy (oracle; test infrastructure only).

The paper fixes no layer math beyond "one type of layer (like Transformers)"
 and BERT; the block below is reading c1 of
DESIGN.md: a pre-LN Transformer block with biases everywhere, no dropout, no
final LN.  Every op follows its textbook definition, written out; matmul is a
library primitive (NumPy / BLAS dgemm).  Row-major conventions: Y = X.W + b
with W stored [d_in][d_out]; QKV columns are [Q | K | V], head h using columns
h*dh..(h+1)*dh-1 of each third.

Fig. 5(a) of the paper lists what a backward task needs: output
grad dY, stashed input X, weight W.  `*_fwd` therefore returns a cache of the
op inputs (the "stash"), and `*_bwd` consumes exactly that cache.
"""
from __future__ import annotations

import numpy as np

LN_EPS = 1e-5                   # reading c10
GELU_C = np.sqrt(2.0 / np.pi)   # reading c12 (tanh approximation, GPT-2)
GELU_A = 0.044715


# ----------------------------------------------------------------------------- linear
def linear_fwd(X, W, b):
    """Y = X.W + b (reading c1; canonical layout W[d_in][d_out])."""
    return X @ W + b


def linear_bwd(dY, X, W):
    """dX = dY.W^T, dW = X^T.dY, db = sum_rows dY."""
    return dY @ W.T, X.T @ dY, dY.sum(axis=0)


# ----------------------------------------------------------------------------- activations
def relu(x):
    return np.maximum(x, 0.0)


def relu_grad(x):
    return (x > 0.0).astype(x.dtype)


def gelu_tanh(x):
    """0.5 x (1 + tanh(sqrt(2/pi)(x + 0.044715 x^3)))  (reading c12)."""
    return 0.5 * x * (1.0 + np.tanh(GELU_C * (x + GELU_A * x ** 3)))


def gelu_tanh_grad(x):
    """d/dx gelu_tanh = 0.5(1 + tanh u) + 0.5 x (1 - tanh^2 u) sqrt(2/pi)(1 + 3*0.044715 x^2)."""
    u = GELU_C * (x + GELU_A * x ** 3)
    t = np.tanh(u)
    return 0.5 * (1.0 + t) + 0.5 * x * (1.0 - t * t) * GELU_C * (1.0 + 3.0 * GELU_A * x * x)


def act_fwd(act, z):
    if act == 0:
        return z
    if act == 1:
        return relu(z)
    if act == 2:
        return gelu_tanh(z)
    raise ValueError(act)


def act_grad(act, z):
    if act == 0:
        return np.ones_like(z)
    if act == 1:
        return relu_grad(z)
    if act == 2:
        return gelu_tanh_grad(z)
    raise ValueError(act)


# ----------------------------------------------------------------------------- layernorm
def layernorm_fwd(x, g, b, eps=LN_EPS):
    """Row-wise LN over the last axis: biased variance, eps inside the sqrt (reading c10).

    Returns (y, cache) with cache = (xhat, rstd, g)."""
    mu = x.mean(axis=-1, keepdims=True)
    xc = x - mu
    var = (xc * xc).mean(axis=-1, keepdims=True)
    rstd = 1.0 / np.sqrt(var + eps)
    xhat = xc * rstd
    return xhat * g + b, (xhat, rstd, g)


def layernorm_bwd(dy, cache):
    """dxhat = dy.g; dx = rstd (dxhat - mean(dxhat) - xhat mean(dxhat xhat)); dg = sum dy xhat; db = sum dy."""
    xhat, rstd, g = cache
    dxhat = dy * g
    dx = rstd * (dxhat - dxhat.mean(axis=-1, keepdims=True) - xhat * (dxhat * xhat).mean(axis=-1, keepdims=True))
    red = tuple(range(dy.ndim - 1))
    return dx, (dy * xhat).sum(axis=red), dy.sum(axis=red)


# ----------------------------------------------------------------------------- softmax
def softmax_fwd(z):
    """Row softmax; subtracting the row max is math-neutral (reading c11); -inf entries give exactly 0."""
    zmax = z.max(axis=-1, keepdims=True)
    e = np.exp(z - zmax)
    return e / e.sum(axis=-1, keepdims=True)


def softmax_bwd(dp, p):
    """dZ = P .* (dP - rowsum(dP .* P))."""
    return p * (dp - (dp * p).sum(axis=-1, keepdims=True))


# ----------------------------------------------------------------------------- attention
def _split_heads(M, B, S, h):
    """[B*S, h*dh] -> [B, h, S, dh]."""
    dh = M.shape[1] // h
    return M.reshape(B, S, h, dh).transpose(0, 2, 1, 3)


def _merge_heads(M):
    B, h, S, dh = M.shape
    return M.transpose(0, 2, 1, 3).reshape(B * S, h * dh)


def attention_fwd(qkv, B, S, h, causal):
    """Multi-head scaled dot-product attention on packed QKV [B*S, 3d].

    Z = Q_h K_h^T / sqrt(dh) (+ -inf above the diagonal if causal), P = softmax(Z), C_h = P V_h,
    heads merged back to [B*S, d] (reading c11)."""
    d = qkv.shape[1] // 3
    dh = d // h
    Q = _split_heads(qkv[:, :d], B, S, h)
    K = _split_heads(qkv[:, d:2 * d], B, S, h)
    V = _split_heads(qkv[:, 2 * d:], B, S, h)
    scale = 1.0 / np.sqrt(dh)
    Z = np.einsum("bhqe,bhke->bhqk", Q, K) * scale
    if causal:
        mask = np.triu(np.ones((S, S), dtype=bool), k=1)
        Z = np.where(mask, -np.inf, Z)
    P = softmax_fwd(Z)
    C = np.einsum("bhqk,bhke->bhqe", P, V)
    return _merge_heads(C), (Q, K, V, P, scale)


def attention_bwd(dC, cache):
    """dP = dC V^T, dV = P^T dC, dZ = P.(dP - rowsum(dP.P)), dQ = dZ K/sqrt(dh), dK = dZ^T Q/sqrt(dh).

    Returns dQKV [B*S, 3d] in the packed [Q | K | V] column layout."""
    Q, K, V, P, scale = cache
    B, h, S, dh = Q.shape
    dCh = _split_heads(dC, B, S, h)
    dP = np.einsum("bhqe,bhke->bhqk", dCh, V)
    dV = np.einsum("bhqk,bhqe->bhke", P, dCh)
    dZ = softmax_bwd(dP, P)
    dQ = np.einsum("bhqk,bhke->bhqe", dZ, K) * scale
    dK = np.einsum("bhqk,bhqe->bhke", dZ, Q) * scale
    return np.concatenate([_merge_heads(dQ), _merge_heads(dK), _merge_heads(dV)], axis=1)


# ----------------------------------------------------------------------------- transformer block
def transformer_block_fwd(X, p, B, S, h, causal):
    """Pre-LN block (reading c1), X: [B*S, d].

      U = LN1(X); QKV = U W_qkv + b_qkv; C = MHA(QKV); X2 = X + C W_o + b_o;
      U2 = LN2(X2); H = U2 W_fc1 + b_fc1; G = GeLU(H); Y = X2 + G W_fc2 + b_fc2.
    """
    U, ln1 = layernorm_fwd(X, p["ln1_g"], p["ln1_b"])
    QKV = linear_fwd(U, p["w_qkv"], p["b_qkv"])
    C, att = attention_fwd(QKV, B, S, h, causal)
    X2 = X + linear_fwd(C, p["w_o"], p["b_o"])
    U2, ln2 = layernorm_fwd(X2, p["ln2_g"], p["ln2_b"])
    H = linear_fwd(U2, p["w_fc1"], p["b_fc1"])
    G = gelu_tanh(H)
    Y = X2 + linear_fwd(G, p["w_fc2"], p["b_fc2"])
    return Y, dict(U=U, ln1=ln1, C=C, att=att, U2=U2, ln2=ln2, H=H, G=G)


def transformer_block_bwd(dY, cache, p):
    """Manual backward of transformer_block_fwd; residual gradients add. Returns dX and a grads dict."""
    g = {}
    dX2 = dY.copy()
    dG, g["w_fc2"], g["b_fc2"] = linear_bwd(dY, cache["G"], p["w_fc2"])
    dH = dG * gelu_tanh_grad(cache["H"])
    dU2, g["w_fc1"], g["b_fc1"] = linear_bwd(dH, cache["U2"], p["w_fc1"])
    dX2_ln, g["ln2_g"], g["ln2_b"] = layernorm_bwd(dU2, cache["ln2"])
    dX2 = dX2 + dX2_ln
    dC, g["w_o"], g["b_o"] = linear_bwd(dX2, cache["C"], p["w_o"])
    dQKV = attention_bwd(dC, cache["att"])
    dU, g["w_qkv"], g["b_qkv"] = linear_bwd(dQKV, cache["U"], p["w_qkv"])
    dX_ln, g["ln1_g"], g["ln1_b"] = layernorm_bwd(dU, cache["ln1"])
    return dX2 + dX_ln, g


# ----------------------------------------------------------------------------- MLP layer
def mlp_layer_fwd(X, p, act):
    """Y = act(X W + b) (reading c1)."""
    Z = linear_fwd(X, p["w"], p["b"])
    return act_fwd(act, Z), dict(X=X, Z=Z)


def mlp_layer_bwd(dY, cache, p, act):
    dZ = dY * act_grad(act, cache["Z"])
    dX, dW, db = linear_bwd(dZ, cache["X"], p["w"])
    return dX, {"w": dW, "b": db}
