"""The plain single-device training step (oracle; test infrastructure only).

PAPER.md P:129-136 / P:573-575: users write the model "as if running
sequentially on a single device", and Harmony adds collectives "to preserve the
semantics of the original tasks".  The reference result is therefore one
full-batch step: forward through every layer, loss, backward, Adam.  Readings
(DESIGN.md): c2 loss = (1/B) sum_b 1/2 ||Y_b - T_b||^2 over the GLOBAL batch;
c3 Adam with bias correction, eps outside the sqrt, t from 1; c4 the update of
layer l may run right after its backward ("JIT") because no weight
is read after its own backward.
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

from synth import LAYER_MLP, unpack, pack, segments
from .layers import transformer_block_fwd, transformer_block_bwd, mlp_layer_fwd, mlp_layer_bwd


def _as_rows(X, desc):
    """[B, S, d] -> [B*S, d] for transformer stacks; MLP input is already [B, d]."""
    return X.reshape(-1, X.shape[-1])


def stack_forward(descs, params, X):
    """Forward through the stack. params: list of flat fp64 vectors (canonical packing)."""
    B = X.shape[0]
    A = _as_rows(np.asarray(X, dtype=np.float64), descs[0])
    caches = []
    for desc, flat in zip(descs, params):
        p = unpack(desc, np.asarray(flat, dtype=np.float64))
        if desc.kind == LAYER_MLP:
            A, c = mlp_layer_fwd(A, p, desc.act)
        else:
            A, c = transformer_block_fwd(A, p, B, desc.seq_len, desc.n_heads, bool(desc.causal))
        caches.append((p, c))
    return A, caches


def mse_loss(Y, T, B):
    """L = (1/B) sum_b 1/2 ||Y_b - T_b||_F^2 and dL/dY = (Y - T)/B (reading c2)."""
    D = Y - T.reshape(Y.shape)
    return 0.5 * float(np.sum(D * D)) / B, D / B


def stack_loss_and_grads(descs, params, X, T, loss_batch=None):
    """Loss and per-layer flat gradients.  loss_batch = the B of the 1/B scaling
    (defaults to X.shape[0]; a microbatch passes the global B, reading c2)."""
    B = X.shape[0] if loss_batch is None else loss_batch
    Y, caches = stack_forward(descs, params, X)
    loss, dA = mse_loss(Y, np.asarray(T, dtype=np.float64), B)
    grads = [None] * len(descs)
    for li in range(len(descs) - 1, -1, -1):
        desc = descs[li]
        p, c = caches[li]
        if desc.kind == LAYER_MLP:
            dA, g = mlp_layer_bwd(dA, c, p, desc.act)
        else:
            dA, g = transformer_block_bwd(dA, c, p)
        grads[li] = pack(desc, g)
    return loss, grads, Y


@dataclass
class AdamState:
    m: list = field(default_factory=list)
    v: list = field(default_factory=list)
    t: int = 0

    @staticmethod
    def zeros(params):
        return AdamState([np.zeros_like(np.asarray(p, np.float64)) for p in params],
                         [np.zeros_like(np.asarray(p, np.float64)) for p in params], 0)


def adam_update(W, g, m, v, t, lr, beta1, beta2, eps):
    """Kingma & Ba [30], Algorithm 1, one step at time t >= 1:
       m = b1 m + (1-b1) g;  v = b2 v + (1-b2) g^2;  mh = m/(1-b1^t);  vh = v/(1-b2^t);
       W = W - lr mh / (sqrt(vh) + eps)."""
    m = beta1 * m + (1.0 - beta1) * g
    v = beta2 * v + (1.0 - beta2) * g * g
    mh = m / (1.0 - beta1 ** t)
    vh = v / (1.0 - beta2 ** t)
    return W - lr * mh / (np.sqrt(vh) + eps), m, v


def train_step(descs, params, state: AdamState, X, T, lr=1e-3, beta1=0.9, beta2=0.999, eps=1e-8):
    """One full-batch step. Returns (loss, grads, new_params, new_state)."""
    loss, grads, _ = stack_loss_and_grads(descs, params, X, T)
    t = state.t + 1
    new_p, new_m, new_v = [], [], []
    for W, g, m, v in zip(params, grads, state.m, state.v):
        W2, m2, v2 = adam_update(np.asarray(W, np.float64), g, m, v, t, lr, beta1, beta2, eps)
        new_p.append(W2), new_m.append(m2), new_v.append(v2)
    return loss, grads, new_p, AdamState(new_m, new_v, t)


def n_params(descs):
    return sum(int(np.prod(s)) for d in descs for _, s in segments(d))
