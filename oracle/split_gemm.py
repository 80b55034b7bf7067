"""Operator decomposition of one GEMM fwd+bwd (oracle; test infrastructure only).

PAPER.md P:137-138: Harmony can "further decompose individual operations—such
as a matrix multiplication—into subtasks that can run on different physical
devices".  cfg5 (BASELINE.json configs[4]) is a single M x N x K GEMM with its
backward; reading c19: X [M,K], W [K,N], Y = X.W [M,N], dY given,
dX = dY.W^T, dW = X^T.dY.
"""
from __future__ import annotations

import numpy as np


def gemm_fwd_bwd(X, W, dY):
    """The plain (undecomposed) definition, fp64."""
    X = np.asarray(X, np.float64); W = np.asarray(W, np.float64); dY = np.asarray(dY, np.float64)
    return X @ W, dY @ W.T, X.T @ dY


def split_gemm_fwd_bwd(X, W, dY, n_k_splits=1, m_tiles=1, n_tiles=1):
    """The decomposed GEMM: K split into n_k_splits contiguous slices (one per device, the
    partial products summed = the reduce-scatter's sum), and the output cut into m_tiles x n_tiles
    tiles (tile subtasks).  dX and dW come out per K slice, locally, then are concatenated.
    Equal to gemm_fwd_bwd by the block-matrix identity (self-check ii)."""
    X = np.asarray(X, np.float64); W = np.asarray(W, np.float64); dY = np.asarray(dY, np.float64)
    M, K = X.shape
    N = W.shape[1]
    kb = np.linspace(0, K, n_k_splits + 1).astype(int)
    mb = np.linspace(0, M, m_tiles + 1).astype(int)
    nb = np.linspace(0, N, n_tiles + 1).astype(int)
    Y = np.zeros((M, N))
    for i in range(m_tiles):
        for j in range(n_tiles):
            acc = np.zeros((mb[i + 1] - mb[i], nb[j + 1] - nb[j]))
            for r in range(n_k_splits):
                acc += X[mb[i]:mb[i + 1], kb[r]:kb[r + 1]] @ W[kb[r]:kb[r + 1], nb[j]:nb[j + 1]]
            Y[mb[i]:mb[i + 1], nb[j]:nb[j + 1]] = acc
    dX = np.concatenate([dY @ W[kb[r]:kb[r + 1], :].T for r in range(n_k_splits)], axis=1)
    dW = np.concatenate([X[:, kb[r]:kb[r + 1]].T @ dY for r in range(n_k_splits)], axis=0)
    return Y, dX, dW


def sampled_gemm_entries(X, W, dY, rows, cols, which):
    """Single entries of Y, dX or dW as fp64 dot products (for full-size sampled checks).
    which = 'Y': Y[r,c] = sum_k X[r,k] W[k,c];  'dX': dX[r,c] = sum_n dY[r,n] W[c,n];
    'dW': dW[r,c] = sum_m X[m,r] dY[m,c]."""
    out = np.empty(len(rows))
    for i, (r, c) in enumerate(zip(rows, cols)):
        if which == "Y":
            out[i] = np.dot(np.asarray(X[r, :], np.float64), np.asarray(W[:, c], np.float64))
        elif which == "dX":
            out[i] = np.dot(np.asarray(dY[r, :], np.float64), np.asarray(W[c, :], np.float64))
        elif which == "dW":
            out[i] = np.dot(np.asarray(X[:, r], np.float64), np.asarray(dY[:, c], np.float64))
        else:
            raise ValueError(which)
    return out
