"""Kernel-level parity on a B200: each kernel of the step, called through the C ABI
(include/harmony_kernels.h), against the fp64 oracle's definition of the same op on the same
seeded inputs.  Shapes span several tiles and ragged tails."""
import ctypes as C

import numpy as np
import pytest

import oracle
from oracle import layers as OL
from synth import bf16_exact

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
from paper_conf_hotos_lipmk21_b200 import harmony as H  # noqa: E402


def rel(a, b):
    a = np.asarray(a, np.float64); b = np.asarray(b, np.float64)
    return np.linalg.norm(a - b) / max(np.linalg.norm(b), 1e-30)


_KEEP = []  # keep device buffers alive until the asynchronous kernels that read them are done


def dev(a, dtype):
    t = torch.tensor(np.asarray(a, np.float32), device="cuda").to(dtype).contiguous()
    _KEEP.append(t)
    if len(_KEEP) > 64:
        torch.cuda.synchronize()
        del _KEEP[:32]
    return t


def host(t):
    return t.float().cpu().numpy().astype(np.float64)


def gemm(args):
    H.hk("hk_gemm", C.byref(args), None)
    H.hk("hk_sync")


def mk(dtype, M, N, K, A, amn, lda, B, bmn, ldb, Cout, ldc, epi, **kw):
    a = H.hk_gemm_args()
    a.dtype, a.M, a.N, a.K, a.nz0, a.nz1 = dtype, M, N, K, kw.get("nz0", 1), kw.get("nz1", 1)
    a.A, a.a_mn_major, a.lda = A.data_ptr(), amn, lda
    a.a_sz0, a.a_sz1 = kw.get("a_sz0", 0), kw.get("a_sz1", 0)
    a.B, a.b_mn_major, a.ldb = B.data_ptr(), bmn, ldb
    a.b_sz0, a.b_sz1 = kw.get("b_sz0", 0), kw.get("b_sz1", 0)
    a.C, a.ldc = Cout.data_ptr(), ldc
    a.c_sz0, a.c_sz1 = kw.get("c_sz0", 0), kw.get("c_sz1", 0)
    a.epilogue, a.act, a.accumulate, a.alpha = epi, kw.get("act", 0), kw.get("accumulate", 0), kw.get("alpha", 1.0)
    a.bias = kw["bias"].data_ptr() if "bias" in kw else None
    a.aux = kw["aux"].data_ptr() if "aux" in kw else None
    a.aux_out = kw["aux_out"].data_ptr() if "aux_out" in kw else None
    return a


def operand(rng, rows, K, mn_major, dtype):
    """Logical [rows, K] operand stored K-major ([rows][K]) or MN-major ([K][rows])."""
    X = bf16_exact(rng.standard_normal((rows, K)).astype(np.float32))
    store = X.T.copy() if mn_major else X
    return X, dev(store, dtype), (rows if mn_major else K)


@pytest.mark.parametrize("amn,bmn", [(0, 0), (0, 1), (1, 0), (1, 1)])
@pytest.mark.parametrize("M,N,K", [(128, 128, 64), (200, 136, 104), (384, 520, 1000), (64, 40, 24), (1, 8, 8)])
def test_gemm_bf16_tcgen05_majors_and_tails(amn, bmn, M, N, K):
    if (M if amn else K) % 8 or (N if bmn else K) % 8:
        pytest.skip("TMA needs 16-byte row strides (ld % 8 == 0)")
    rng = np.random.default_rng(M * 7 + N * 3 + K + amn * 2 + bmn)
    A, Ad, lda = operand(rng, M, K, amn, torch.bfloat16)
    B, Bd, ldb = operand(rng, N, K, bmn, torch.bfloat16)
    Cd = torch.zeros(M, N, device="cuda")
    gemm(mk(1, M, N, K, Ad, amn, lda, Bd, bmn, ldb, Cd, N, H.HK_EPI_STORE_F32))
    ref = A.astype(np.float64) @ B.astype(np.float64).T
    assert rel(host(Cd), ref) < 2e-6  # fp32 accumulation of exact bf16 products


@pytest.mark.parametrize("amn,bmn", [(0, 0), (1, 1), (0, 1)])
def test_gemm_fp32_simt(amn, bmn):
    rng = np.random.default_rng(5)
    M, N, K = 150, 70, 90
    A = rng.standard_normal((M, K)).astype(np.float32); B = rng.standard_normal((N, K)).astype(np.float32)
    Ad = dev(A.T.copy() if amn else A, torch.float32); Bd = dev(B.T.copy() if bmn else B, torch.float32)
    Cd = torch.zeros(M, N, device="cuda")
    gemm(mk(0, M, N, K, Ad, amn, M if amn else K, Bd, bmn, N if bmn else K, Cd, N, H.HK_EPI_STORE_F32))
    assert rel(host(Cd), A.astype(np.float64) @ B.astype(np.float64).T) < 1e-6


@pytest.mark.parametrize("dtype", [0, 1])
def test_gemm_epilogues(dtype):
    tdt = torch.bfloat16 if dtype else torch.float32
    rng = np.random.default_rng(9)
    M, N, K = 136, 200, 72
    A, Ad, lda = operand(rng, M, K, 0, tdt)
    B, Bd, ldb = operand(rng, N, K, 1, tdt)
    acc = A.astype(np.float64) @ B.astype(np.float64).T
    bias = bf16_exact(rng.standard_normal(N).astype(np.float32)); bd = dev(bias, tdt)
    tol = 1e-2 if dtype else 1e-5
    # bias + GeLU (FC1): z and act(z)
    Z = torch.zeros(M, N, device="cuda", dtype=tdt); G = torch.zeros_like(Z)
    gemm(mk(dtype, M, N, K, Ad, 0, lda, Bd, 1, ldb, Z, N, H.HK_EPI_BIAS_ACT, act=2, bias=bd, aux_out=G))
    assert rel(host(Z), acc + bias) < tol and rel(host(G), OL.gelu_tanh(acc + bias)) < tol
    # residual add into fp32
    R = rng.standard_normal((M, N)).astype(np.float32); Rd = dev(R, torch.float32)
    O = torch.zeros(M, N, device="cuda")
    gemm(mk(dtype, M, N, K, Ad, 0, lda, Bd, 1, ldb, O, N, H.HK_EPI_RESID_F32, bias=bd, aux=Rd))
    assert rel(host(O), R + acc + bias) < 1e-6
    # accumulate (wgrad): write then add
    W = torch.full((M, N), 7.0, device="cuda")
    gemm(mk(dtype, M, N, K, Ad, 0, lda, Bd, 1, ldb, W, N, H.HK_EPI_ACC_F32, accumulate=0))
    gemm(mk(dtype, M, N, K, Ad, 0, lda, Bd, 1, ldb, W, N, H.HK_EPI_ACC_F32, accumulate=1, alpha=0.5))
    assert rel(host(W), 1.5 * acc) < 1e-6
    # activation backward (dG -> dH)
    Hh = bf16_exact(rng.standard_normal((M, N)).astype(np.float32)); Hd = dev(Hh, tdt)
    D = torch.zeros(M, N, device="cuda", dtype=tdt)
    gemm(mk(dtype, M, N, K, Ad, 0, lda, Bd, 1, ldb, D, N, H.HK_EPI_ACT_BWD, act=2, aux=Hd))
    assert rel(host(D), acc * OL.gelu_tanh_grad(Hh.astype(np.float64))) < tol
    # plain store with alpha
    S = torch.zeros(M, N, device="cuda", dtype=tdt)
    gemm(mk(dtype, M, N, K, Ad, 0, lda, Bd, 1, ldb, S, N, H.HK_EPI_STORE_T, alpha=0.25))
    assert rel(host(S), 0.25 * acc) < tol


@pytest.mark.parametrize("dtype", [0, 1])
@pytest.mark.parametrize("S,dh,h,b", [(136, 40, 3, 2), (256, 64, 2, 1)])
def test_batched_attention_gemms_on_packed_qkv(dtype, S, dh, h, b):
    """Z = Q_h K_h^T on the packed [T, 3d] QKV layout (strided batch over heads and sequences),
    C_h = P V_h written head-interleaved into [T, d]  (the forward's two batched contractions)."""
    tdt = torch.bfloat16 if dtype else torch.float32
    d = h * dh
    rng = np.random.default_rng(S + dh)
    qkv = bf16_exact(rng.standard_normal((b * S, 3 * d)).astype(np.float32))
    Qd = dev(qkv, tdt)
    Z = torch.zeros(b, h, S, S, device="cuda")
    esz = 2 if dtype else 4
    a = mk(dtype, S, S, dh, Qd, 0, 3 * d, Qd, 0, 3 * d, Z, S, H.HK_EPI_STORE_F32, nz0=h, nz1=b,
           a_sz0=dh, a_sz1=S * 3 * d, b_sz0=dh, b_sz1=S * 3 * d, c_sz0=S * S, c_sz1=h * S * S)
    a.B = Qd.data_ptr() + d * esz
    gemm(a)
    Q = qkv[:, :d].reshape(b, S, h, dh).transpose(0, 2, 1, 3).astype(np.float64)
    K = qkv[:, d:2 * d].reshape(b, S, h, dh).transpose(0, 2, 1, 3).astype(np.float64)
    V = qkv[:, 2 * d:].reshape(b, S, h, dh).transpose(0, 2, 1, 3).astype(np.float64)
    assert rel(host(Z), np.einsum("bhqe,bhke->bhqk", Q, K)) < 1e-5
    P = bf16_exact(rng.random((b, h, S, S)).astype(np.float32))
    Pd = dev(P, tdt)
    Cd = torch.zeros(b * S, d, device="cuda")
    a = mk(dtype, S, dh, S, Pd, 0, S, Qd, 1, 3 * d, Cd, d, H.HK_EPI_STORE_F32, nz0=h, nz1=b,
           a_sz0=S * S, a_sz1=h * S * S, b_sz0=dh, b_sz1=S * 3 * d, c_sz0=dh, c_sz1=S * d)
    a.B = Qd.data_ptr() + 2 * d * esz
    gemm(a)
    ref = np.einsum("bhqk,bhke->bhqe", P.astype(np.float64), V).transpose(0, 2, 1, 3).reshape(b * S, d)
    assert rel(host(Cd), ref) < 1e-5


@pytest.mark.parametrize("dtype", [0, 1])
@pytest.mark.parametrize("rows,d", [(37, 64), (300, 1024), (5, 1600)])
def test_layernorm_fwd_bwd(dtype, rows, d):
    tdt = torch.bfloat16 if dtype else torch.float32
    rng = np.random.default_rng(rows + d)
    X = (rng.standard_normal((rows, d)) * 2 + 0.5).astype(np.float32)
    g = bf16_exact((1 + 0.1 * rng.standard_normal(d)).astype(np.float32)); bb = bf16_exact(0.1 * rng.standard_normal(d).astype(np.float32))
    U = torch.zeros(rows, d, device="cuda", dtype=tdt)
    mean = torch.zeros(rows, device="cuda"); rstd = torch.zeros(rows, device="cuda")
    Xd = dev(X, torch.float32)
    H.hk("hk_layernorm_fwd", dtype, rows, d, Xd.data_ptr(), dev(g, tdt).data_ptr(), dev(bb, tdt).data_ptr(),
         U.data_ptr(), mean.data_ptr(), rstd.data_ptr(), None)
    H.hk("hk_sync")
    ref, cache = OL.layernorm_fwd(X.astype(np.float64), g.astype(np.float64), bb.astype(np.float64))
    assert rel(host(U), ref) < (4e-3 if dtype else 1e-6)
    dU = rng.standard_normal((rows, d)).astype(np.float32)
    dres = rng.standard_normal((rows, d)).astype(np.float32)
    dX = torch.zeros(rows, d, device="cuda")
    dg = torch.full((d,), 1.0, device="cuda"); db = torch.full((d,), 2.0, device="cuda")
    H.hk("hk_layernorm_bwd", dtype, rows, d, dev(dU, torch.float32).data_ptr(), Xd.data_ptr(), mean.data_ptr(),
         rstd.data_ptr(), dev(g, tdt).data_ptr(), dev(dres, torch.float32).data_ptr(), dX.data_ptr(), dg.data_ptr(),
         db.data_ptr(), 1, None)
    rdx, rdg, rdb = OL.layernorm_bwd(dU.astype(np.float64), cache)
    assert rel(host(dX), rdx + dres) < 1e-5
    assert rel(host(dg), 1.0 + rdg) < 1e-5 and rel(host(db), 2.0 + rdb) < 1e-5


@pytest.mark.parametrize("dtype", [0, 1])
@pytest.mark.parametrize("causal", [0, 1])
def test_softmax_fwd_bwd(dtype, causal):
    tdt = torch.bfloat16 if dtype else torch.float32
    S, nrows = 136, 3 * 136
    rng = np.random.default_rng(3 + causal)
    Z = (rng.standard_normal((nrows, S)) * 3).astype(np.float32)
    scale = 0.125
    P = torch.zeros(nrows, S, device="cuda", dtype=tdt)
    H.hk("hk_softmax_fwd", dtype, nrows, S, causal, scale, dev(Z, torch.float32).data_ptr(), P.data_ptr(), None)
    H.hk("hk_sync")
    Zs = Z.astype(np.float64).reshape(-1, S, S) * scale
    if causal:
        Zs = np.where(np.triu(np.ones((S, S), bool), 1), -np.inf, Zs)
    ref = OL.softmax_fwd(Zs).reshape(nrows, S)
    assert rel(host(P), ref) < (4e-3 if dtype else 1e-6)
    if causal:
        assert np.all(host(P).reshape(-1, S, S)[:, np.triu(np.ones((S, S), bool), 1)] == 0)
    dP = rng.standard_normal((nrows, S)).astype(np.float32)
    dZ = torch.zeros(nrows, S, device="cuda", dtype=tdt)
    H.hk("hk_softmax_bwd", dtype, nrows, S, scale, dev(dP, torch.float32).data_ptr(), P.data_ptr(), dZ.data_ptr(), None)
    H.hk("hk_sync")
    assert rel(host(dZ), scale * OL.softmax_bwd(dP.astype(np.float64), host(P))) < (4e-3 if dtype else 1e-6)


@pytest.mark.parametrize("dtype", [0, 1])
def test_adam_matches_oracle(dtype):
    rng = np.random.default_rng(4)
    n = 10007
    W = rng.standard_normal(n).astype(np.float32); m = (0.01 * rng.standard_normal(n)).astype(np.float32)
    v = (0.001 * rng.random(n)).astype(np.float32); g = rng.standard_normal(n).astype(np.float32)
    Wd, md, vd, gd = (dev(x, torch.float32) for x in (W, m, v, g))
    Wc = torch.zeros(n, device="cuda", dtype=torch.bfloat16 if dtype else torch.float32)
    H.hk("hk_adam", dtype, n, Wd.data_ptr(), md.data_ptr(), vd.data_ptr(), gd.data_ptr(), Wc.data_ptr(),
         1e-3, 0.9, 0.999, 1e-8, 3, None)
    H.hk("hk_sync")
    W2, m2, v2 = oracle.adam_update(W.astype(np.float64), g.astype(np.float64), m.astype(np.float64),
                                    v.astype(np.float64), 3, 1e-3, 0.9, 0.999, 1e-8)
    assert rel(host(Wd), W2) < 1e-6 and rel(host(md), m2) < 1e-6 and rel(host(vd), v2) < 1e-6
    assert rel(host(Wc), W2) < (4e-3 if dtype else 1e-6)


def test_mse_and_colsum():
    rng = np.random.default_rng(1)
    n = 4 * 1000 + 3
    Y = rng.standard_normal(n).astype(np.float32); T = rng.standard_normal(n).astype(np.float32)
    dY = torch.zeros(n, device="cuda"); loss = torch.zeros(1, dtype=torch.float64, device="cuda")
    H.hk("hk_mse", n, dev(Y, torch.float32).data_ptr(), dev(T, torch.float32).data_ptr(), 1 / 8, dY.data_ptr(),
         loss.data_ptr(), None)
    l_ref, d_ref = oracle.mse_loss(Y.astype(np.float64), T.astype(np.float64), 8)
    assert abs(loss.item() - l_ref) < 1e-9 * l_ref and rel(host(dY), d_ref) < 1e-7
    X = rng.standard_normal((777, 300)).astype(np.float32)
    out = torch.zeros(300, device="cuda")
    H.hk("hk_colsum", 0, 777, 300, dev(X, torch.float32).data_ptr(), 300, out.data_ptr(), 0, None)
    assert rel(host(out), X.astype(np.float64).sum(0)) < 1e-6


@pytest.mark.parametrize("S,dh,h,b,causal", [(128, 64, 2, 1, 0), (256, 64, 3, 2, 1), (512, 64, 2, 1, 0),
                                             (384, 128, 2, 1, 1), (1024, 64, 1, 1, 1)])
def test_fused_attention_forward(S, dh, h, b, causal):
    """softmax(Q K^T / sqrt(dh)) V per head without materialising the scores (scores in TMEM, P in
    shared memory), vs the oracle's attention on the same packed QKV; LSE vs the fp64 log-sum-exp."""
    d = h * dh
    rng = np.random.default_rng(S + dh + causal)
    qkv = bf16_exact((rng.standard_normal((b * S, 3 * d)) * 1.5).astype(np.float32))
    Qd = dev(qkv, torch.bfloat16)
    C_ = torch.zeros(b * S, d, device="cuda", dtype=torch.bfloat16)
    lse = torch.zeros(b, h, S, device="cuda")
    H.hk("hk_attention_fwd", b, S, h, dh, causal, Qd.data_ptr(), C_.data_ptr(), lse.data_ptr(), None)
    H.hk("hk_sync")
    ref, (Q, K, V, P, scale) = OL.attention_fwd(qkv.astype(np.float64), b, S, h, bool(causal))
    assert rel(host(C_), ref) < 1e-2
    Z = np.einsum("bhqe,bhke->bhqk", Q, K) * scale
    if causal:
        Z = np.where(np.triu(np.ones((S, S), bool), 1), -np.inf, Z)
    zmax = Z.max(-1, keepdims=True)
    lse_ref = (zmax + np.log(np.exp(Z - zmax).sum(-1, keepdims=True)))[..., 0]
    assert np.max(np.abs(host(lse) - lse_ref)) < 2e-3


@pytest.mark.parametrize("S,dh,h,b,causal", [(128, 64, 2, 1, 0), (256, 64, 2, 2, 1), (512, 64, 2, 1, 0),
                                             (384, 128, 2, 1, 1), (512, 64, 1, 1, 1),
                                             # more (key tile, head, sequence) items than SMs: every
                                             # pipeline counter of the persistent kernel wraps across items
                                             (512, 64, 16, 4, 0), (512, 64, 16, 4, 1)])
def test_fused_attention_backward(S, dh, h, b, causal):
    """dQKV of the fused backward (S^T, dP^T in TMEM; P^T, dS^T in smem; dQ by GEMM on dS^T) vs the
    oracle's attention_bwd on the same inputs."""
    d = h * dh
    rng = np.random.default_rng(7 * S + dh + causal)
    qkv = bf16_exact((rng.standard_normal((b * S, 3 * d)) * 1.5).astype(np.float32))
    dC = bf16_exact(rng.standard_normal((b * S, d)).astype(np.float32))
    Qd = dev(qkv, torch.bfloat16); dCd = dev(dC, torch.bfloat16)
    C_ = torch.zeros(b * S, d, device="cuda", dtype=torch.bfloat16)
    lse = torch.zeros(b, h, S, device="cuda")
    H.hk("hk_attention_fwd", b, S, h, dh, causal, Qd.data_ptr(), C_.data_ptr(), lse.data_ptr(), None)
    dQKV = torch.zeros(b * S, 3 * d, device="cuda", dtype=torch.bfloat16)
    H.hk("hk_attention_bwd", b, S, h, dh, causal, Qd.data_ptr(), C_.data_ptr(), dCd.data_ptr(), lse.data_ptr(),
         dQKV.data_ptr(), None)
    H.hk("hk_sync")
    _, cache = OL.attention_fwd(qkv.astype(np.float64), b, S, h, bool(causal))
    ref = OL.attention_bwd(dC.astype(np.float64), cache)
    got = host(dQKV)
    for part, sl in (("dQ", slice(0, d)), ("dK", slice(d, 2 * d)), ("dV", slice(2 * d, 3 * d))):
        assert rel(got[:, sl], ref[:, sl]) < 2e-2, part
