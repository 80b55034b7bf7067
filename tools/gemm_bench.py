"""Time the step's GEMMs (cfg2: one microbatch of T tokens, d = 1024 — T = 16384 for the bench's
m=2 x b=32, --tokens to change; the 12 linear GEMMs of a transformer layer with their in-step
epilogues) through hk_gemm.

    python tools/gemm_bench.py [--reps 20] [--only NAME]

Each shape is timed with CUDA events on the launching stream (warm-up first); prints one JSON
line per shape with TFLOP/s and, for ncu, keeps launches back to back.
"""
import argparse
import ctypes as C
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_hotos_lipmk21_b200 import harmony as H  # noqa: E402

T, D, S, B, NH = int(os.environ.get("GEMM_BENCH_TOKENS", "16384")), int(os.environ.get("GEMM_BENCH_D", "1024")), 512, 8, 16
DH = D // NH


def shapes():
    bf = torch.bfloat16
    x = torch.randn(T, 4 * D, device="cuda").to(bf)
    w = torch.randn(4 * D, 4 * D, device="cuda").to(bf) * 0.02
    qkv = torch.randn(T, 3 * D, device="cuda").to(bf)
    p = torch.rand(B * NH * S * S, device="cuda").to(bf)
    c32 = torch.zeros(max(T * 4 * D, B * NH * S * S), device="cuda")
    c16 = torch.zeros(T * 4 * D, device="cuda", dtype=bf)
    out = []

    def g(name, M, N, K, A, amn, lda, Bm, bmn, ldb, Cm, ldc, epi, **kw):
        a = H.hk_gemm_args()
        a.dtype, a.M, a.N, a.K, a.nz0, a.nz1 = 1, M, N, K, kw.get("nz0", 1), kw.get("nz1", 1)
        a.A, a.a_mn_major, a.lda, a.a_sz0, a.a_sz1 = A, amn, lda, kw.get("a_sz0", 0), kw.get("a_sz1", 0)
        a.B, a.b_mn_major, a.ldb, a.b_sz0, a.b_sz1 = Bm, bmn, ldb, kw.get("b_sz0", 0), kw.get("b_sz1", 0)
        a.C, a.ldc, a.c_sz0, a.c_sz1 = Cm, ldc, kw.get("c_sz0", 0), kw.get("c_sz1", 0)
        a.epilogue, a.alpha, a.accumulate = epi, 1.0, kw.get("acc", 0)
        a.bias, a.aux, a.aux_out, a.act = kw.get("bias"), kw.get("aux"), kw.get("aux_out"), kw.get("act", 0)
        out.append((name, a, 2.0 * M * N * K * a.nz0 * a.nz1))

    X, W, Q, P, C32, C16 = (t.data_ptr() for t in (x, w, qkv, p, c32, c16))
    bias = torch.randn(4 * D, device="cuda").to(bf)
    aux32 = torch.randn(T * D, device="cuda")
    aux16 = torch.randn(T * 4 * D, device="cuda").to(bf)
    out16 = torch.zeros(T * 4 * D, device="cuda", dtype=bf)
    keep = [bias, aux32, aux16, out16]
    BI, A32, A16, O16 = (t.data_ptr() for t in keep)

    def lin_fwd(name, n, k, C, epi, **kw):  # Y[T][n] = X[T][k] . W[k][n]
        g(name, T, n, k, X, 0, k, W, 1, n, C, n, epi, **kw)

    def lin_dgrad(name, n, k, C, epi, **kw):  # dX[T][k] = dY[T][n] . W^T
        g(name, T, k, n, X, 0, n, W, 0, n, C, k, epi, **kw)

    def lin_wgrad(name, n, k):  # dW[k][n] += X^T . dY
        g(name, k, n, T, X, 1, k, X, 1, n, C32, n, H.HK_EPI_ACC_F32, acc=1)

    # the per-microbatch GEMMs of one transformer layer, in-step epilogues (layers.cu fwd_core/bwd_core)
    lin_fwd("qkv_fwd", 3 * D, D, C16, H.HK_EPI_STORE_T, bias=BI)
    lin_fwd("out_fwd", D, D, C32, H.HK_EPI_RESID_F32, bias=BI, aux=A32)
    lin_fwd("fc1_fwd", 4 * D, D, C16, H.HK_EPI_BIAS_ACT, bias=BI, act=2, aux_out=O16)
    lin_fwd("fc2_fwd", D, 4 * D, C32, H.HK_EPI_RESID_F32, bias=BI, aux=A32)
    lin_dgrad("fc2_dgrad", D, 4 * D, C16, H.HK_EPI_ACT_BWD, act=2, aux=A16)
    lin_dgrad("fc1_dgrad", 4 * D, D, C32, H.HK_EPI_STORE_F32)
    lin_dgrad("out_dgrad", D, D, C16, H.HK_EPI_STORE_T)
    lin_dgrad("qkv_dgrad", 3 * D, D, C32, H.HK_EPI_STORE_F32)
    lin_wgrad("fc2_wgrad", D, 4 * D)
    lin_wgrad("fc1_wgrad", 4 * D, D)
    lin_wgrad("out_wgrad", D, D)
    lin_wgrad("qkv_wgrad", 3 * D, D)
    # the d x d weight gradient as the step runs it: S token slices (batched) into fp32 partials
    for S_ in (2, 4, 8):
        ks = T // S_
        g(f"out_wgrad_split{S_}", D, D, ks, X, 1, D, X, 1, D, C32, D, H.HK_EPI_STORE_F32, nz0=S_,
          a_sz0=ks * D, b_sz0=ks * D, c_sz0=D * D)
    return out, (x, w, qkv, p, c32, c16, keep)


def sweep():
    """M = 4096, N in {3072, 4096}, K in {256 .. 4096}: time = mainloop(K) + per-tile overhead."""
    bf = torch.bfloat16
    x = torch.randn(T, 4 * D, device="cuda").to(bf)
    w = torch.randn(4 * D, 4 * D, device="cuda").to(bf) * 0.02
    c16 = torch.zeros(T * 4 * D, device="cuda", dtype=bf)
    o16 = torch.zeros(T * 4 * D, device="cuda", dtype=bf)
    c32 = torch.zeros(T * 4 * D, device="cuda")
    bias = torch.randn(4 * D, device="cuda").to(bf)
    out = []
    for n in (3072, 4096):
        for k in (256, 512, 1024, 2048, 4096):
            for epi, nm in ((H.HK_EPI_STORE_T, "T"), (H.HK_EPI_STORE_F32, "F32"), (H.HK_EPI_BIAS_ACT, "BACT")):
                a = H.hk_gemm_args()
                a.dtype, a.M, a.N, a.K, a.nz0, a.nz1 = 1, T, n, k, 1, 1
                a.A, a.a_mn_major, a.lda = x.data_ptr(), 0, k
                a.B, a.b_mn_major, a.ldb = w.data_ptr(), 1, n
                a.C, a.ldc = (c32 if epi == H.HK_EPI_STORE_F32 else c16).data_ptr(), n
                a.epilogue, a.alpha, a.accumulate = epi, 1.0, 0
                a.bias, a.aux_out, a.act = bias.data_ptr(), o16.data_ptr(), 2
                out.append((f"sweep_{nm}_n{n}_k{k}", a, 2.0 * T * n * k))
    return out, (x, w, c16, o16, c32, bias)


def library_equivalent(a, A_, B_):
    """cuBLAS(Lt) + PyTorch elementwise kernels computing what hk_gemm's fused epilogue computes for
    the descriptor a (same operand majors, same output dtypes); None for batched products."""
    import torch.nn.functional as F
    bf = torch.bfloat16
    M, N = a.M, a.N
    bias = torch.randn(N, device="cuda").to(bf)
    e = a.epilogue
    if e == H.HK_EPI_STORE_T:  # bf16 Y = A B + b (cuBLASLt bias epilogue)
        out = torch.empty(M, N, device="cuda", dtype=bf)
        return lambda: torch.addmm(bias, A_, B_, out=out)
    if e == H.HK_EPI_RESID_F32:  # fp32 C = R + (A B + b)
        y = torch.empty(M, N, device="cuda", dtype=bf)
        R = torch.randn(M, N, device="cuda")
        C32 = torch.empty(M, N, device="cuda")
        return lambda: (torch.addmm(bias, A_, B_, out=y), torch.add(R, y, out=C32))
    if e == H.HK_EPI_BIAS_ACT:  # H = A B + b (bf16) and G = gelu_tanh(H) (bf16)
        Hh = torch.empty(M, N, device="cuda", dtype=bf)
        return lambda: F.gelu(torch.addmm(bias, A_, B_, out=Hh), approximate="tanh")
    if e == H.HK_EPI_ACT_BWD:  # dH = (dG W^T) * gelu'(H)
        dG = torch.empty(M, N, device="cuda", dtype=bf)
        Hs = torch.randn(M, N, device="cuda").to(bf)
        return lambda: torch.ops.aten.gelu_backward(torch.matmul(A_, B_, out=dG), Hs, approximate="tanh")
    if e in (H.HK_EPI_STORE_F32, H.HK_EPI_ACC_F32):  # fp32 output (+= for the weight gradient)
        C32 = torch.zeros(M, N, device="cuda")
        try:
            torch.mm(A_, B_, out_dtype=torch.float32)
            mm32 = lambda: torch.mm(A_, B_, out_dtype=torch.float32)  # noqa: E731
        except (TypeError, RuntimeError):
            mm32 = lambda: torch.matmul(A_, B_).float()  # noqa: E731
        if e == H.HK_EPI_STORE_F32:
            return mm32
        try:  # one cuBLAS call with beta = 1 on the fp32 C
            C2 = torch.empty_like(C32)
            torch.addmm(C32, A_, B_, out_dtype=torch.float32, out=C2)
            return lambda: torch.addmm(C32, A_, B_, out_dtype=torch.float32, out=C2)
        except (TypeError, RuntimeError):
            return lambda: C32.add_(mm32())
    return None


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--only", default=None)
    ap.add_argument("--graph", action="store_true", help="time a CUDA-graph replay of the reps")
    ap.add_argument("--sweep", action="store_true", help="K sweep of the QKV / FC1 shapes (epilogue vs mainloop)")
    ap.add_argument("--cublas", action="store_true", help="also time torch.matmul (cuBLAS) on the same shape/majors")
    args = ap.parse_args()
    sh, keep = sweep() if args.sweep else shapes()
    st = torch.cuda.current_stream()
    total_f = total_t = 0.0
    for name, a, fl in sh:
        if args.only and args.only != name:
            continue
        for _ in range(3):
            H.hk("hk_gemm", C.byref(a), C.c_void_p(st.cuda_stream))
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        if args.graph:  # replay a captured sequence: no host launch cost between kernels (as in the step)
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g):
                cs = torch.cuda.current_stream()
                for _ in range(args.reps):
                    H.hk("hk_gemm", C.byref(a), C.c_void_p(cs.cuda_stream))
            g.replay()
            torch.cuda.synchronize()
            e0.record()
            g.replay()
            e1.record()
        else:
            e0.record()
            for _ in range(args.reps):
                H.hk("hk_gemm", C.byref(a), C.c_void_p(st.cuda_stream))
            e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / args.reps
        total_f += fl; total_t += ms
        rec = {"gemm": name, "M": a.M, "N": a.N, "K": a.K, "batch": a.nz0 * a.nz1, "us": ms * 1e3,
               "tflops": fl / (ms * 1e-3) / 1e12}
        if args.cublas and a.nz0 * a.nz1 == 1:
            bf = torch.bfloat16
            A_ = (torch.randn(a.K, a.M, device="cuda").to(bf).t() if a.a_mn_major else torch.randn(a.M, a.K, device="cuda").to(bf))
            B_ = (torch.randn(a.K, a.N, device="cuda").to(bf) if a.b_mn_major else torch.randn(a.N, a.K, device="cuda").to(bf).t())
            C_ = torch.empty(a.M, a.N, device="cuda", dtype=bf)
            for _ in range(3):
                torch.matmul(A_, B_, out=C_)
            torch.cuda.synchronize()
            e0.record()
            for _ in range(args.reps):
                torch.matmul(A_, B_, out=C_)
            e1.record()
            torch.cuda.synchronize()
            cms = e0.elapsed_time(e1) / args.reps
            rec["cublas_us"] = cms * 1e3
            rec["cublas_tflops"] = fl / (cms * 1e-3) / 1e12
            # the same fused op from library calls: cuBLASLt (bias epilogue where it has one) + the
            # PyTorch elementwise kernels for what it lacks — what a library user would run
            lib = library_equivalent(a, A_, B_)
            if lib is not None:
                for _ in range(3):
                    lib()
                torch.cuda.synchronize()
                e0.record()
                for _ in range(args.reps):
                    lib()
                e1.record()
                torch.cuda.synchronize()
                lms = e0.elapsed_time(e1) / args.reps
                rec["cublas_fused_us"] = lms * 1e3
                rec["vs_cublas_fused"] = lms / ms
        print(json.dumps(rec))
    print(json.dumps({"gemm": "ALL", "tflops": total_f / (total_t * 1e-3) / 1e12}))


if __name__ == "__main__":
    main()
