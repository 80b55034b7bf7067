"""Time the step's GEMM shapes (cfg2, one microbatch of 4096 tokens, d = 1024) through hk_gemm.

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

T, D, S, B, NH = 4096, 1024, 512, 8, 16
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
        out.append((name, a, 2.0 * M * N * K * a.nz0 * a.nz1))

    X, W, Q, P, C32, C16 = (t.data_ptr() for t in (x, w, qkv, p, c32, c16))
    g("fc1_fwd", T, 4 * D, D, X, 0, D, W, 1, 4 * D, C16, 4 * D, H.HK_EPI_STORE_T)
    g("fc2_fwd", T, D, 4 * D, X, 0, 4 * D, W, 1, D, C32, D, H.HK_EPI_STORE_F32)
    g("qkv_fwd", T, 3 * D, D, X, 0, D, W, 1, 3 * D, C16, 3 * D, H.HK_EPI_STORE_T)
    g("fc1_dgrad", T, D, 4 * D, X, 0, 4 * D, W, 0, 4 * D, C32, D, H.HK_EPI_STORE_F32)
    g("fc1_wgrad", D, 4 * D, T, X, 1, D, X, 1, 4 * D, C32, 4 * D, H.HK_EPI_ACC_F32, acc=1)
    g("fc2_wgrad", 4 * D, D, T, X, 1, 4 * D, X, 1, D, C32, D, H.HK_EPI_ACC_F32, acc=1)
    g("attn_qk", S, S, DH, Q, 0, 3 * D, Q + 2 * D, 0, 3 * D, C32, S, H.HK_EPI_STORE_F32, nz0=NH, nz1=B,
      a_sz0=DH, a_sz1=S * 3 * D, b_sz0=DH, b_sz1=S * 3 * D, c_sz0=S * S, c_sz1=NH * S * S)
    g("attn_pv", S, DH, S, P, 0, S, Q + 4 * D, 1, 3 * D, C16, D, H.HK_EPI_STORE_T, nz0=NH, nz1=B,
      a_sz0=S * S, a_sz1=NH * S * S, b_sz0=DH, b_sz1=S * 3 * D, c_sz0=DH, c_sz1=S * D)
    g("attn_dv", S, DH, S, P, 1, S, Q, 1, 3 * D, C16, D, H.HK_EPI_STORE_T, nz0=NH, nz1=B,
      a_sz0=S * S, a_sz1=NH * S * S, b_sz0=DH, b_sz1=S * 3 * D, c_sz0=DH, c_sz1=S * D)
    return out, (x, w, qkv, p, c32, c16)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--only", default=None)
    args = ap.parse_args()
    sh, keep = shapes()
    st = torch.cuda.current_stream()
    total_f = total_t = 0.0
    for name, a, fl in sh:
        if args.only and args.only != name:
            continue
        for _ in range(3):
            H.hk("hk_gemm", C.byref(a), C.c_void_p(st.cuda_stream))
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(args.reps):
            H.hk("hk_gemm", C.byref(a), C.c_void_p(st.cuda_stream))
        e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / args.reps
        total_f += fl; total_t += ms
        print(json.dumps({"gemm": name, "M": a.M, "N": a.N, "K": a.K, "batch": a.nz0 * a.nz1, "us": ms * 1e3,
                          "tflops": fl / (ms * 1e-3) / 1e12}))
    print(json.dumps({"gemm": "ALL", "tflops": total_f / (total_t * 1e-3) / 1e12}))


if __name__ == "__main__":
    main()
