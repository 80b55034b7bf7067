"""Fused attention on the cfg2 per-microbatch shape (b=16 sequences, S=512, 16 heads, dh=64).

    python tools/attn_bench.py [--reps 20] [--causal 0]

Forward timed with CUDA events over back-to-back launches (TFLOP/s of the QK^T and PV
contractions); the backward (synchronous C-ABI call) is launched --reps times for an ncu
launch list (its kernels' durations come from ncu, not from this script).
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


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--causal", type=int, default=0)
    ap.add_argument("--b", type=int, default=16)
    ap.add_argument("--S", type=int, default=512)
    ap.add_argument("--h", type=int, default=16)
    ap.add_argument("--dh", type=int, default=64)
    a = ap.parse_args()
    b, S, h, dh = a.b, a.S, a.h, a.dh
    d = h * dh
    g = torch.Generator(device="cuda").manual_seed(0)
    qkv = (torch.randn(b * S, 3 * d, device="cuda", generator=g) * 1.5).to(torch.bfloat16)
    dC = torch.randn(b * S, d, device="cuda", generator=g).to(torch.bfloat16)
    C_ = torch.zeros(b * S, d, device="cuda", dtype=torch.bfloat16)
    lse = torch.zeros(b, h, S, device="cuda")
    dQKV = torch.zeros(b * S, 3 * d, device="cuda", dtype=torch.bfloat16)
    st = torch.cuda.current_stream()
    sp = C.c_void_p(st.cuda_stream)

    def fwd():
        H.hk("hk_attention_fwd", b, S, h, dh, a.causal, qkv.data_ptr(), C_.data_ptr(), lse.data_ptr(), sp)

    for _ in range(3):
        fwd()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(a.reps):
        fwd()
    e1.record()
    torch.cuda.synchronize()
    us = e0.elapsed_time(e1) / a.reps * 1e3
    fl = 4.0 * b * h * S * S * dh * (0.5 if a.causal else 1.0)
    print(json.dumps({"attn_fwd_us": us, "tflops": fl / (us * 1e-6) / 1e12}))
    for _ in range(a.reps):
        H.hk("hk_attention_bwd", b, S, h, dh, a.causal, qkv.data_ptr(), C_.data_ptr(), dC.data_ptr(), lse.data_ptr(),
             dQKV.data_ptr(), sp)
    torch.cuda.synchronize()


if __name__ == "__main__":
    main()
