"""Per-event timeline of the fused attention forward's CTA 0 (HM_ATTN_TRACE build).

    HARMONY_NVCC_EXTRA=-DHM_ATTN_TRACE python -m paper_conf_hotos_lipmk21_b200.build
    python tools/attn_trace.py [--b 32] [--causal 0]

Prints, per role (softmax warp 2 / MMA issuer / TMA producer), each event's clock relative to the
first, and the mean gap between consecutive event codes over the steady state."""
import argparse
import collections
import ctypes as C
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

from paper_conf_hotos_lipmk21_b200 import harmony as H  # noqa: E402

NAMES = {1: "tma:Q", 2: "tma:K", 3: "tma:V", 10: "mma:S", 11: "mma:PV", 12: "mma:S_B", 13: "mma:PV_B", 14: "mma:PV_issued", 15: "mma:S_issued", 30: "b:s_full", 31: "b:ld", 33: "b:p_empty", 34: "b:p_full",
         40: "bm:p_full", 41: "bm:dVdK_issued", 42: "bm:S_start", 43: "bm:S_issued", 20: "sm:s_full", 21: "sm:ld", 22: "sm:max_bar",
         23: "sm:exps", 24: "sm:p_empty", 25: "sm:p_full", 26: "sm:o_full", 27: "sm:o_read"}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--b", type=int, default=32)
    ap.add_argument("--causal", type=int, default=0)
    ap.add_argument("--show", type=int, default=60)
    ap.add_argument("--fwd2", type=int, default=0, help="trace the two-query-tile kernel (HARMONY_ATTN_FWD=2)")
    ap.add_argument("--bwd", type=int, default=0, help="trace the persistent backward (its first CTA)")
    a = ap.parse_args()
    b, S, h, dh = a.b, 512, 16, 64
    d = h * dh
    qkv = (torch.randn(b * S, 3 * d, device="cuda") * 1.5).to(torch.bfloat16)
    C_ = torch.zeros(b * S, d, device="cuda", dtype=torch.bfloat16)
    lse = torch.zeros(b, h, S, device="cuda")
    lib = H.lib()
    fn = lib.hm_attn2_trace_read if a.fwd2 else lib.hm_attn_trace_read
    out = np.zeros((3, 2048), np.uint64)
    cnt = np.zeros(3, np.int32)
    dC = torch.randn(b * S, d, device="cuda").to(torch.bfloat16)
    dQKV = torch.zeros(b * S, 3 * d, device="cuda", dtype=torch.bfloat16)
    for _ in range(2):
        H.hk("hk_attention_fwd", b, S, h, dh, a.causal, qkv.data_ptr(), C_.data_ptr(), lse.data_ptr(), None)
        fn(out.ctypes.data_as(C.c_void_p), cnt.ctypes.data_as(C.c_void_p))
        if a.bwd:
            H.hk("hk_attention_bwd", b, S, h, dh, a.causal, qkv.data_ptr(), C_.data_ptr(), dC.data_ptr(),
                 lse.data_ptr(), dQKV.data_ptr(), None)
            fn(out.ctypes.data_as(C.c_void_p), cnt.ctypes.data_as(C.c_void_p))
    t0 = None
    roles = ["softmax warp 4 (tile A)", "MMA", "softmax warp 8 (tile B)"] if a.fwd2 else ["softmax warp 2", "MMA", "TMA"]
    for row, name in enumerate(roles):
        n = min(int(cnt[row]), 2048)
        ev = [(int(x) >> 56, int(x) & ((1 << 56) - 1)) for x in out[row, :n]]
        if t0 is None:
            t0 = min(t for _, t in ev)
        print(f"== {name}: {n} events")
        for code, t in ev[: a.show]:
            print(f"  {t - t0:8d}  {NAMES.get(code, code)}")
        gaps = collections.defaultdict(list)
        for (c0, t0_), (c1, t1_) in zip(ev[8:], ev[9:]):
            gaps[(NAMES.get(c0, c0), NAMES.get(c1, c1))].append(t1_ - t0_)
        for k, v in sorted(gaps.items(), key=lambda kv: -np.sum(kv[1])):
            print(f"  {k[0]:>12} -> {k[1]:<12} n={len(v):4d} mean {np.mean(v):7.1f} cycles  total {np.sum(v)}")


if __name__ == "__main__":
    main()
