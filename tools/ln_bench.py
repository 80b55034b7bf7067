"""LayerNorm forward / backward at the cfg2 per-microbatch shape (16384 x 1024) through hk_*, graph
replay, warm and with an L2 flush between launches: achieved GB/s of the algorithmic bytes.

    python tools/ln_bench.py [--rows 16384] [--d 1024]
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


def timeit(fn, reps, flush=None):
    g = torch.cuda.CUDAGraph()
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        fn(s)
        torch.cuda.synchronize()
        with torch.cuda.graph(g, stream=s):
            for _ in range(reps):
                if flush is not None:
                    flush.add_(1.0)
                fn(s)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    g.replay()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps * 1e3


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--rows", type=int, default=16384)
    ap.add_argument("--d", type=int, default=1024)
    ap.add_argument("--reps", type=int, default=20)
    a = ap.parse_args()
    R, D = a.rows, a.d
    X = torch.randn(R, D, device="cuda")
    g = (1 + 0.1 * torch.randn(D, device="cuda")).to(torch.bfloat16)
    b = (0.02 * torch.randn(D, device="cuda")).to(torch.bfloat16)
    U = torch.empty(R, D, device="cuda", dtype=torch.bfloat16)
    mean, rstd = torch.empty(R, device="cuda"), torch.empty(R, device="cuda")
    dU, dres, dX = torch.randn(R, D, device="cuda"), torch.randn(R, D, device="cuda"), torch.empty(R, D, device="cuda")
    dg, db = torch.empty(D, device="cuda"), torch.empty(D, device="cuda")
    flush = torch.empty(64 << 20, device="cuda")  # 256 MB > L2

    def fwd(s):
        H.hk("hk_layernorm_fwd", 1, R, D, X.data_ptr(), g.data_ptr(), b.data_ptr(), U.data_ptr(), mean.data_ptr(),
             rstd.data_ptr(), C.c_void_p(s.cuda_stream))

    def bwd(s):
        H.hk("hk_layernorm_bwd", 1, R, D, dU.data_ptr(), X.data_ptr(), mean.data_ptr(), rstd.data_ptr(), g.data_ptr(),
             dres.data_ptr(), dX.data_ptr(), dg.data_ptr(), db.data_ptr(), 0, C.c_void_p(s.cuda_stream))

    fb = R * D * (4 + 2) + R * 8
    bb = R * D * 4 * 4
    for name, fn, by in (("ln_fwd", fwd, fb), ("ln_bwd", bwd, bb)):
        warm = timeit(fn, a.reps)
        ft = timeit(fn, a.reps, flush)
        fl = timeit(lambda s: None, a.reps, flush)
        cold = ft - fl
        print(json.dumps({"kernel": name, "bytes": by, "warm_us": warm, "warm_gbs": by / warm / 1e3,
                          "cold_us": cold, "cold_gbs": by / cold / 1e3}))


if __name__ == "__main__":
    main()
