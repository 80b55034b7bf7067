"""Kernel-level timeline of one profiled step (harmony_read_kernel_timeline): every launch's class,
stream and span.  Prints per-stream busy time by kernel class and shape, the compute stream's idle
time, and how much of each class ran concurrently with another class.

    python tools/ktimeline.py [--workload cfg2] [--stash-policy 2] [--out gpurun_out/ktl.json]
"""
import argparse
import json
import os
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
import synth  # noqa: E402
from paper_conf_hotos_lipmk21_b200 import harmony as H  # noqa: E402
from timeline import union, total, intersect  # noqa: E402

CLS = ("gemm", "adam", "ln", "softmax", "other", "attn")
STREAM = {0: "compute", 1: "h2d", 2: "d2h", 3: "comm", 4: "side", -1: "?"}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="cfg2")
    ap.add_argument("--stash-policy", type=int, default=2)
    ap.add_argument("--microbatches", type=int, default=0)
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    wl = bench.WORKLOADS[a.workload]
    descs = wl["descs"]()
    B, m = wl["per_gpu_batch"], a.microbatches or wl["m"]
    prec = wl.get("precision", 1)
    params = synth.gen_params(descs, prec)
    X, T = synth.gen_batch(descs, B, 1, prec)
    Xd, Td = torch.tensor(X, device="cuda"), torch.tensor(T, device="cuda")
    with H.Harmony(descs, params, microbatches=m, microbatch_size=B // m, precision=prec,
                   stash_policy=a.stash_policy if prec else 0, hbm_cap_bytes=wl["cap"], lr=1e-4) as h:
        del params
        for _ in range(2):
            h.step(Xd, Td)
        _, plain = h.step(Xd, Td)
        H.harmony_set_profiling(h.ctx, 1)
        _, st = h.step(Xd, Td)
        recs = H.harmony_read_kernel_timeline(h.ctx)
        prof = H.harmony_read_profile(h.ctx).as_dict()
        H.harmony_set_profiling(h.ctx, 0)
    out = {"plain_step_ms": plain.step_seconds * 1e3, "profiled_step_ms": st.step_seconds * 1e3, "launches": len(recs)}
    by = defaultdict(lambda: [0, 0.0, 0.0])  # (stream, class, work) -> launches, seconds, work
    for r in recs:
        k = (STREAM[r["stream"]], CLS[r["cat"]], round(r["work"] / 1e9, 2))
        by[k][0] += 1
        by[k][1] += r["t1"] - r["t0"]
        by[k][2] += r["work"]
    rows = sorted(by.items(), key=lambda kv: -kv[1][1])
    out["by_stream_class_work"] = [
        {"stream": k[0], "class": k[1], "work_G": k[2], "launches": v[0], "ms": round(v[1] * 1e3, 3),
         "avg_us": round(v[1] / v[0] * 1e6, 2),
         "tflops_or_gbs": round(v[2] / v[1] / 1e12, 1) if v[1] and k[1] in ("gemm", "attn") else
         (round(v[2] / v[1] / 1e9, 1) if v[1] else None)} for k, v in rows]
    comp = union([(r["t0"], r["t1"]) for r in recs if r["stream"] == 0])
    side = union([(r["t0"], r["t1"]) for r in recs if r["stream"] == 4])
    out["compute_busy_ms"] = total(comp) * 1e3
    out["side_busy_ms"] = total(side) * 1e3
    out["compute_side_overlap_ms"] = total(intersect(comp, side)) * 1e3
    any_k = union([(r["t0"], r["t1"]) for r in recs])
    out["any_kernel_busy_ms"] = total(any_k) * 1e3
    out["class_busy_ms"] = {}
    for c in range(6):
        iv = union([(r["t0"], r["t1"]) for r in recs if r["cat"] == c])
        out["class_busy_ms"][CLS[c]] = round(total(iv) * 1e3, 3)
    out["profile"] = prof
    print(json.dumps(out, indent=1))
    if a.out:
        with open(a.out, "w") as f:
            json.dump({"summary": out, "records": recs}, f)


if __name__ == "__main__":
    main()
