"""Step timeline of a bench workload (harmony_read_timeline): where the swap bytes move, how the
host link overlaps compute, and where the compute stream idles.

    python tools/timeline.py [--workload cfg3] [--out gpurun_out/timeline_cfg3.json]

One profiled step after 2 warm-up steps (events around every op; the per-op spans include the
profiling events, so the step is a few % slower than the bench's).  Prints per-stream busy time,
host-link GB/s while active, H2D/D2H overlap, and the compute stream's idle gaps by what it waited
for; writes the raw records to --out.
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
import synth  # noqa: E402
from paper_conf_hotos_lipmk21_b200 import harmony as H  # noqa: E402

KIND = {0: "INPUT", 1: "H2D", 2: "D2H", 3: "FWD", 4: "LOSS", 5: "BWD", 6: "UPD", 7: "AG", 8: "RS", 9: "LGATH", 10: "LOUT"}
CAT = {0: "weight", 1: "state", 2: "stash", 3: "input", 4: "output", 5: "grad", 6: "-"}


def union(iv):
    iv = sorted(iv)
    out = []
    for a, b in iv:
        if out and a <= out[-1][1]:
            out[-1][1] = max(out[-1][1], b)
        else:
            out.append([a, b])
    return out


def total(iv):
    return sum(b - a for a, b in iv)


def intersect(x, y):
    i = j = 0
    out = []
    while i < len(x) and j < len(y):
        a, b = max(x[i][0], y[j][0]), min(x[i][1], y[j][1])
        if a < b:
            out.append([a, b])
        if x[i][1] < y[j][1]:
            i += 1
        else:
            j += 1
    return out


def summarise(recs, step_s):
    s = {"step_ms": step_s * 1e3}
    for name, st in (("compute", 0), ("h2d", 1), ("d2h", 2), ("comm", 3)):
        iv = union([(r["t0"], r["t1"]) for r in recs if r["stream"] == st])
        by = sum(r["bytes"] for r in recs if r["stream"] == st and r["kind"] in (0, 1, 2))
        s[name] = {"busy_ms": total(iv) * 1e3, "util": total(iv) / step_s if step_s else None, "bytes": by,
                   "gbs_while_active": by / total(iv) / 1e9 if by and total(iv) else None}
    h = union([(r["t0"], r["t1"]) for r in recs if r["stream"] == 1])
    d = union([(r["t0"], r["t1"]) for r in recs if r["stream"] == 2])
    s["h2d_d2h_overlap_ms"] = total(intersect(h, d)) * 1e3
    fwd_end = max([r["t1"] for r in recs if r["kind"] == 3] or [0.0])
    s["forward_ms"] = fwd_end * 1e3
    for nm, st in (("h2d", 1), ("d2h", 2)):
        s[nm]["bytes_in_forward"] = sum(r["bytes"] for r in recs if r["stream"] == st and r["t1"] <= fwd_end)
        s[nm]["by_class"] = {}
        for r in recs:
            if r["stream"] == st:
                c = CAT.get(r["cat"], "?")
                s[nm]["by_class"][c] = s[nm]["by_class"].get(c, 0) + r["bytes"]
    comp = sorted([r for r in recs if r["stream"] == 0], key=lambda r: r["t0"])
    gaps, prev = [], 0.0
    for r in comp:
        if r["t0"] - prev > 2e-6:
            gaps.append((r["t0"] - prev, KIND[r["kind"]], r["layer"], r["micro"]))
        prev = max(prev, r["t1"])
    # direction balance over the step: the busy fraction of each stream in 20 equal windows
    t_end = max(r["t1"] for r in recs)
    nb = 20
    s["windows"] = []
    for k in range(nb):
        w = [[k * t_end / nb, (k + 1) * t_end / nb]]
        row = {}
        for nm, st in (("compute", 0), ("h2d", 1), ("d2h", 2)):
            iv = union([(r["t0"], r["t1"]) for r in recs if r["stream"] == st])
            row[nm] = round(total(intersect(iv, w)) / (t_end / nb), 2)
        s["windows"].append(row)
    s["compute_idle_ms"] = sum(g[0] for g in gaps) * 1e3
    s["compute_idle_top"] = [{"ms": round(g[0] * 1e3, 3), "before": f"{g[1]}(l={g[2]}, i={g[3]})"}
                             for g in sorted(gaps, reverse=True)[:12]]
    return s


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="cfg3", choices=[k for k in bench.WORKLOADS if k != "cfg5"])
    ap.add_argument("--stash-policy", type=int, default=2)
    ap.add_argument("--out", default=None)
    ap.add_argument("--microbatches", type=int, default=0)
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
        _, st_plain = h.step(Xd, Td)
        H.harmony_set_profiling(h.ctx, 1)
        _, st = h.step(Xd, Td)
        recs = H.harmony_read_timeline(h.ctx)
        H.harmony_set_profiling(h.ctx, 0)
        plan = h.plan().as_dict()
    summ = summarise(recs, st.step_seconds)
    summ["plain_step_ms"] = st_plain.step_seconds * 1e3
    summ["workload"] = wl["name"]
    summ["plan"] = {k: plan[k] for k in ("arena_bytes", "resident_state_bytes", "total_state_bytes",
                                         "resident_stash_bytes", "total_stash_bytes", "pred_h2d_bytes",
                                         "pred_d2h_bytes", "weight_slots", "stash_slots", "state_slots")}
    print(json.dumps(summ, indent=1))
    if a.out:
        with open(a.out, "w") as f:
            json.dump({"summary": summ, "records": recs}, f)


if __name__ == "__main__":
    main()
