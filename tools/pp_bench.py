"""Harmony-PP (reading c27) on the available GPUs: one process drives N ranks (ranks share a GPU when
there are fewer GPUs than ranks — the loopback), layer l on rank l % N, activations / gradients handed
rank to rank.  Prints one JSON line: step time, samples/s, the weight swap ledger (3|W| per iteration for
the whole box) and the peer-to-peer bytes; the same model as Harmony-DP on one rank beside it.

    python tools/pp_bench.py [--ranks 2] [--layers 8] [--cap-gib 4] [--steps 5]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_hotos_lipmk21_b200 import harmony as H  # noqa: E402


def run(descs, params, X, T, steps, **cfg):
    with H.Harmony(descs, params, **cfg) as h:
        for _ in range(2):
            h.step(X, T)
        tot, st = 0.0, None
        for _ in range(steps):
            _, st = h.step(X, T)
            tot += st.step_seconds
        return tot / steps, st.as_dict(), h.plan().as_dict()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--ranks", type=int, default=2)
    ap.add_argument("--layers", type=int, default=8)
    ap.add_argument("--cap-gib", type=float, default=2.0)
    ap.add_argument("--steps", type=int, default=5)
    a = ap.parse_args()
    ngpu = torch.cuda.device_count()
    devices = [r % ngpu for r in range(a.ranks)]
    descs = synth.transformer_stack(a.layers, 1024, 16, 512, False)  # cfg2 blocks
    params = synth.gen_params(descs, 1)
    m, b = 2, 32
    X, T = synth.gen_batch(descs, m * b, 1, 1)
    Xd, Td = torch.tensor(X, device="cuda"), torch.tensor(T, device="cuda")
    cap = int(a.cap_gib * (1 << 30))
    common = dict(microbatches=m, microbatch_size=b, precision=1, stash_policy=2, hbm_cap_bytes=cap, lr=1e-4)
    pp_s, pp_st, pp_plan = run(descs, params, Xd, Td, a.steps, group=devices, schedule=H.HARMONY_SCHED_HARMONY_PP,
                               **common)
    dp_s, dp_st, dp_plan = run(descs, params, Xd, Td, a.steps, **common)
    W = sum(-(-d.n_params() // 1024) * 1024 * 2 for d in descs)  # bf16 compute copies, padded
    line = {"workload": f"{a.layers} cfg2 blocks (d1024 h16 S512), {m}x{b} sequences, cap {a.cap_gib} GiB per rank",
            "ranks": a.ranks, "devices": devices,
            "pp": {"ms_per_step": pp_s * 1e3, "samples_per_s": m * b / pp_s, "h2d_weight_bytes": pp_st["h2d_weight_bytes"],
                   "d2h_weight_bytes": pp_st["d2h_weight_bytes"], "p2p_bytes": pp_st["nvlink_bytes"],
                   "weight_swaps_over_W": (pp_st["h2d_weight_bytes"] + pp_st["d2h_weight_bytes"]) / W,
                   "resident_weight_bytes": pp_plan["resident_weight_bytes"]},
            "dp_one_rank": {"ms_per_step": dp_s * 1e3, "samples_per_s": m * b / dp_s,
                            "h2d_weight_bytes": dp_st["h2d_weight_bytes"], "d2h_weight_bytes": dp_st["d2h_weight_bytes"]},
            "W_bytes_bf16": W}
    print(json.dumps(line))


if __name__ == "__main__":
    main()
