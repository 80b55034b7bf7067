"""One Harmony-DP step of the bench workload for ncu launch lists (kernel shares of a step).

    ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
        python tools/profile_step.py --layers 2 --steps 2

Same per-layer shapes and launch configuration as `bench.py` (cfg2: d=1024, h=16, S=512,
m=2 x b=32 by default, stash policy 2); `--layers` trims the stack depth so the list stays short (every layer
runs the identical kernel sequence).  Eager issue (HARMONY_NO_GRAPH=1 is set) so each kernel is
one launch record.
"""
import argparse
import os
import sys

os.environ.setdefault("HARMONY_NO_GRAPH", "1")
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_hotos_lipmk21_b200 import harmony as H  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--layers", type=int, default=2)
    ap.add_argument("--steps", type=int, default=2)
    ap.add_argument("--policy", type=int, default=2)
    ap.add_argument("--microbatches", type=int, default=2)
    ap.add_argument("--cfg3", action="store_true", help="GPT-2 XL geometry (d=1600, h=25, S=1024 causal, 8 seq, 16 GiB)")
    a = ap.parse_args()
    if a.cfg3:
        descs, B, cap = synth.transformer_stack(a.layers, 1600, 25, 1024, True), 8, 16 << 30
    else:
        descs, B, cap = synth.transformer_stack(a.layers, 1024, 16, 512, False), 64, 8 << 30
    params = synth.gen_params(descs, 1)
    X, T = synth.gen_batch(descs, B, 1, 1)
    Xd, Td = torch.tensor(X, device="cuda"), torch.tensor(T, device="cuda")
    with H.Harmony(descs, params, microbatches=a.microbatches, microbatch_size=B // a.microbatches, precision=1,
                   stash_policy=a.policy, hbm_cap_bytes=cap, lr=1e-4) as h:
        for _ in range(a.steps):
            loss, st = h.step(Xd, Td)
            print("step", loss, st.step_seconds, st.kernel_launches)


if __name__ == "__main__":
    main()
