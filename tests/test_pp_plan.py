"""Harmony-PP (Fig. 4; DESIGN reading c27) planned on the
host: the group program has Fig. 4's shape, moves 3|W| of weights per iteration for the whole box
whatever N and m, hands activations / gradients peer to peer, and is race-free (the independent
byte-range validator over every rank's streams)."""
import re

import pytest

import synth
from paper_conf_hotos_lipmk21_b200 import harmony as H


def gplan(descs, N, **kw):
    cfg = H.make_config(schedule=H.HARMONY_SCHED_HARMONY_PP, **kw)
    s, txt = H.harmony_plan_dry_group(cfg, N, descs)
    ops = []
    for line in txt.splitlines()[1:]:
        f = line.split()
        d = dict(kv.split("=", 1) for kv in f[3:])
        ops.append(dict(idx=int(f[0]), kind=f[1], stream=f[2], rank=int(d["rank"]), cat=d["cat"], l=int(d["l"]),
                        i=int(d["i"]), bytes=int(d["bytes"]), peer=int(d.get("peer", -1)),
                        waits=[int(w) for w in d["waits"].split(",") if w]))
    return s, ops


def weight_bytes(descs, bf16=False):
    return sum(d.n_params() * (2 if bf16 else 4) for d in descs)


def test_fig4_schedule_four_layers_two_gpus_two_microbatches():
    """Fig. 4: a four-layer model on two GPUs, layer-level tasks, two microbatches:
    GPU1 runs L1 and L3, GPU2 runs L2 and L4; each layer's task runs both microbatches back to back
    (input-batch grouping) before the next layer; the update of a layer follows its backward group;
    all inputs / outputs of a layer move GPU to GPU."""
    descs = synth.mlp_stack(4, 32)
    s, ops = gplan(descs, 2, microbatches=2, microbatch_size=4, hbm_cap_bytes=0)
    assert s.hazards == 0
    comp = {r: [(o["kind"], o["l"], o["i"]) for o in ops if o["rank"] == r and o["stream"] == "compute"] for r in (0, 1)}
    assert comp[0] == [("FWD", 0, 0), ("FWD", 0, 1), ("FWD", 2, 0), ("FWD", 2, 1),
                       ("BWD", 2, 0), ("BWD", 2, 1), ("UPD", 2, -1), ("BWD", 0, 0), ("BWD", 0, 1), ("UPD", 0, -1)]
    assert comp[1] == [("FWD", 1, 0), ("FWD", 1, 1), ("FWD", 3, 0), ("FWD", 3, 1), ("LOSS", -1, 0), ("LOSS", -1, 1),
                       ("BWD", 3, 0), ("BWD", 3, 1), ("UPD", 3, -1), ("BWD", 1, 0), ("BWD", 1, 1), ("UPD", 1, -1)]
    p2p = [o for o in ops if o["kind"] == "P2P"]
    assert len(p2p) == 2 * 3 * 2  # activations forward and gradients backward over the 3 layer boundaries, per microbatch
    assert all(o["peer"] != o["rank"] for o in p2p)
    # pipelining: GPU2's first forward waits only for microbatch 0's activations, not for L1's whole group
    f10 = next(o for o in ops if o["kind"] == "FWD" and o["l"] == 1 and o["i"] == 0)
    assert any(ops[w]["kind"] == "P2P" and ops[w]["i"] == 0 for w in f10["waits"])
    f01 = next(o for o in ops if o["kind"] == "FWD" and o["l"] == 0 and o["i"] == 1)
    assert f10["idx"] > f01["idx"] or all(ops[w]["kind"] != "FWD" for w in f10["waits"])


@pytest.mark.parametrize("N", [2, 3, 4])
@pytest.mark.parametrize("m", [1, 2, 4])
def test_weight_swap_volume_is_3W_for_the_whole_box(N, m):
    """Harmony-PP's per-iteration weight swap volume is 3|W| across all m microbatches and
    all N GPUs (swap in once for the forward group, once for the backward group, out once after the
    JIT update), vs (4m+2)N|W| for DP with per-GPU virtualization."""
    descs = synth.mlp_stack(8, 256)
    W = weight_bytes(descs)
    tiny, _ = gplan(descs, N, microbatches=m, microbatch_size=8, hbm_cap_bytes=1 << 40)
    cap = int(tiny.min_working_set_bytes * 1.05)  # nothing resident: every layer streams
    s, ops = gplan(descs, N, microbatches=m, microbatch_size=8, hbm_cap_bytes=cap)
    assert s.hazards == 0 and s.resident_weight_bytes == 0
    h2d_w = sum(o["bytes"] for o in ops if o["kind"] == "H2D" and o["cat"] == "weight")
    d2h_w = sum(o["bytes"] for o in ops if o["kind"] == "D2H" and o["cat"] == "weight")
    pad = sum(-(-d.n_params() // 1024) * 1024 * 4 for d in descs)  # each layer's copy padded to 1024 elements
    assert h2d_w == 2 * pad and d2h_w == pad and pad >= W and pad - W < len(descs) * 4096
    assert s.pred_h2d_weight_bytes == h2d_w and s.pred_d2h_weight_bytes == d2h_w


@pytest.mark.parametrize("cap_factor", [0, 1.05, 1.5, 3.0])
def test_pp_plans_are_hazard_free_transformer(cap_factor):
    descs = synth.transformer_stack(6, 64, 2, 64, True)
    kw = dict(microbatches=2, microbatch_size=2, precision=1, stash_policy=2)
    base, _ = gplan(descs, 3, hbm_cap_bytes=1 << 40, **kw)
    cap = 0 if cap_factor == 0 else int(base.min_working_set_bytes * cap_factor)
    s, ops = gplan(descs, 3, hbm_cap_bytes=cap, **kw)
    assert s.hazards == 0
    # each rank's layers and only those
    for o in ops:
        if o["kind"] in ("FWD", "BWD", "UPD"):
            assert o["l"] % 3 == o["rank"]


def test_pp_needs_a_group_and_enough_layers():
    descs = synth.mlp_stack(2, 32)
    with pytest.raises(H.HarmonyError):
        gplan(descs, 3, microbatches=1, microbatch_size=2)
    with pytest.raises(H.HarmonyError):
        H.harmony_plan_dry(H.make_config(schedule=H.HARMONY_SCHED_HARMONY_PP), descs, text_len=0)
