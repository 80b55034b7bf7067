"""The C-ABI library on a host without a GPU: it loads, exports every declared symbol, its
ABI structs match the binding, and the host-only planner (harmony_plan_dry) builds programs
with the paper's scheduling properties (grouping, JIT update, swap volumes, Fig. 5(a) swap
sets) and no data races (independent byte-range validator)."""
import ctypes as C
import os
import re

import numpy as np
import pytest

import oracle
import synth
from paper_conf_hotos_lipmk21_b200 import harmony as H

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_functions():
    names = set()
    for h in ("harmony.h", "harmony_kernels.h"):
        src = open(os.path.join(ROOT, "include", h)).read()
        src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
        for m in re.finditer(r"^\s*(?:const\s+)?[A-Za-z_][A-Za-z0-9_]*\s*\**\s+\**\s*((?:harmony|hk)_[a-z0-9_]+)\s*\(",
                             src, flags=re.M):
            names.add(m.group(1))
    return sorted(names)


def test_library_loads_and_exports_every_declared_symbol():
    L = H.lib()
    names = declared_functions()
    assert len(names) >= 20, names
    for n in names:
        assert hasattr(L, n), f"libharmony.so does not export {n}"
    assert L.harmony_abi_version() == 1


def test_abi_struct_sizes_match_binding():
    out = (C.c_uint64 * 6)()
    H.lib().harmony_abi_sizes(out)
    assert list(out) == [C.sizeof(H.harmony_config), C.sizeof(H.harmony_layer_desc),
                         C.sizeof(H.harmony_step_stats), C.sizeof(H.harmony_plan_summary), C.sizeof(H.hk_gemm_args),
                         C.sizeof(H.harmony_kernel_profile)]


def test_library_is_built_for_sm100a():
    import subprocess
    out = subprocess.run(["cuobjdump", "-lelf", H.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out
    sass = subprocess.run(["cuobjdump", "-sass", H.LIB_PATH], capture_output=True, text=True).stdout
    assert "UTCHMMA" in sass and "UTMALDG" in sass and "LDTM" in sass  # tcgen05.mma, TMA, tcgen05.ld


def plan(descs, **kw):
    cfg = H.make_config(**kw)
    s, txt = H.harmony_plan_dry(cfg, descs)
    ops = []
    for line in txt.splitlines()[1:]:
        f = line.split()
        d = dict(kv.split("=", 1) for kv in f[3:])
        ops.append(dict(idx=int(f[0]), kind=f[1], stream=f[2], cat=d["cat"], l=int(d["l"]), i=int(d["i"]),
                        bytes=int(d["bytes"]), waits=[int(w) for w in d["waits"].split(",") if w]))
    return s, ops


MLP = synth.mlp_stack(4, 256)
CFG1 = dict(microbatches=4, microbatch_size=8, hbm_cap_bytes=synth.CONFIGS["cfg1"]["cap"])


def min_cap(descs, **kw):
    s, _ = plan(descs, **dict(kw, hbm_cap_bytes=1 << 40))
    return s.min_working_set_bytes


@pytest.mark.parametrize("kw", [CFG1, dict(CFG1, hbm_cap_bytes=0), dict(CFG1, microbatches=1, microbatch_size=32),
                                dict(CFG1, hbm_cap_bytes=3_000_000), dict(CFG1, retain_grads=1)])
def test_plans_are_hazard_free(kw):
    s, ops = plan(MLP, **kw)
    assert s.hazards == 0
    assert s.arena_bytes <= (kw["hbm_cap_bytes"] or 1 << 62)


@pytest.mark.parametrize("policy", [0, 1, 2])
@pytest.mark.parametrize("S,L,m", [(16, 6, 3), (64, 3, 2), (128, 4, 4)])
def test_transformer_plans_hazard_free_over_caps(policy, S, L, m):
    """Plan fuzz: every cap between the minimum working set and all-resident, for each stash policy,
    gives a program without races and without a read of a spilled stash before its spill (the
    independent validator; a regression of the latter was caught this way)."""
    descs = synth.transformer_stack(L, 64, 4, S, True)
    kw = dict(microbatches=m, microbatch_size=2, precision=1, stash_policy=policy)
    base = min_cap(descs, **kw)
    for f in (1.0, 1.05, 1.1, 1.2, 1.3, 1.5, 2.0, 3.0, 6.0):
        s, _ = plan(descs, **dict(kw, hbm_cap_bytes=int(base * f)))
        assert s.hazards == 0, (policy, S, f)


def test_cap_too_small_is_reported():
    cap = min_cap(MLP, **dict(CFG1))
    s, ops = plan(MLP, **dict(CFG1, hbm_cap_bytes=cap))
    assert s.hazards == 0 and sum(o["kind"] == "FWD" for o in ops) == 4 * 4
    # below the unsplit minimum the fp32 layers run as column panels (operator split, row a15) ...
    s, ops = plan(MLP, **dict(CFG1, hbm_cap_bytes=cap - 1))
    assert s.hazards == 0 and sum(o["kind"] == "FWD" for o in ops) > 4 * 4
    # ... until not even the activations and one panel fit
    with pytest.raises(H.HarmonyError) as e:
        plan(MLP, **dict(CFG1, hbm_cap_bytes=cap // 8))
    assert e.value.code == H.HARMONY_E_CAP_TOO_SMALL


def test_harmony_dp_weight_swap_volume_is_3W():
    """Harmony-DP swaps W in once for the forward and once for the backward (grouping)
    and out once after the update (JIT): 3N|W| per iteration; here N = 1 and nothing resident."""
    cap = min_cap(MLP, **CFG1)
    s, ops = plan(MLP, **dict(CFG1, hbm_cap_bytes=cap))
    assert s.resident_weight_bytes == 0
    Wb = s.total_weight_bytes
    assert s.pred_h2d_weight_bytes + s.pred_d2h_weight_bytes == oracle.weight_swap_harmony_dp(Wb, 4, 1)
    assert s.pred_h2d_weight_bytes == 2 * Wb and s.pred_d2h_weight_bytes == Wb
    assert s.pred_h2d_weight_bytes + s.pred_d2h_weight_bytes < oracle.weight_swap_baseline_dp(Wb, 4, 1)


@pytest.mark.parametrize("m", [1, 2, 4])
def test_baseline_schedule_weight_swap_volume(m):
    """P:726-731 (Fig. 5(b)): DP with per-GPU memory virtualization swaps W in and out for the
    forward and the backward of every microbatch, plus in and out for the update: (4m+2)N|W| in the
    paper's count.  Here the update's swap-in of W is the fp32 master copy inside the Adam state, so
    the compute-copy ledger is (4m+1)|W| — against Harmony-DP's 3|W| at the same cap.  The baseline
    updates after the whole backward, so each layer's gradient is parked on the host and comes back."""
    kw = dict(CFG1, microbatches=m, microbatch_size=32 // m)
    cap = min_cap(MLP, **dict(kw, schedule=H.HARMONY_SCHED_PER_GPU_VIRT))
    s, ops = plan(MLP, **dict(kw, hbm_cap_bytes=cap, schedule=H.HARMONY_SCHED_PER_GPU_VIRT))
    Wb = s.total_weight_bytes
    assert s.resident_weight_bytes == 0 and s.hazards == 0
    assert s.pred_h2d_weight_bytes == 2 * m * Wb and s.pred_d2h_weight_bytes == (2 * m + 1) * Wb
    assert s.pred_h2d_weight_bytes + s.pred_d2h_weight_bytes + Wb == oracle.weight_swap_baseline_dp(Wb, m, 1)
    grad = [o for o in ops if o["cat"] == "grad"]
    assert sorted((o["kind"], o["l"]) for o in grad) == sorted([("D2H", l) for l in range(4)] + [("H2D", l) for l in range(4)])
    # every update after the last backward
    comp = [(o["kind"], o["l"]) for o in ops if o["stream"] == "compute"]
    last_bwd = max(k for k, (kind, _) in enumerate(comp) if kind == "BWD")
    assert all(k > last_bwd for k, (kind, _) in enumerate(comp) if kind == "UPD")
    s2, _ = plan(MLP, **dict(kw, hbm_cap_bytes=cap))
    assert s2.pred_h2d_weight_bytes + s2.pred_d2h_weight_bytes == oracle.weight_swap_harmony_dp(Wb, m, 1)


@pytest.mark.parametrize("m", [1, 2, 4, 8])
def test_grouping_weight_traffic_independent_of_m(m):
    """a task runs over its group of m microbatches back to back, so W is swapped once."""
    cap = min_cap(MLP, microbatches=8, microbatch_size=4)
    s, ops = plan(MLP, microbatches=m, microbatch_size=4, hbm_cap_bytes=cap)
    assert s.pred_h2d_weight_bytes == 2 * s.total_weight_bytes - 2 * s.resident_weight_bytes
    n_w_in = sum(1 for o in ops if o["kind"] == "H2D" and o["cat"] == "weight")
    streamed_layers = 4 - s.resident_weight_bytes // (s.total_weight_bytes // 4)
    assert n_w_in == 2 * streamed_layers  # one swap-in per layer per pass, whatever m is


def test_jit_update_right_after_backward():
    """UPD(l) is scheduled right after BWD(l, m) — before any BWD of layer l-1."""
    s, ops = plan(MLP, **CFG1)
    comp = [o for o in ops if o["stream"] == "compute"]
    seq = [(o["kind"], o["l"], o["i"]) for o in comp]
    for l in range(4):
        u = seq.index(("UPD", l, -1))
        last_b = max(k for k, t in enumerate(seq) if t[0] == "BWD" and t[1] == l)
        assert u == last_b + 1
        if l > 0:
            assert u < min(k for k, t in enumerate(seq) if t[0] == "BWD" and t[1] == l - 1)


def test_no_gradient_bytes_cross_pcie_and_swap_sets_follow_fig5a():
    """Fig. 5(a) / readings c5, c6: dW stays resident across the group (0 bytes), reset on device;
    forward swaps in W, swaps out stash; backward swaps in W and stash; update swaps K in and W', K' out."""
    cap = min_cap(MLP, **CFG1)
    s, ops = plan(MLP, **dict(CFG1, hbm_cap_bytes=cap))
    assert not any(o["cat"] == "grad" and o["kind"] in ("H2D", "D2H") for o in ops)
    compute = {o["idx"]: o for o in ops if o["stream"] == "compute"}
    for o in ops:
        if o["kind"] == "D2H":
            assert o["cat"] in ("stash", "state", "weight")
            src = [compute[w] for w in o["waits"] if w in compute]
            assert src, o
            task = src[-1]["kind"]
            assert (o["cat"], task) in {("stash", "FWD"), ("state", "UPD"), ("weight", "UPD")}, (o, task)
        if o["kind"] == "H2D":
            assert o["cat"] in ("stash", "state", "weight")


def test_uncapped_moves_only_inputs_and_loss():
    s, ops = plan(MLP, **dict(CFG1, hbm_cap_bytes=0))
    assert {o["kind"] for o in ops if o["stream"] in ("h2d", "d2h")} == {"INPUT", "LOSS_OUT"}
    assert s.pred_h2d_bytes == 2 * 32 * 256 * 4 and s.pred_d2h_bytes == 4 * 8


@pytest.mark.parametrize("mult", [4, 6, 8])
def test_spilled_stash_is_spread_over_the_backward(mult):
    """Equal-size stash entries: the spilled (layer, microbatch) entries are spread evenly over the
    backward order (layer L-1 first, microbatches in canonical order), so each one's swap-in
    overlaps the backward of resident entries; every spilled entry leaves once (D2H) and comes
    back once (H2D)."""
    L, m = 8, 2
    descs = synth.transformer_stack(L, 64, 4, 16, False)
    base = min_cap(descs, microbatches=m, microbatch_size=2, precision=1)
    s, ops = plan(descs, microbatches=m, microbatch_size=2, precision=1, hbm_cap_bytes=int(base * mult))
    out = sorted((o["l"], o["i"]) for o in ops if o["kind"] == "D2H" and o["cat"] == "stash")
    back = sorted((o["l"], o["i"]) for o in ops if o["kind"] == "H2D" and o["cat"] == "stash")
    assert out == back
    n = len(out)
    if 0 < n < L * m:
        expect = sorted((L - 1 - j // m, j % m) for j in range(L * m) if (j + 1) * n // (L * m) > j * n // (L * m))
        assert out == expect
    assert s.hazards == 0


@pytest.mark.parametrize("extra", [6, 8, 10, 12])
def test_streamed_state_is_spread_over_the_backward(extra):
    """With equal per-layer state, the layers whose master/m/v stream through the host are spread
    evenly over the backward order (each one's swap-in overlaps the backward of resident layers
    before it) instead of being the last ones updated; the plan stays hazard free."""
    L = 12
    descs = synth.transformer_stack(L, 256, 4, 128, True)
    kw = dict(microbatches=2, microbatch_size=2, precision=1, stash_policy=2)
    base = min_cap(descs, **kw)
    state = 12 * (12 * 256 * 256 + 13 * 256)
    s, ops = plan(descs, **dict(kw, hbm_cap_bytes=base + extra * state))
    streamed = sorted({o["l"] for o in ops if o["kind"] == "H2D" and o["cat"] == "state"}, reverse=True)
    n = len(streamed)
    assert 0 < n < L, streamed
    padded = next(o["bytes"] for o in ops if o["kind"] == "H2D" and o["cat"] == "state")
    assert s.resident_state_bytes == (L - n) * padded
    expect = sorted([L - 1 - j for j in range(L) if (j + 1) * n // L > j * n // L], reverse=True)
    assert streamed == expect
    pos = [L - 1 - l for l in streamed]  # backward positions
    gaps = [b - a for a, b in zip(pos, pos[1:])]
    assert not gaps or max(gaps) - min(gaps) <= 1, gaps
    assert s.hazards == 0


def test_config_validation_errors():
    with pytest.raises(H.HarmonyError) as e:
        plan([synth.LayerDesc(1, 64, 64, n_heads=5, seq_len=8)], microbatches=1, microbatch_size=1)
    assert e.value.code == H.HARMONY_E_INVALID_ARG  # d % h != 0
    with pytest.raises(H.HarmonyError) as e:
        plan([synth.LayerDesc(0, 12, 12)], microbatches=1, microbatch_size=1, precision=1)
    assert e.value.code == H.HARMONY_E_UNSUPPORTED  # bf16 needs widths % 8
    with pytest.raises(H.HarmonyError) as e:
        plan(MLP, microbatches=1, microbatch_size=1, weight_decay=0.1)
    assert e.value.code == H.HARMONY_E_UNSUPPORTED
    with pytest.raises(H.HarmonyError) as e:
        plan([synth.LayerDesc(0, 8, 16), synth.LayerDesc(0, 8, 8)], microbatches=1, microbatch_size=1)
    assert e.value.code == H.HARMONY_E_INVALID_ARG  # widths do not chain


def test_init_without_gpu_fails_cleanly():
    cfg = H.make_config(microbatches=1, microbatch_size=1)
    try:
        import torch
        if torch.cuda.is_available():
            pytest.skip("GPU present")
    except Exception:
        pass
    with pytest.raises(H.HarmonyError) as e:
        H.harmony_init(cfg)
    assert e.value.code in (H.HARMONY_E_CUDA, H.HARMONY_E_INVALID_ARG)


def test_plan_scales_to_paper_configs():
    for name in ("cfg2", "cfg3"):
        c = synth.CONFIGS[name]
        s, _ = plan(c["descs"](), microbatches=c["m"], microbatch_size=c["batch"] // c["m"], precision=1,
                    hbm_cap_bytes=c["cap"])
        assert s.hazards == 0 and s.arena_bytes <= c["cap"]
        assert s.pred_h2d_bytes > 10e9  # op-input stash spills: host-link bound


def test_plan_cfg3_at_a_quarter_of_its_state():
    """north_star's >= 4x claim as a plan: full cfg3 (48 blocks, d = 1600; 18 B/param of
    model + Adam state = 26.6 GB) under a 6 GiB cap is race-free, inside the cap, and streams nearly
    all of its state and stash each step (bench.py --workload cfg3s runs it)."""
    c = synth.CONFIGS["cfg3"]
    descs = c["descs"]()
    cap = 6 << 30
    n_params = sum(12 * d.d_in * d.d_in + 13 * d.d_in for d in descs)
    assert 18 * n_params > 4 * cap
    s, _ = plan(descs, microbatches=2, microbatch_size=4, precision=1, hbm_cap_bytes=cap, stash_policy=2)
    assert s.hazards == 0 and s.arena_bytes <= cap
    assert s.pred_h2d_bytes > 15e9 and s.pred_d2h_bytes > 15e9


def test_operator_split_column_panels_only_when_the_cap_forces_them():
    """Row a15 inside the step: an fp32 MLP layer whose working set does not fit the cap is
    decomposed into column-panel sub-tasks (each needs only W[:, panel]); the plan stays race-free and
    moves each panel's weights as the unsplit layer would (same total bytes per pass)."""
    from synth import LayerDesc, LAYER_MLP, ACT_GELU, ACT_NONE
    descs = [LayerDesc(LAYER_MLP, 256, 2048, act=ACT_GELU), LayerDesc(LAYER_MLP, 2048, 256, act=ACT_GELU),
             LayerDesc(LAYER_MLP, 256, 256, act=ACT_NONE)]
    kw = dict(microbatches=2, microbatch_size=8)
    base, _ = plan(descs, hbm_cap_bytes=1 << 40, **kw)
    counts = []
    for f in (2.0, 0.9, 0.4, 0.25):
        s, ops = plan(descs, hbm_cap_bytes=int(base.min_working_set_bytes * f), **kw)
        assert s.hazards == 0 and s.arena_bytes <= int(base.min_working_set_bytes * f)
        counts.append(sum(1 for o in ops if o["kind"] == "FWD"))
    assert counts[0] == 3 * 2  # fits: no split
    assert counts[1] > counts[0] and counts[3] > counts[2] > counts[1]  # more panels as the cap shrinks
    with pytest.raises(H.HarmonyError) as e:  # bf16 layers are not split: the cap is simply too small
        plan(descs, hbm_cap_bytes=int(base.min_working_set_bytes * 0.4), precision=1, **kw)
    assert e.value.code == H.HARMONY_E_CAP_TOO_SMALL


@pytest.mark.parametrize("G", [2, 4])
def test_microbatch_groups_interleave_backward_with_the_next_forward(G):
    """SURVEY §8(d) direction balance: G microbatch groups; group g's backward is interleaved layer by
    layer with group g+1's forward (stash fetches and spills on both host-link directions at once);
    each layer's update follows the LAST group's backward; the plan stays race-free."""
    descs = synth.transformer_stack(4, 128, 2, 128, True)
    kw = dict(microbatches=4, microbatch_size=2, precision=1, stash_policy=0)
    base, _ = plan(descs, hbm_cap_bytes=1 << 40, **kw)
    s, ops = plan(descs, hbm_cap_bytes=int(base.min_working_set_bytes * 1.5), groups=G, **kw)
    assert s.hazards == 0
    comp = [(o["kind"], o["l"], o["i"]) for o in ops if o["stream"] == "compute"]
    mg = 4 // G
    first_bwd = next(k for k, c in enumerate(comp) if c[0] == "BWD")
    assert all(c[2] < mg for c in comp[:first_bwd] if c[0] in ("FWD", "LOSS"))  # only group 0 before
    # after the first backward, the next group's forward tasks appear between backward tasks
    later_fwd = [k for k, c in enumerate(comp) if c[0] == "FWD" and c[2] >= mg]
    assert later_fwd and later_fwd[0] > first_bwd and later_fwd[0] < max(k for k, c in enumerate(comp) if c[0] == "BWD")
    for l in range(4):  # UPD(l) after every microbatch's backward of layer l
        upd = next(k for k, c in enumerate(comp) if c[0] == "UPD" and c[1] == l)
        assert all(k < upd for k, c in enumerate(comp) if c[0] == "BWD" and c[1] == l)
    with pytest.raises(H.HarmonyError):
        plan(descs, hbm_cap_bytes=0, groups=3, **kw)  # m % G != 0


def test_forward_pack_halves_the_forward_tasks_and_keeps_the_traffic():
    """SURVEY NEXT-4's pack size per pass: fwd_pack = 2 runs each layer's forward on
    two consecutive microbatches in one task (the backward stays per microbatch).  The plan stays
    race-free and inside the cap, has half the forward tasks, and moves exactly the same bytes."""
    c = synth.CONFIGS["cfg2"]
    kw = dict(microbatches=4, microbatch_size=16, precision=1, hbm_cap_bytes=c["cap"], stash_policy=2)
    one, ops1 = plan(c["descs"](), **kw)
    two, ops2 = plan(c["descs"](), fwd_pack=2, **kw)
    assert two.hazards == 0 and two.arena_bytes <= c["cap"]
    n1 = sum(o["kind"] == "FWD" for o in ops1)
    n2 = sum(o["kind"] == "FWD" for o in ops2)
    assert n1 == 24 * 4 and n2 == n1 // 2
    assert sum(o["kind"] == "BWD" for o in ops1) == sum(o["kind"] == "BWD" for o in ops2)
    assert (two.pred_h2d_bytes, two.pred_d2h_bytes) == (one.pred_h2d_bytes, one.pred_d2h_bytes)
    # outside its domain the pack is refused
    with pytest.raises(H.HarmonyError) as e:
        plan(c["descs"](), fwd_pack=2, **dict(kw, stash_policy=0))
    assert e.value.code == H.HARMONY_E_UNSUPPORTED
