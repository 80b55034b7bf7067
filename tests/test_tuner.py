"""Microbatch-size tuner: host logic on CPU with a synthetic step-time model; the
planner decides feasibility under the cap (harmony_plan_dry), the measurement picks the winner."""
import pytest

import synth
from paper_conf_hotos_lipmk21_b200 import harmony as H
from paper_conf_hotos_lipmk21_b200 import tuner


def test_candidates_divide_the_batch():
    assert tuner.candidates(64) == [1, 2, 4, 8, 16]
    assert tuner.candidates(6) == [1, 2]
    assert tuner.candidates(1) == [1]


def test_tuner_skips_infeasible_and_picks_fastest():
    descs = synth.transformer_stack(4, 64, 4, 16, False)
    cfg = dict(precision=1, stash_policy=2)
    # a cap the widest microbatch (m=1, 8 sequences) cannot meet, but m >= 2 can
    s1, _ = H.harmony_plan_dry(H.make_config(microbatches=1, microbatch_size=8, hbm_cap_bytes=1 << 40, **cfg), descs,
                               text_len=0)
    s2, _ = H.harmony_plan_dry(H.make_config(microbatches=2, microbatch_size=4, hbm_cap_bytes=1 << 40, **cfg), descs,
                               text_len=0)
    assert s2.min_working_set_bytes < s1.min_working_set_bytes
    cap = s2.min_working_set_bytes
    seen = []

    def measure(m, b):  # per-launch overhead vs. nothing else: fewer, larger microbatches win
        seen.append(m)
        return 1e-3 * m + 1e-4

    r = tuner.tune_microbatches(descs, 8, dict(cfg, hbm_cap_bytes=cap), measure)
    trials = {t.microbatches: t for t in r.trials}
    assert not trials[1].feasible and trials[1].reason
    assert 1 not in seen and r.best == 2
    d = r.as_dict()
    assert d["best_microbatches"] == 2 and len(d["trials"]) == len(tuner.candidates(8))


def test_tuner_breaks_ties_toward_larger_microbatches_and_raises_when_nothing_fits():
    descs = synth.mlp_stack(4, 256)
    r = tuner.tune_microbatches(descs, 32, dict(hbm_cap_bytes=0), lambda m, b: 1.0)
    assert r.best == 1
    with pytest.raises(H.HarmonyError):
        tuner.tune_microbatches(descs, 32, dict(hbm_cap_bytes=1024), lambda m, b: 1.0)


def test_tango_ranks_by_the_cost_model_and_measures_only_the_top():
    """(m, G, policy, forward pack): infeasible points are recorded, the feasible ones ranked by the
    plan-implied time (GEMM work vs host traffic with direction balance), only the top few are
    measured — plus, for each, its forward-pack-2 twin where the planner accepts one (same bytes and
    FLOPs: the model cannot rank it, so it is measured beside it)."""
    descs = synth.transformer_stack(4, 128, 2, 128, True)
    cfg = dict(precision=1)
    s, _ = H.harmony_plan_dry(H.make_config(microbatches=4, microbatch_size=2, stash_policy=2,
                                            hbm_cap_bytes=1 << 40), descs, text_len=0)
    cap = int(s.min_working_set_bytes * 1.6)
    seen = []

    def measure(m, G, pol, pack):
        seen.append((m, G, pol, pack))
        return 1.0 / m + 0.01 * G + 0.001 * pol - 0.0001 * pack

    best, cands = tuner.tune(descs, 8, dict(cfg, hbm_cap_bytes=cap), measure, top=3, per_policy=1,
                             incumbent=(2, 1, 2))
    feas = [c for c in cands if c.feasible]
    inc = (2, 1, 2, 1)
    assert best.key() in seen and inc in seen  # the incumbent is always measured
    singles = [k for k in seen if k[3] == 1 and k != inc]
    pols = [k[2] for k in singles]
    assert len(pols) == len(set(pols)) <= 3  # at most one per stash policy (per_policy=1)
    for k in singles:  # each measured non-incumbent candidate is its policy's best prediction
        c = next(c for c in feas if c.key() == k)
        assert c.pred_seconds == min(x.pred_seconds for x in feas if x.stash_policy == k[2])
    for k in seen:  # pack-2 twins: only for block recompute (the pack's domain), beside their pack-1 point
        if k[3] == 2:
            assert k[2] == 2 and k[:3] + (1,) in seen
    assert any(k[3] == 2 for k in seen)
    assert all(c.pred_seconds > 0 for c in feas)
    # more groups overlap the two host-link directions: never a worse prediction for the same plan bytes
    s0, _ = H.harmony_plan_dry(H.make_config(microbatches=4, microbatch_size=2, stash_policy=0, hbm_cap_bytes=cap,
                                             **cfg), descs, text_len=0)
    assert tuner.predict_seconds(s0, 0, 4) <= tuner.predict_seconds(s0, 0, 1)
