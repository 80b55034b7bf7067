"""Performance tuner (the paper's "memory-performance tango" and task-packing knobs,
P:749-757, 783-810): microbatch count, microbatch groups (direction balance), stash policy and the
forward pack size (microbatches per forward task).

The same global batch per GPU can be run as m microbatches of b = batch / m sequences.  Larger
microbatches amortise every kernel's launch and tail cost; a wider microbatch also widens the
task workspace, which under a fixed HBM cap pushes block inputs (stash) and streamed state out to
the host link.  Which m is fastest depends on the model, the cap and the link, so the tuner asks
the planner which candidates fit the cap (host-only `harmony_plan_dry`) and then times a few steps
of each feasible one through the C ABI (device time of the step program, CUDA events in the
library).  Configuration-time orchestration only: every step it times runs the library's program.
"""
from __future__ import annotations

from dataclasses import dataclass, field

from . import harmony as H


@dataclass
class Trial:
    microbatches: int
    microbatch_size: int
    feasible: bool
    reason: str = ""
    pred_h2d_bytes: int = 0
    pred_d2h_bytes: int = 0
    step_seconds: float | None = None


@dataclass
class TuneResult:
    best: int
    trials: list = field(default_factory=list)

    def as_dict(self):
        return {"best_microbatches": self.best,
                "trials": [dict(m=t.microbatches, b=t.microbatch_size, feasible=t.feasible, reason=t.reason,
                                pred_h2d_bytes=t.pred_h2d_bytes, pred_d2h_bytes=t.pred_d2h_bytes,
                                ms_per_step=None if t.step_seconds is None else t.step_seconds * 1e3)
                           for t in self.trials]}


def candidates(batch: int, limit=(1, 2, 4, 8, 16)):
    """Microbatch counts that divide the per-GPU batch."""
    return [m for m in limit if m <= batch and batch % m == 0]


def tune_microbatches(descs, batch: int, cfg: dict, measure, cands=None) -> TuneResult:
    """Pick the microbatch count m (batch = m * b) with the smallest measured step time.

    cfg     -- harmony config keywords without microbatches / microbatch_size (cap, precision, ...)
    measure -- callable(m, b) -> seconds per step (e.g. a few timed steps through the C ABI)
    Candidates the planner rejects under the cap are recorded as infeasible and not measured.
    Ties go to the larger microbatch (fewer tasks)."""
    trials = []
    for m in (cands or candidates(batch)):
        b = batch // m
        t = Trial(m, b, True)
        try:
            s, _ = H.harmony_plan_dry(H.make_config(microbatches=m, microbatch_size=b, **cfg), descs, text_len=0)
            t.pred_h2d_bytes, t.pred_d2h_bytes = int(s.pred_h2d_bytes), int(s.pred_d2h_bytes)
        except H.HarmonyError as e:
            t.feasible, t.reason = False, str(e)
        if t.feasible:
            t.step_seconds = float(measure(m, b))
        trials.append(t)
    ok = [t for t in trials if t.feasible]
    if not ok:
        raise H.HarmonyError(H.HARMONY_E_CAP_TOO_SMALL, "no microbatch count fits the cap")
    best = min(ok, key=lambda t: (t.step_seconds, t.microbatches))
    return TuneResult(best.microbatches, trials)


# ------------------------------------------------------------------------------------------------ (m, G, policy)
@dataclass
class Candidate:
    microbatches: int
    groups: int
    stash_policy: int
    fwd_pack: int = 1                   # microbatches per forward task (the backward's pack is 1)
    feasible: bool = True
    reason: str = ""
    pred_seconds: float | None = None   # cost model (host-only plan + link / tensor rates)
    step_seconds: float | None = None   # measured (top candidates only)

    def key(self):
        return (self.microbatches, self.groups, self.stash_policy, self.fwd_pack)


# executed GEMM FLOPs per algorithmic FLOP: block recompute re-runs the forward (without its last
# projection, ~2/3 of it); policy 3 also skips the attention forward — the same to this model
EXEC = {0: 1.0, 1: 1.0, 2: 1.0 + 1.0 / 3.0 * 0.67 + 0.1, 3: 1.0 + 1.0 / 3.0 * 0.67}


def predict_seconds(summary, policy, groups, tflops=1000.0, link_gbs=55.0):
    """The step time the plan implies: the slower of its GEMM work at `tflops` and its host traffic at
    `link_gbs` per direction, where one group moves the forward's spills and the backward's fetches in
    two phases (the sum) and G groups overlap all but 1/G of them (SURVEY §8(d) direction balance)."""
    compute = summary.flops_per_step * EXEC.get(policy, 1.0) / (tflops * 1e12)
    h2d, d2h = summary.pred_h2d_bytes / 1e9, summary.pred_d2h_bytes / 1e9
    overlapped = max(h2d, d2h) + min(h2d, d2h) / groups
    return max(compute, overlapped / link_gbs)


def tune(descs, batch: int, cfg: dict, measure, ms=None, groups=(1, 2, 4), policies=(0, 2, 3), top=4,
         per_policy=2, incumbent=None, packs=(1, 2), **model) -> "tuple[Candidate, list]":
    """The memory-performance tango: over microbatch count m, microbatch groups G and stash
    policy, the planner says what fits the cap, a cost model ranks what fits, and the best-ranked are
    measured (`measure(m, G, policy)` -> seconds per step); the fastest measured wins.  The model only
    ranks (it knows GEMM work and host traffic, not kernel efficiency), so the measured set takes at
    most `per_policy` candidates of each stash policy (up to `top` in all) plus the `incumbent`
    (m, G, policy) when given.  The fp32 path has no recompute policies (0 only).  Forward packs of 2
    (where the planner accepts them) move the same bytes and FLOPs, so the model cannot rank them:
    each measured candidate's pack-2 twin is measured beside it.  `measure(m, G, policy, pack)`."""
    if cfg.get("precision", 0) == 0:
        policies = (0,)
    cands = []
    for m in (ms or candidates(batch)):
        for G in groups:
            if m % G:
                continue
            for pol in policies:
                for pack in packs:
                    c = Candidate(m, G, pol, pack)
                    try:
                        s, _ = H.harmony_plan_dry(H.make_config(microbatches=m, microbatch_size=batch // m, groups=G,
                                                                stash_policy=pol, fwd_pack=pack, **cfg), descs,
                                                  text_len=0)
                        c.pred_seconds = predict_seconds(s, pol, G, **model)
                    except H.HarmonyError as e:
                        c.feasible, c.reason = False, str(e)
                        if pack > 1:
                            continue  # outside the pack's domain: not a candidate
                    cands.append(c)
    ok = sorted((c for c in cands if c.feasible), key=lambda c: (c.pred_seconds, c.groups, c.fwd_pack))
    if not ok:
        raise H.HarmonyError(H.HARMONY_E_CAP_TOO_SMALL, "no (microbatches, groups, policy) fits the cap")
    chosen, taken = [], {}
    for c in ok:
        if len(chosen) >= top:
            break
        if c.fwd_pack == 1 and taken.get(c.stash_policy, 0) < per_policy:
            chosen.append(c)
            taken[c.stash_policy] = taken.get(c.stash_policy, 0) + 1
    if incumbent is not None:
        inc_key = tuple(incumbent) + ((1,) if len(incumbent) == 3 else ())
        inc = next((c for c in ok if c.key() == inc_key), None)
        if inc is not None and inc not in chosen:
            chosen.append(inc)
    twins = [t for c in chosen for t in ok
             if t.fwd_pack > 1 and t.key()[:3] == c.key()[:3] and t not in chosen]
    for c in chosen + twins:
        c.step_seconds = float(measure(c.microbatches, c.groups, c.stash_policy, c.fwd_pack))
    best = min((c for c in ok if c.step_seconds is not None), key=lambda c: (c.step_seconds, c.groups))
    return best, cands


def measure_on_device(descs, params, X, T, cfg: dict, steps=2, warmup=1):
    """A `measure` callable: builds a context per candidate and returns its mean device step time."""
    def run(m, b, **extra):
        with H.Harmony(descs, params, microbatches=m, microbatch_size=b, **dict(cfg, **extra)) as h:
            for _ in range(warmup):
                h.step(X, T)
            tot = 0.0
            for _ in range(steps):
                _, st = h.step(X, T)
                tot += st.step_seconds
        return tot / steps
    return run
