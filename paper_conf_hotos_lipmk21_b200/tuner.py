"""Microbatch-size tuner (the paper's "task packing" knob: pack size and microbatch
size per pass).

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


def measure_on_device(descs, params, X, T, cfg: dict, steps=2, warmup=1):
    """A `measure` callable: builds a context per candidate and returns its mean device step time."""
    def run(m, b):
        with H.Harmony(descs, params, microbatches=m, microbatch_size=b, **cfg) as h:
            for _ in range(warmup):
                h.step(X, T)
            tot = 0.0
            for _ in range(steps):
                _, st = h.step(X, T)
                tot += st.step_seconds
        return tot / steps
    return run
