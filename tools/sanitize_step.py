"""Small steps for compute-sanitizer (memcheck / racecheck / synccheck): the cfg1 MLP fp32 step under
its cap (swapping), a tiny bf16 transformer (tcgen05 GEMMs, fused attention) under a cap, and a
2-rank loopback group.  Eager issue (HARMONY_NO_GRAPH=1 is set by the caller) so every launch is
checked individually.
    compute-sanitizer --tool memcheck python tools/sanitize_step.py"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synth  # noqa: E402
from paper_conf_hotos_lipmk21_b200 import harmony as H  # noqa: E402

which = sys.argv[1:] or ["cfg1", "tiny", "pack", "group"]
if "cfg1" in which:
    descs = synth.mlp_stack(4, 256)
    params = synth.gen_params(descs)
    X, T = synth.gen_batch(descs, 32, 1)
    with H.Harmony(descs, params, microbatches=4, microbatch_size=8, hbm_cap_bytes=synth.CONFIGS["cfg1"]["cap"]) as h:
        for _ in range(2):
            print("cfg1 loss", h.step(X, T)[0])
if "tiny" in which:
    descs = synth.transformer_stack(2, 128, 2, 128, True)
    params = synth.gen_params(descs, 1)
    X, T = synth.gen_batch(descs, 4, 1, 1)
    kw = dict(microbatches=2, microbatch_size=2, precision=1)
    for pol in (0, 2):
        s, _ = H.harmony_plan_dry(H.make_config(hbm_cap_bytes=1 << 40, stash_policy=pol, **kw), descs, text_len=0)
        with H.Harmony(descs, params, hbm_cap_bytes=int(s.min_working_set_bytes * 1.2), stash_policy=pol, **kw) as h:
            for _ in range(2):
                print("tiny policy", pol, "loss", h.step(X, T)[0])
if "pack" in which:  # forward packs (two microbatches per forward task), capped with stash spills
    descs = synth.transformer_stack(2, 128, 2, 128, False)
    params = synth.gen_params(descs, 1)
    X, T = synth.gen_batch(descs, 8, 1, 1)
    kw = dict(microbatches=4, microbatch_size=2, precision=1, stash_policy=2, fwd_pack=2)
    s, _ = H.harmony_plan_dry(H.make_config(hbm_cap_bytes=1 << 40, **kw), descs, text_len=0)
    with H.Harmony(descs, params, hbm_cap_bytes=int(s.min_working_set_bytes * 1.2), **kw) as h:
        for _ in range(2):
            print("pack loss", h.step(X, T)[0])
if "group" in which:
    descs = synth.mlp_stack(4, 256)
    params = synth.gen_params(descs)
    X, T = synth.gen_batch(descs, 64, 1)
    with H.Harmony(descs, params, group=[0, 0], microbatches=4, microbatch_size=8,
                   hbm_cap_bytes=synth.CONFIGS["cfg1"]["cap"]) as h:
        for _ in range(2):
            print("group loss", h.step(X, T)[0])
print("SANITIZE_DONE")
