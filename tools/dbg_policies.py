"""Debug helper: compare capped vs uncapped runs of one stash policy (bitwise)."""
import sys
sys.path.insert(0, '.')
import numpy as np  # noqa: E402
import synth  # noqa: E402
from paper_conf_hotos_lipmk21_b200 import harmony as H  # noqa: E402

for S in (64, 128):
    for pol in (0, 2):
        descs = synth.transformer_stack(3, 128, 2, S, True)
        params = synth.gen_params(descs, 1)
        X, T = synth.gen_batch(descs, 4, 1, 1)
        kw = dict(microbatches=2, microbatch_size=2, precision=1, stash_policy=pol)
        s, txt = H.harmony_plan_dry(H.make_config(hbm_cap_bytes=1 << 40, **kw), descs, text_len=0)
        res = {}
        for cap in (0, int(s.min_working_set_bytes * 1.2)):
            with H.Harmony(descs, params, retain_grads=1, hbm_cap_bytes=cap, **kw) as h:
                loss, st = h.step(X, T)
                res[cap] = (loss, [h.read(l, H.HARMONY_GRAD) for l in range(3)], h.plan().as_dict())
        caps = list(res)
        print("S", S, "policy", pol, "loss", res[caps[0]][0], res[caps[1]][0], "plan", {k: res[caps[1]][2][k] for k in ("weight_slots", "stash_slots", "state_slots", "resident_stash_bytes", "resident_weight_bytes")})
        for l in range(3):
            a, b = res[caps[0]][1][l], res[caps[1]][1][l]
            print("  layer", l, "maxdiff", np.abs(a - b).max())
