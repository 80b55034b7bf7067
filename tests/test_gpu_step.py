"""End-to-end parity of the swapped, microbatched, JIT-updated step (the C ABI) with the plain
full-batch fp64 oracle, on a B200.

Tolerances (BASELINE.json north_star, reading c16): relative L2 per tensor <= 1e-5 on the fp32
path, <= 2e-2 on the bf16 tensor-core path, for the loss, every gradient, W, m and sqrt(v) after
each of 3 steps.  Capped (swapping) and uncapped runs must be bit-identical (reading c21)."""
import json
import os

import numpy as np
import pytest

import oracle
import synth
from synth import LayerDesc, LAYER_MLP, ACT_RELU, ACT_NONE, pack, unpack

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")
from paper_conf_hotos_lipmk21_b200 import harmony as H  # noqa: E402

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def rel(a, b):
    a = np.asarray(a, np.float64); b = np.asarray(b, np.float64)
    nb = np.linalg.norm(b)
    return np.linalg.norm(a - b) / (nb if nb > 1e-30 else 1.0)


def run_gpu(descs, params, batches, **cfg):
    """Run len(batches) steps; returns per-step (loss, grads, W, m, v, stats)."""
    out = []
    with H.Harmony(descs, params, retain_grads=1, **cfg) as h:
        for X, T in batches:
            loss, st = h.step(np.ascontiguousarray(X), np.ascontiguousarray(T))
            out.append(dict(loss=loss, stats=st.as_dict(),
                            g=[h.read(l, H.HARMONY_GRAD) for l in range(len(descs))],
                            W=[h.read(l, H.HARMONY_PARAM) for l in range(len(descs))],
                            m=[h.read(l, H.HARMONY_ADAM_M) for l in range(len(descs))],
                            v=[h.read(l, H.HARMONY_ADAM_V) for l in range(len(descs))]))
        plan = h.plan().as_dict()
    return out, plan


def run_oracle(descs, params, batches, lr=1e-3):
    P = [p.astype(np.float64) for p in params]
    st = oracle.AdamState.zeros(P)
    out = []
    for X, T in batches:
        loss, grads, P, st = oracle.train_step(descs, P, st, X.astype(np.float64), T.astype(np.float64), lr=lr)
        out.append(dict(loss=loss, g=grads, W=P, m=st.m, v=st.v))
    return out


def compare(gpu, ref, tol):
    worst = {}
    for s, (a, b) in enumerate(zip(gpu, ref)):
        worst["loss"] = max(worst.get("loss", 0), abs(a["loss"] - b["loss"]) / abs(b["loss"]))
        for key in ("g", "W", "m"):
            for x, y in zip(a[key], b[key]):
                worst[key] = max(worst.get(key, 0), rel(x, y))
        for x, y in zip(a["v"], b["v"]):
            worst["sqrt_v"] = max(worst.get("sqrt_v", 0), rel(np.sqrt(np.maximum(x, 0)), np.sqrt(y)))
    for k, v in worst.items():
        assert v <= tol, (k, v, worst)
    return worst


def batches_for(descs, B, steps, precision):
    return [synth.gen_batch(descs, B, t, precision) for t in range(1, steps + 1)]


def bitwise_equal(a, b):
    for s1, s2 in zip(a, b):
        assert s1["loss"] == s2["loss"]
        for key in ("g", "W", "m", "v"):
            for x, y in zip(s1[key], s2[key]):
                assert np.array_equal(x.view(np.uint32), y.view(np.uint32)), key


# --------------------------------------------------------------------------------------- Appendix A
def test_appendix_a_bitwise_on_gpu():
    """the fp32 GPU path reproduces the hand-computed loss and gradients
    bit for bit (every intermediate is a short dyadic rational), W' within 1e-7."""
    g = json.load(open(os.path.join(GOLD, "appendix_a_mlp_step.json")))
    descs = [LayerDesc(LAYER_MLP, 2, 2, act=ACT_RELU), LayerDesc(LAYER_MLP, 2, 2, act=ACT_NONE)]
    params = [pack(descs[0], {"w": g["W1"], "b": g["b1"]}, np.float32),
              pack(descs[1], {"w": g["W2"], "b": g["b2"]}, np.float32)]
    X = np.array(g["x"], np.float32); T = np.array(g["t"], np.float32)
    (res,), _ = run_gpu(descs, params, [(X, T)], microbatches=2, microbatch_size=1)
    assert res["loss"] == g["loss_num"] / g["loss_den"]
    g1 = unpack(descs[0], res["g"][0]); g2 = unpack(descs[1], res["g"][1])
    assert np.array_equal(g1["w"], np.array(g["dW1"], np.float32)) and np.array_equal(g1["b"], np.array(g["db1"], np.float32))
    assert np.array_equal(g2["w"], np.array(g["dW2"], np.float32)) and np.array_equal(g2["b"], np.array(g["db2"], np.float32))
    W1 = unpack(descs[0], res["W"][0])
    assert np.max(np.abs(W1["w"] - np.array(g["W1_new"])) / np.abs(np.array(g["W1_new"]))) < 1e-7


# --------------------------------------------------------------------------------------- cfg1 (fp32, capped)
CFG1 = synth.CONFIGS["cfg1"]


def test_cfg1_mlp_fp32_matches_oracle_and_capped_equals_uncapped():
    descs = CFG1["descs"]()
    params = synth.gen_params(descs)
    batches = batches_for(descs, CFG1["batch"], 3, 0)
    kw = dict(microbatches=CFG1["m"], microbatch_size=CFG1["batch"] // CFG1["m"])
    capped, plan = run_gpu(descs, params, batches, hbm_cap_bytes=CFG1["cap"], **kw)
    assert plan["arena_bytes"] <= CFG1["cap"]
    st = capped[0]["stats"]
    assert st["h2d_weight_bytes"] + st["h2d_state_bytes"] + st["h2d_stash_bytes"] > 0  # it really swaps
    assert st["h2d_grad_bytes"] == 0
    ref = run_oracle(descs, params, batches)
    compare(capped, ref, 1e-5)
    uncapped, _ = run_gpu(descs, params, batches, hbm_cap_bytes=0, **kw)
    bitwise_equal(capped, uncapped)
    # ledger == plan
    assert st["h2d_bytes"] == plan["pred_h2d_bytes"] and st["d2h_bytes"] == plan["pred_d2h_bytes"]


def test_rerun_is_deterministic():
    descs = CFG1["descs"]()
    params = synth.gen_params(descs)
    batches = batches_for(descs, 32, 2, 0)
    a, _ = run_gpu(descs, params, batches, microbatches=4, microbatch_size=8, hbm_cap_bytes=CFG1["cap"])
    b, _ = run_gpu(descs, params, batches, microbatches=4, microbatch_size=8, hbm_cap_bytes=CFG1["cap"])
    bitwise_equal(a, b)


# --------------------------------------------------------------------------------------- transformer
def tiny_transformer(causal, precision, L=2, d=64, h=4, S=32, B=4, m=2):
    descs = synth.transformer_stack(L, d, h, S, causal)
    params = synth.gen_params(descs, precision)
    if precision == 0:  # larger weights so attention is non-trivial at fp32 parity
        params = [p * 1.0 for p in params]
    batches = batches_for(descs, B, 3, precision)
    return descs, params, batches, dict(microbatches=m, microbatch_size=B // m, precision=precision)


def teacher_forced(descs, params, batches, gpu, tol, lr=1e-3):
    """DESIGN.md reading c16a: per step, (i) the GPU gradient vs the oracle's full-batch gradient at
    the GPU's own pre-step weights, (ii) the GPU's W, m, sqrt(v) vs the oracle's Adam (fp64) applied
    to the GPU's pre-step state and its own gradient, (iii) the loss trajectory.  Adam's step
    lr*g/(|g|+eps) is ill-conditioned where g is a structural zero (e.g. the key bias: softmax is
    shift invariant), so the untouched trajectory would compare floating-point noise there."""
    W = [p.astype(np.float64) for p in params]
    m = [np.zeros_like(w) for w in W]; v = [np.zeros_like(w) for w in W]
    worst = dict(loss=0.0, g=0.0, W=0.0, m=0.0, sqrt_v=0.0)
    for t, ((X, T), st) in enumerate(zip(batches, gpu), start=1):
        loss, g_ref, _ = oracle.stack_loss_and_grads(descs, W, X.astype(np.float64), T.astype(np.float64))
        worst["loss"] = max(worst["loss"], abs(st["loss"] - loss) / abs(loss))
        for l in range(len(descs)):
            worst["g"] = max(worst["g"], rel(st["g"][l], g_ref[l]))
            W2, m2, v2 = oracle.adam_update(W[l], st["g"][l].astype(np.float64), m[l], v[l], t, lr, 0.9, 0.999, 1e-8)
            worst["W"] = max(worst["W"], rel(st["W"][l], W2))
            worst["m"] = max(worst["m"], rel(st["m"][l], m2))
            worst["sqrt_v"] = max(worst["sqrt_v"], rel(np.sqrt(st["v"][l]), np.sqrt(v2)))
        W = [w.astype(np.float64) for w in st["W"]]
        m = [x.astype(np.float64) for x in st["m"]]; v = [x.astype(np.float64) for x in st["v"]]
    for k, x in worst.items():
        assert x <= tol, (k, x, worst)
    return worst


@pytest.mark.parametrize("causal", [False, True])
def test_transformer_fp32_matches_oracle(causal):
    descs, params, batches, kw = tiny_transformer(causal, 0)
    gpu, _ = run_gpu(descs, params, batches, **kw)
    print("fp32 transformer teacher-forced worst rel", teacher_forced(descs, params, batches, gpu, 1e-5))


@pytest.mark.parametrize("S", [136, 256])  # 136: GEMM + softmax attention path; 256: fused tcgen05 attention
@pytest.mark.parametrize("causal", [False, True])
def test_transformer_bf16_matches_oracle_and_capped_bitwise(causal, S):
    descs, params, batches, kw = tiny_transformer(causal, 1, L=3, d=128, h=2, S=S, B=4, m=2)
    uncapped, plan = run_gpu(descs, params, batches, **kw)
    ref = run_oracle(descs, params, batches)
    w = compare(uncapped, ref, 2e-2)
    print("bf16 worst rel", w)
    s, _ = H.harmony_plan_dry(H.make_config(hbm_cap_bytes=1 << 40, **kw), descs, text_len=0)
    cap = int(s.min_working_set_bytes * 1.5)
    capped, plan_c = run_gpu(descs, params, batches, hbm_cap_bytes=cap, **kw)
    assert plan_c["arena_bytes"] <= cap
    assert capped[0]["stats"]["h2d_stash_bytes"] > 0 or capped[0]["stats"]["h2d_weight_bytes"] > 0
    bitwise_equal(capped, uncapped)


@pytest.mark.parametrize("bf16", [False, True])
def test_baseline_schedule_is_bitwise_identical_to_harmony_dp(bf16):
    """The per-GPU-virtualization baseline (Fig. 5(b): per-microbatch weight swaps, updates after the
    whole backward, gradients parked on the host) computes exactly what Harmony-DP computes (reading
    c4: no layer's W is read after its own backward), while moving (4m+1)|W| of weights instead of 3|W|."""
    if bf16:
        descs, params, batches, kw = tiny_transformer(True, 1, L=3, d=128, h=2, S=128, B=4, m=2)
    else:
        descs = CFG1["descs"]()
        params = synth.gen_params(descs)
        batches = batches_for(descs, CFG1["batch"], 2, 0)
        kw = dict(microbatches=CFG1["m"], microbatch_size=CFG1["batch"] // CFG1["m"])
    s, _ = H.harmony_plan_dry(H.make_config(hbm_cap_bytes=1 << 40, schedule=H.HARMONY_SCHED_PER_GPU_VIRT, **kw),
                              descs, text_len=0)
    cap = int(s.min_working_set_bytes * 1.2)
    a, pa = run_gpu(descs, params, batches, hbm_cap_bytes=cap, **kw)
    b, pb = run_gpu(descs, params, batches, hbm_cap_bytes=cap, schedule=H.HARMONY_SCHED_PER_GPU_VIRT, **kw)
    bitwise_equal(a, b)
    wa = a[-1]["stats"]["h2d_weight_bytes"] + a[-1]["stats"]["d2h_weight_bytes"]
    wb = b[-1]["stats"]["h2d_weight_bytes"] + b[-1]["stats"]["d2h_weight_bytes"]
    assert wb > wa, (wa, wb)
    assert b[-1]["stats"]["d2h_grad_bytes"] > 0


@pytest.mark.parametrize("S", [64, 128])
@pytest.mark.parametrize("policy", [1, 2, 3])
def test_transformer_bf16_recompute_policies_are_bitwise_identical(policy, S):
    """stash_policy 1 recomputes LN outputs and GeLU, 2 recomputes the whole block from its input, in
    the backward: the same kernels recompute the same bits, so the step is bit-identical to policy 0
    with fewer stash bytes; capped (swapping) runs included."""
    descs, params, batches, kw = tiny_transformer(True, 1, L=3, d=128, h=2, S=S, B=4, m=2)
    a, pa = run_gpu(descs, params, batches, **kw)
    b, pb = run_gpu(descs, params, batches, stash_policy=policy, **kw)
    bitwise_equal(a, b)
    assert pb["total_stash_bytes"] < pa["total_stash_bytes"]
    s, _ = H.harmony_plan_dry(H.make_config(hbm_cap_bytes=1 << 40, stash_policy=policy, **kw), descs, text_len=0)
    c, pc = run_gpu(descs, params, batches, stash_policy=policy, hbm_cap_bytes=int(s.min_working_set_bytes * 1.2), **kw)
    bitwise_equal(a, c)
    compare(b, run_oracle(descs, params, batches), 2e-2)


def test_device_pointer_inputs_match_host_inputs():
    descs = CFG1["descs"]()
    params = synth.gen_params(descs)
    X, T = synth.gen_batch(descs, 32, 1)
    with H.Harmony(descs, params, microbatches=4, microbatch_size=8, hbm_cap_bytes=CFG1["cap"]) as h:
        l1, s1 = h.step(torch.tensor(X, device="cuda"), torch.tensor(T, device="cuda"))
        assert s1.h2d_input_bytes == 0
    with H.Harmony(descs, params, microbatches=4, microbatch_size=8, hbm_cap_bytes=CFG1["cap"]) as h:
        l2, s2 = h.step(X, T)
        assert s2.h2d_input_bytes == 2 * X.nbytes
    assert l1 == l2


def test_step_errors():
    descs = CFG1["descs"]()
    params = synth.gen_params(descs)
    with H.Harmony(descs, params, microbatches=4, microbatch_size=8) as h:
        X, T = synth.gen_batch(descs, 32, 1)
        with pytest.raises(H.HarmonyError) as e:
            H.harmony_step(h.ctx, X, T, 31)
        assert e.value.code == H.HARMONY_E_INVALID_ARG
        with pytest.raises(H.HarmonyError) as e:
            H.harmony_read_state(h.ctx, 0, H.HARMONY_GRAD, params[0].size)
        assert e.value.code == H.HARMONY_E_BAD_STATE
    ctx = H.harmony_init(H.make_config(microbatches=1, microbatch_size=1))
    with pytest.raises(H.HarmonyError) as e:
        H.harmony_step(ctx, X, T, 1)
    assert e.value.code == H.HARMONY_E_BAD_STATE
    H.harmony_finalize(ctx)


def test_graph_replay_equals_eager_and_tracks_input_pointers():
    """Pinned or device inputs replay the captured CUDA graph (input copy nodes re-pointed every
    step); pageable inputs are staged into pinned buffers and replay it too; HARMONY_NO_GRAPH=1 issues
    the same program eagerly.  All bit-identical."""
    descs, params, batches, kw = tiny_transformer(True, 1, L=2, d=64, h=2, S=64, B=4, m=2)
    s, _ = H.harmony_plan_dry(H.make_config(hbm_cap_bytes=1 << 40, **kw), descs, text_len=0)
    kw["hbm_cap_bytes"] = int(s.min_working_set_bytes * 1.3)
    os.environ["HARMONY_NO_GRAPH"] = "1"
    try:
        eager, _ = run_gpu(descs, params, batches, **kw)
    finally:
        del os.environ["HARMONY_NO_GRAPH"]
    assert eager[0]["stats"]["graph"] == 0
    staged, _ = run_gpu(descs, params, batches, **kw)  # pageable numpy inputs
    assert staged[0]["stats"]["graph"] == 1
    bitwise_equal(eager, staged)
    pinned = [(torch.tensor(X).pin_memory(), torch.tensor(T).pin_memory()) for X, T in batches]
    res = []
    with H.Harmony(descs, params, retain_grads=1, **kw) as h:
        for X, T in pinned:
            loss, st = h.step(X, T)
            assert st.graph == 1
            res.append(dict(loss=loss, g=[h.read(l, H.HARMONY_GRAD) for l in range(len(descs))],
                            W=[h.read(l) for l in range(len(descs))],
                            m=[h.read(l, H.HARMONY_ADAM_M) for l in range(len(descs))],
                            v=[h.read(l, H.HARMONY_ADAM_V) for l in range(len(descs))]))
    bitwise_equal(eager, res)


@pytest.mark.parametrize("frac", [0.9, 0.25])
def test_operator_split_panels_match_oracle_and_are_bitwise_the_unsplit_step(frac):
    """Row a15 inside the step: under a cap smaller than the wide layers' working set the planner runs
    them as column-panel sub-tasks (forward and weight gradient split along N, dX one K reduction
    continued panel to panel); the result is the oracle's full-batch step (1e-5, fp32) and bit for bit
    the uncapped, unsplit run (reading c21)."""
    descs = [LayerDesc(LAYER_MLP, 256, 2048, act=synth.ACT_GELU), LayerDesc(LAYER_MLP, 2048, 256, act=synth.ACT_GELU),
             LayerDesc(LAYER_MLP, 256, 256, act=ACT_NONE)]
    params = synth.gen_params(descs)
    batches = batches_for(descs, 16, 3, 0)
    kw = dict(microbatches=2, microbatch_size=8)
    s, _ = H.harmony_plan_dry(H.make_config(hbm_cap_bytes=1 << 40, **kw), descs, text_len=0)
    cap = int(s.min_working_set_bytes * frac)
    split, plan = run_gpu(descs, params, batches, hbm_cap_bytes=cap, **kw)
    assert plan["arena_bytes"] <= cap and plan["n_ops"] > 40
    compare(split, run_oracle(descs, params, batches), 1e-5)
    whole, _ = run_gpu(descs, params, batches, hbm_cap_bytes=0, **kw)
    bitwise_equal(split, whole)


@pytest.mark.parametrize("G", [2, 4])
def test_microbatch_groups_are_bitwise_identical_to_one_group(G):
    """Direction-balancing microbatch groups only reorder tasks: the microbatches keep their canonical
    order in every dW accumulation, so any G gives the one-group step bit for bit (reading c21),
    capped with stash spills (op-input stash policy) included."""
    descs, params, batches, kw = tiny_transformer(True, 1, L=3, d=128, h=2, S=128, B=8, m=4)
    s, _ = H.harmony_plan_dry(H.make_config(hbm_cap_bytes=1 << 40, groups=G, **kw), descs, text_len=0)
    cap = int(s.min_working_set_bytes * 1.3)
    one, _ = run_gpu(descs, params, batches, hbm_cap_bytes=cap, **kw)
    grouped, plan = run_gpu(descs, params, batches, hbm_cap_bytes=cap, groups=G, **kw)
    assert grouped[0]["stats"]["h2d_stash_bytes"] > 0
    bitwise_equal(one, grouped)


def _step_in_subprocess(env, L, d, h, S, B, m):
    """Run tiny_transformer steps in a fresh process (library knobs are read once per process)."""
    import os
    import pickle
    import subprocess
    import sys
    import tempfile
    code = f"""
import pickle, sys
sys.path.insert(0, {repr(os.path.dirname(os.path.abspath(__file__)))})
sys.path.insert(0, {repr(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))})
from test_gpu_step import tiny_transformer, run_gpu
descs, params, batches, kw = tiny_transformer(False, 1, L={L}, d={d}, h={h}, S={S}, B={B}, m={m})
res, _ = run_gpu(descs, params, batches, **kw)
pickle.dump([{{k: r[k] for k in ('loss', 'g', 'W', 'm', 'v')}} for r in res], open(sys.argv[1], 'wb'))
"""
    with tempfile.NamedTemporaryFile(suffix=".pkl", delete=False) as f:
        path = f.name
    try:
        subprocess.run([sys.executable, "-c", code, path], check=True, env=dict(os.environ, **env), timeout=600)
        return pickle.load(open(path, "rb"))
    finally:
        os.unlink(path)


def test_per_kind_gemm_kernels_are_bitwise_the_generic_kernel():
    """The CTA-pair GEMM compiled per epilogue kind (default; the ACT_BWD one also column-sums its
    output for the FC1 bias gradient) vs the generic kernel + the separate 32-row-block column-sum
    pass (HARMONY_GEMM_SPECIALIZE=0): bit-identical steps.  d = 256, 3072 tokens per microbatch, so
    the FC2 dgrad runs on 48 CTA-pair tiles (the fused path)."""
    shape = dict(L=2, d=256, h=4, S=512, B=12, m=2)
    spec = _step_in_subprocess({}, **shape)
    generic = _step_in_subprocess({"HARMONY_GEMM_SPECIALIZE": "0"}, **shape)
    bitwise_equal(spec, generic)
    descs, params, batches, kw = tiny_transformer(False, 1, **shape)
    compare(spec, run_oracle(descs, params, batches), 2e-2)


def test_programmatic_dependent_launch_is_bitwise_plain_stream_order():
    """Every kernel is launched with programmatic stream serialisation and waits (griddepcontrol.wait)
    before touching global memory; the step must equal the one launched in plain stream order
    (HARMONY_PDL=0) bit for bit — a kernel reading its predecessor's output early would show here."""
    shape = dict(L=2, d=256, h=4, S=512, B=12, m=2)
    pdl = _step_in_subprocess({}, **shape)
    plain = _step_in_subprocess({"HARMONY_PDL": "0"}, **shape)
    bitwise_equal(pdl, plain)


@pytest.mark.parametrize("capped", [False, True])
def test_forward_pack_is_bitwise_the_per_microbatch_forward(capped):
    """fwd_pack = 2 (pack size per pass): each layer's forward runs on two consecutive
    microbatches in one task — GEMMs of 2*b*S rows, attention over 2*b sequences, LayerNorm per row —
    while the backward stays per microbatch.  Every output element keeps its reduction order, so the
    step is bit-identical to one forward task per microbatch, with stash spills (capped) or without,
    and matches the oracle."""
    descs, params, batches, kw = tiny_transformer(False, 1, L=3, d=128, h=2, S=128, B=8, m=4)
    kw["stash_policy"] = 2
    cap = 0
    if capped:
        s, _ = H.harmony_plan_dry(H.make_config(hbm_cap_bytes=1 << 40, fwd_pack=2, **kw), descs, text_len=0)
        cap = int(s.min_working_set_bytes * 1.2)
    one, plan1 = run_gpu(descs, params, batches, hbm_cap_bytes=cap, **kw)
    two, plan2 = run_gpu(descs, params, batches, hbm_cap_bytes=cap, fwd_pack=2, **kw)
    assert plan2["n_ops"] < plan1["n_ops"]
    if capped:
        assert two[0]["stats"]["d2h_stash_bytes"] > 0
    bitwise_equal(one, two)
    compare(two, run_oracle(descs, params, batches), 2e-2)
