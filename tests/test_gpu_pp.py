"""Harmony-PP on one B200 (ranks sharing the GPU; the activation / gradient hand-offs are device
copies between the ranks' arenas): the result is the plain full-batch step of the oracle at the
minibatch B = m*b, and bit for bit the single-rank Harmony-DP step with the same m, b
(same kernels, same microbatch accumulation order; reading c21) — capped or not, eager or replayed."""
import numpy as np
import pytest

import synth
from test_gpu_step import batches_for, bitwise_equal, compare, run_gpu, run_oracle, tiny_transformer

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")
from paper_conf_hotos_lipmk21_b200 import harmony as H  # noqa: E402

PP = H.HARMONY_SCHED_HARMONY_PP


def pp_cap(descs, N, **kw):
    s, _ = H.harmony_plan_dry_group(H.make_config(schedule=PP, hbm_cap_bytes=1 << 40, **kw), N, descs, text_len=0)
    return int(s.min_working_set_bytes * 1.1)


@pytest.mark.parametrize("N", [2, 4])
def test_pp_mlp_fp32_matches_oracle_and_is_bitwise_the_single_rank_step(N):
    descs = synth.mlp_stack(8, 256)  # two or more layers per rank, so a capped rank must stream
    params = synth.gen_params(descs)
    m, b = 4, 8
    batches = batches_for(descs, m * b, 3, 0)
    kw = dict(microbatches=m, microbatch_size=b)
    cap = pp_cap(descs, N, **kw)
    pp, _ = run_gpu(descs, params, batches, group=[0] * N, schedule=PP, hbm_cap_bytes=cap, **kw)
    st = pp[-1]["stats"]
    assert st["nvlink_bytes"] > 0 and st["h2d_weight_bytes"] > 0
    compare(pp, run_oracle(descs, params, batches), 1e-5)
    dp, _ = run_gpu(descs, params, batches, hbm_cap_bytes=0, **kw)
    bitwise_equal(pp, dp)
    unc, _ = run_gpu(descs, params, batches, group=[0] * N, schedule=PP, hbm_cap_bytes=0, **kw)
    bitwise_equal(pp, unc)


def test_pp_weight_ledger_is_3W_and_equals_the_plan():
    descs = synth.mlp_stack(4, 256)
    params = synth.gen_params(descs)
    m, b, N = 4, 8, 2
    kw = dict(microbatches=m, microbatch_size=b)
    s, _ = H.harmony_plan_dry_group(H.make_config(schedule=PP, hbm_cap_bytes=1 << 40, **kw), N, descs, text_len=0)
    cap = int(s.min_working_set_bytes * 1.02)
    plan, _ = H.harmony_plan_dry_group(H.make_config(schedule=PP, hbm_cap_bytes=cap, **kw), N, descs, text_len=0)
    X, T = synth.gen_batch(descs, m * b, 1)
    with H.Harmony(descs, params, group=[0] * N, schedule=PP, hbm_cap_bytes=cap, **kw) as h:
        _, st = h.step(X, T)
    assert st.h2d_bytes == plan.pred_h2d_bytes and st.d2h_bytes == plan.pred_d2h_bytes
    W = sum(-(-d.n_params() // 1024) * 1024 * 4 for d in descs)
    assert plan.resident_weight_bytes == 0
    assert st.h2d_weight_bytes == 2 * W and st.d2h_weight_bytes == W  # 3|W| for the box


@pytest.mark.parametrize("causal", [False, True])
def test_pp_transformer_bf16_matches_oracle_and_single_rank_bitwise(causal):
    descs, params, batches, kw = tiny_transformer(causal, 1, L=4, d=128, h=2, S=256, B=4, m=2)
    kw["stash_policy"] = 2
    pp, _ = run_gpu(descs, params, batches, group=[0, 0], schedule=PP, hbm_cap_bytes=pp_cap(descs, 2, **kw), **kw)
    w = compare(pp, run_oracle(descs, params, batches), 2e-2)
    print("pp bf16 worst rel", w)
    dp, _ = run_gpu(descs, params, batches, **kw)
    bitwise_equal(pp, dp)


def test_pp_graph_replay_equals_eager():
    descs, params, batches, kw = tiny_transformer(True, 1, L=3, d=64, h=2, S=64, B=4, m=2)
    kw.update(group=[0, 0, 0], schedule=PP)
    eager, _ = run_gpu(descs, params, batches, **kw)
    res = []
    with H.Harmony(descs, params, retain_grads=1, **kw) as h:
        for X, T in batches:
            loss, st = h.step(torch.tensor(X).pin_memory(), torch.tensor(T).pin_memory())
            assert st.graph == 1
            res.append(dict(loss=loss, g=[h.read(l, H.HARMONY_GRAD) for l in range(len(descs))],
                            W=[h.read(l) for l in range(len(descs))],
                            m=[h.read(l, H.HARMONY_ADAM_M) for l in range(len(descs))],
                            v=[h.read(l, H.HARMONY_ADAM_V) for l in range(len(descs))]))
    bitwise_equal(eager, res)
