"""The N > 1 data path on one B200: a single-process group of N data-parallel ranks sharing the GPU
(harmony_init_group; SURVEY §8(b) primary mode), with the library's own collectives pulling from the
peers' arenas — the reduce-scatter of fp32 dW (rank-order sum), the sharded Adam on each rank's
shard, the all-gather of bf16/fp32 weight shards ("p2p swap") and of the loss partials.

Every result is compared with the plain full-batch fp64 oracle at the GLOBAL batch B = N*m*b
(the collectives "preserve the semantics"), within reading c16's budgets, and capped
(swapping) runs are bit-identical to uncapped ones at the same N (reading c21)."""
import numpy as np
import pytest

import synth
from test_gpu_step import (CFG1, batches_for, bitwise_equal, compare, run_gpu, run_oracle, tiny_transformer)

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")
from paper_conf_hotos_lipmk21_b200 import harmony as H  # noqa: E402


@pytest.mark.parametrize("N", [2, 4])
def test_group_mlp_fp32_matches_full_batch_oracle_and_capped_bitwise(N):
    descs = CFG1["descs"]()
    params = synth.gen_params(descs)
    m, b = CFG1["m"], CFG1["batch"] // CFG1["m"]
    batches = batches_for(descs, N * m * b, 3, 0)
    kw = dict(microbatches=m, microbatch_size=b, group=[0] * N)
    capped, plan = run_gpu(descs, params, batches, hbm_cap_bytes=CFG1["cap"], **kw)
    st = capped[-1]["stats"]
    assert st["nvlink_bytes"] > 0 and st["h2d_grad_bytes"] == 0
    assert st["h2d_weight_bytes"] + st["h2d_state_bytes"] > 0  # it really swaps
    w = compare(capped, run_oracle(descs, params, batches), 1e-5)
    print(f"N={N} fp32 group worst rel", w)
    uncapped, _ = run_gpu(descs, params, batches, hbm_cap_bytes=0, **kw)
    bitwise_equal(capped, uncapped)


def test_group_ledger_per_rank_equals_plan_and_weight_shards_cross_the_link_once():
    """Each rank swaps in only its 1/N shard of a streamed layer and all-gathers the rest over the
    GPU interconnect, so the box moves each streamed layer across the host link once per pass, not N
    times."""
    descs = CFG1["descs"]()
    params = synth.gen_params(descs)
    N, m, b = 2, 4, 8
    X, T = synth.gen_batch(descs, N * m * b, 1)
    cfg = dict(microbatches=m, microbatch_size=b, hbm_cap_bytes=CFG1["cap"])
    with H.Harmony(descs, params, group=[0] * N, **cfg) as h:
        _, tot = h.step(X, T)
        ranks = [h.rank_stats(r) for r in range(N)]
    preds = [H.harmony_plan_dry(H.make_config(rank=r, world_size=N, **cfg), descs, text_len=0)[0] for r in range(N)]
    for r in range(N):
        assert ranks[r].h2d_bytes == preds[r].pred_h2d_bytes and ranks[r].d2h_bytes == preds[r].pred_d2h_bytes
        assert ranks[r].h2d_weight_bytes == preds[r].pred_h2d_weight_bytes
    assert tot.h2d_bytes == sum(r.h2d_bytes for r in ranks)
    # streamed layers: the ranks' weight swap-ins together equal one copy per pass (2 passes + shards)
    one, _ = H.harmony_plan_dry(H.make_config(**dict(cfg, hbm_cap_bytes=CFG1["cap"])), descs, text_len=0)
    if one.pred_h2d_weight_bytes and preds[0].resident_weight_bytes == one.resident_weight_bytes:
        assert sum(p.pred_h2d_weight_bytes for p in preds) == one.pred_h2d_weight_bytes


@pytest.mark.parametrize("causal", [False, True])
def test_group_transformer_bf16_matches_oracle_and_capped_bitwise(causal):
    N = 2
    descs, params, _, kw = tiny_transformer(causal, 1, L=3, d=128, h=2, S=256, B=4, m=2)
    batches = batches_for(descs, N * 4, 3, 1)
    kw["group"] = [0] * N
    uncapped, _ = run_gpu(descs, params, batches, **kw)
    w = compare(uncapped, run_oracle(descs, params, batches), 2e-2)
    print("bf16 group worst rel", w)
    cfg = {k: v for k, v in kw.items() if k != "group"}
    s, _ = H.harmony_plan_dry(H.make_config(hbm_cap_bytes=1 << 40, rank=0, world_size=N, **cfg), descs, text_len=0)
    capped, plan = run_gpu(descs, params, batches, hbm_cap_bytes=int(s.min_working_set_bytes * 1.3), **kw)
    assert capped[0]["stats"]["h2d_weight_bytes"] + capped[0]["stats"]["h2d_stash_bytes"] > 0
    bitwise_equal(capped, uncapped)


def test_group_of_one_is_bitwise_the_single_rank_context():
    descs = CFG1["descs"]()
    params = synth.gen_params(descs)
    batches = batches_for(descs, 32, 2, 0)
    kw = dict(microbatches=4, microbatch_size=8, hbm_cap_bytes=CFG1["cap"])
    a, _ = run_gpu(descs, params, batches, **kw)
    b, _ = run_gpu(descs, params, batches, group=[0], **kw)
    bitwise_equal(a, b)


def test_group_graph_replay_equals_eager():
    """Pinned inputs: the N ranks' programs are captured as ONE CUDA graph (every rank's streams and
    the collectives' rendezvous events) and replayed; HARMONY_NO_GRAPH=1 issues the same program
    eagerly.  Bit-identical."""
    import os
    N = 2
    descs, params, _, kw = tiny_transformer(True, 1, L=2, d=64, h=2, S=64, B=4, m=2)
    batches = batches_for(descs, N * 4, 3, 1)
    kw["group"] = [0] * N
    os.environ["HARMONY_NO_GRAPH"] = "1"
    try:
        eager, _ = run_gpu(descs, params, batches, **kw)
    finally:
        del os.environ["HARMONY_NO_GRAPH"]
    assert eager[0]["stats"]["graph"] == 0
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


def test_group_n2_agrees_with_single_rank_on_the_same_global_batch():
    """Same global batch of 64 rows: one rank with m=8 microbatches vs two ranks with m=4 each. The
    fp32 summation grouping differs (microbatches, then ranks; reading c8), so the tolerance applies."""
    descs = CFG1["descs"]()
    params = synth.gen_params(descs)
    batches = batches_for(descs, 64, 2, 0)
    one, _ = run_gpu(descs, params, batches, microbatches=8, microbatch_size=8)
    two, _ = run_gpu(descs, params, batches, microbatches=4, microbatch_size=8, group=[0, 0])
    for a, b in zip(one, two):
        assert abs(a["loss"] - b["loss"]) <= 1e-6 * abs(a["loss"])
        for x, y in zip(a["W"], b["W"]):
            assert np.linalg.norm(x - y) <= 1e-5 * np.linalg.norm(x)


def test_group_errors():
    descs = CFG1["descs"]()
    params = synth.gen_params(descs)
    with H.Harmony(descs, params, group=[0, 0], microbatches=4, microbatch_size=8) as h:
        X, T = synth.gen_batch(descs, 32, 1)
        with pytest.raises(H.HarmonyError) as e:
            H.harmony_step(h.ctx, X, T, 32)  # the group takes the global batch (64 rows)
        assert e.value.code == H.HARMONY_E_INVALID_ARG
        with pytest.raises(H.HarmonyError) as e:
            H.harmony_set_profiling(h.ctx, 1)
        assert e.value.code == H.HARMONY_E_UNSUPPORTED


def test_group_with_microbatch_groups_is_bitwise_one_group():
    """N = 2 ranks sharing the GPU, each with G = 2 microbatch groups: bit-identical to G = 1 (the
    groups only reorder tasks; the reduce-scatter still follows each layer's last microbatch)."""
    descs = CFG1["descs"]()
    params = synth.gen_params(descs)
    batches = batches_for(descs, 2 * 32, 2, 0)
    kw = dict(microbatches=4, microbatch_size=8, group=[0, 0], hbm_cap_bytes=CFG1["cap"])
    a, _ = run_gpu(descs, params, batches, **kw)
    b, _ = run_gpu(descs, params, batches, groups=2, **kw)
    bitwise_equal(a, b)
