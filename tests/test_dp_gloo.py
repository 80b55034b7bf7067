"""Data-parallel host logic with world_size 2 over gloo on CPU (no GPU):
  * every rank's static program issues the same collectives in the same order with the same
    message sizes (no deadlock by construction), and the per-layer shards partition
    the layer;
  * the DP decomposition the library implements preserves the single-device semantics
    (P:135-136): rank-local oracle gradients of each rank's rows (1/B_global scaling, reading c14)
    summed across ranks equal the full-batch gradient; the K-split operator decomposition
     summed across ranks equals the plain GEMM."""
import os
import re
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import synth
from paper_conf_hotos_lipmk21_b200 import harmony as H


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        out = {}
        # ---- 1. identical collective sequence on every rank
        descs = synth.transformer_stack(4, 64, 4, 16, True)
        cfg = H.make_config(rank=rank, world_size=world, microbatches=2, microbatch_size=2, precision=1,
                            hbm_cap_bytes=0)
        s, txt = H.harmony_plan_dry(cfg, descs)
        comm = [tuple(re.split(r"\s+", l)[1:2] + [l.split("l=")[1].split()[0], l.split("bytes=")[1].split()[0]])
                for l in txt.splitlines()[1:] if " comm " in l]
        seqs = [None] * world
        dist.all_gather_object(seqs, comm)
        out["same_collectives"] = all(x == seqs[0] for x in seqs) and len(comm) > 0
        out["hazards"] = s.hazards
        # capped run with streamed weights: all-gather of weight shards appears
        cap = int(H.harmony_plan_dry(H.make_config(rank=rank, world_size=world, microbatches=2, microbatch_size=2,
                                                   precision=1, hbm_cap_bytes=1 << 40), descs, text_len=0)[0]
                  .min_working_set_bytes)
        s2, txt2 = H.harmony_plan_dry(H.make_config(rank=rank, world_size=world, microbatches=2, microbatch_size=2,
                                                    precision=1, hbm_cap_bytes=cap), descs)
        out["capped_hazards"] = s2.hazards
        out["has_allgather"] = "ALLGATHER" in txt2 and "REDUCESCATTER" in txt2
        # ---- 2. DP gradient semantics: rank rows, global 1/B, sum over ranks == full batch
        mdescs = synth.mlp_stack(3, 16)
        params = [p.astype(np.float64) for p in synth.gen_params(mdescs)]
        B = 8
        X, T = synth.gen_batch(mdescs, B, 1)
        rows = slice(rank * B // world, (rank + 1) * B // world)
        loss, grads, _ = oracle.stack_loss_and_grads(mdescs, params, X[rows], T[rows], loss_batch=B)
        flat = torch.tensor(np.concatenate(grads + [np.array([loss])]))
        dist.all_reduce(flat)  # the reduce-scatter + all-gather sum the library performs
        full_loss, full_g, _ = oracle.stack_loss_and_grads(mdescs, params, X, T)
        ref = np.concatenate(full_g + [np.array([full_loss])])
        out["dp_rel"] = float(np.linalg.norm(flat.numpy() - ref) / np.linalg.norm(ref))
        # ---- 3. K-split operator decomposition: partials summed (reduce-scatter) == plain GEMM
        M, N, K = 16, 12, 32
        Xg, Wg, dYg = synth.gen_gemm_operands(M, N, K)
        ks = slice(rank * K // world, (rank + 1) * K // world)
        part = torch.tensor(Xg[:, ks].astype(np.float64) @ Wg[ks, :].astype(np.float64))
        dist.all_reduce(part)
        Y_ref, dX_ref, dW_ref = oracle.gemm_fwd_bwd(Xg, Wg, dYg)
        my_rows = slice(rank * M // world, (rank + 1) * M // world)
        out["split_rel"] = float(np.linalg.norm(part.numpy()[my_rows] - Y_ref[my_rows]) / np.linalg.norm(Y_ref[my_rows]))
        dX_loc = dYg.astype(np.float64) @ Wg[ks, :].astype(np.float64).T
        out["split_dx_rel"] = float(np.linalg.norm(dX_loc - dX_ref[:, ks]) / np.linalg.norm(dX_ref[:, ks]))
        q.put((rank, out))
    finally:
        dist.destroy_process_group()


def test_dp_world2_gloo():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=240) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    for r in range(world):
        o = res[r]
        assert o["same_collectives"], o
        assert o["hazards"] == 0 and o["capped_hazards"] == 0
        assert o["has_allgather"]
        assert o["dp_rel"] < 1e-12
        assert o["split_rel"] < 1e-12 and o["split_dx_rel"] < 1e-12
