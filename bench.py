"""Benchmark of the Harmony-DP step (BASELINE.json metric: samples/sec/step under an HBM cap,
swap GB/s and % of roofline).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload cfg2] [--impl ours|reference]

N=1: the workload BASELINE.json's metric is quoted on that fits one GPU — configs[1], BERT-Large
(24 pre-LN blocks, d=1024, h=16, S=512), 64 sequences per GPU as 2 microbatches of 32, bf16 tensor-core
compute with fp32 master weights + Adam, per-GPU HBM cap 8 GiB.  N>1 (torchrun, one process per
GPU; `--gpus N` without torchrun re-launches itself under torchrun): the same per-GPU work on every
rank (weak scaling), data-parallel with NCCL reduce-scatter of gradients and all-gather of weight
shards inside the library.

`value` = samples / device time of the K timed steps (CUDA events on the library's streams,
inputs resident in HBM, max over ranks).  `e2e` = the same through the C ABI with pinned HOST
inputs (the H2D of X and T and the D2H of the loss inside the timed region), host wall clock.
`--impl reference` times the CPU oracle (fp64 NumPy): one complete full-depth step at batch 1,
split over the K timed steps; `cpu_baseline` is the same complete step, timed once.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import synth  # noqa: E402

PEAKS_FILE = os.path.join(ROOT, "MEASURED_PEAKS.json")
# per-launch DRAM traffic of the roofline kernel class, from the committed ncu launch list of the
# same step (tools/traffic_summary.py); ncu replays cold, so this is the no-L2-reuse upper end
TRAFFIC_FILES = {"cfg2": os.path.join(ROOT, "profiles", "r02_traffic_cfg2_m2.json")}
FALLBACK = {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0}

WORKLOADS = {
    "cfg2": dict(name="cfg2: BERT-Large 24L d1024 h16 S512, 64 seq/GPU (m=2 x b=32), bf16/fp32-master Adam, "
                      "HBM cap 8 GiB/GPU", model="bert-large-like-preLN", descs=lambda: synth.transformer_stack(24, 1024, 16, 512, False),
                 per_gpu_batch=64, m=2, cap=8 << 30, S=512),
    "cfg3": dict(name="cfg3: GPT-2 XL 48L d1600 h25 S1024 causal, 8 seq/GPU (m=2 x b=4), bf16/fp32-master Adam, "
                      "HBM cap 16 GiB/GPU", model="gpt2-xl-like-preLN", descs=lambda: synth.transformer_stack(48, 1600, 25, 1024, True),
                 per_gpu_batch=8, m=2, cap=16 << 30, S=1024),
    # north_star's ">= 4x the capped HBM": full cfg3 (18 B/param: 26.6 GB of model and
    # optimizer state) under a 6 GiB cap, 4.1x; nearly every weight, state shard and stash crosses the
    # host link each step, so the strict swap roofline is the bound
    "cfg3s": dict(name="cfg3s: GPT-2 XL 48L d1600 h25 S1024 causal, 8 seq/GPU (m=2 x b=4), bf16/fp32-master Adam, "
                       "HBM cap 6 GiB/GPU (model + Adam state 4.1x the cap)", model="gpt2-xl-like-preLN",
                  descs=lambda: synth.transformer_stack(48, 1600, 25, 1024, True), per_gpu_batch=8, m=2, cap=6 << 30,
                  S=1024),
    "cfg4s": dict(name="cfg4s: 8 of cfg4's 36 GPT blocks (d5120 h40 S1024 causal, 2.5B params), 8 seq/GPU (m=4 x b=2), "
                       "bf16/fp32-master Adam, weights + Adam state streamed from pinned host (HBM cap 12 GiB/GPU)",
                  model="gpt-11b-like-preLN-8-of-36", descs=lambda: synth.transformer_stack(8, 5120, 40, 1024, True),
                  per_gpu_batch=8, m=4, cap=12 << 30, S=1024),
    "cfg5": dict(name="cfg5: one 16384 x 16384 x 65536 (M x N x K) bf16 GEMM fwd+bwd, operator split along K into "
                      "8 row-chunk tile subtasks per GPU (harmony_split_gemm_*)", model="gemm-16384x16384x65536",
                 M=16384, N=16384, K=65536, chunks=8, S=1, per_gpu_batch=1, m=1, cap=0),
    "cfg1": dict(name="cfg1: 4-layer MLP d256, batch 32 as 4 microbatches, fp32, cap = 2 layers' state",
                 model="mlp4-d256", descs=lambda: synth.mlp_stack(4, 256), per_gpu_batch=32, m=4,
                 cap=2 * 16 * (256 * 256 + 256), S=1, precision=0),
}


def load_peaks():
    try:
        with open(PEAKS_FILE) as f:
            p = json.load(f)
        return p, "measured"
    except Exception:
        return FALLBACK, "fallback"


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region (B200_PROFILING.md)."""

    def __init__(self, index=0):
        self.index = index
        self.samples = []
        self.proc = None

    def start(self):
        q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
             "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
             "clocks_event_reasons.sw_power_cap")
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={q}",
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.thread = threading.Thread(target=self._read, daemon=True)
            self.thread.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            f = [x.strip() for x in line.split(",")]
            if len(f) >= 8:
                self.samples.append(f)

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        sm = [float(s[0]) for s in self.samples if s[0].replace(".", "").isdigit()]
        mx = [float(s[1]) for s in self.samples if s[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for s in self.samples for i in range(4) if s[4 + i].lower() == "active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.samples)}


def host_link_bandwidth(torch, device):
    """Pinned H2D, D2H and concurrent duplex GB/s (1 GiB in 128 MiB chunks, best of 3)."""
    GiB, chunk = 1 << 30, 128 << 20
    hs = torch.empty(GiB, dtype=torch.uint8).pin_memory()
    hd = torch.empty(GiB, dtype=torch.uint8).pin_memory()
    d1 = torch.empty(GiB, dtype=torch.uint8, device=device)
    d2 = torch.empty(GiB, dtype=torch.uint8, device=device)
    s1, s2 = torch.cuda.Stream(device), torch.cuda.Stream(device)
    out = {}
    for mode in ("h2d", "d2h", "duplex"):
        best = 0.0
        for _ in range(3):
            torch.cuda.synchronize(device)
            t0 = time.perf_counter()
            n = 0
            for off in range(0, GiB, chunk):
                if mode in ("h2d", "duplex"):
                    with torch.cuda.stream(s1):
                        d1[off:off + chunk].copy_(hs[off:off + chunk], non_blocking=True)
                    n += chunk
                if mode in ("d2h", "duplex"):
                    with torch.cuda.stream(s2):
                        hd[off:off + chunk].copy_(d2[off:off + chunk], non_blocking=True)
                    n += chunk
            torch.cuda.synchronize(device)
            best = max(best, n / (time.perf_counter() - t0) / 1e9)
        out[mode] = best
    del hs, hd, d1, d2
    return out


def nvlink_probe(torch, dist, device, layer_params, world, reps=10):
    """Phase 0 of SURVEY §8(d) at N > 1: NCCL reduce-scatter (fp32) and all-gather (bf16) bus bandwidth at
    the step's per-layer message sizes, all ranks at once (a separate NCCL group; max time over ranks)."""
    g = dist.new_group(backend="nccl")
    n = (layer_params + world * 1024 - 1) // (world * 1024) * (world * 1024)
    out = {}
    for name, dt, op in (("reduce_scatter_f32", torch.float32, "rs"), ("all_gather_bf16", torch.bfloat16, "ag")):
        full = torch.ones(n, dtype=dt, device=device)
        shard = torch.empty(n // world, dtype=dt, device=device)
        def run():
            if op == "rs":
                dist.reduce_scatter_tensor(shard, full, group=g)
            else:
                dist.all_gather_into_tensor(full, shard, group=g)
        for _ in range(3):
            run()
        torch.cuda.synchronize(device)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        dist.barrier(group=g)
        e0.record()
        for _ in range(reps):
            run()
        e1.record()
        torch.cuda.synchronize(device)
        t = torch.tensor([e0.elapsed_time(e1) / reps / 1e3], dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        sec = t.item()
        nbytes = n * full.element_size()
        out[name] = {"bytes": nbytes, "us": sec * 1e6, "busbw_gbs": nbytes * (world - 1) / world / sec / 1e9}
    return out


def oracle_step_work(wl, batch=1):
    """One complete oracle training step of the workload's full stack (every layer: forward, the
    loss, backward, Adam) on `batch` sequences, as a list of work items in the step's order (the
    oracle's own block functions, called as oracle.stack_loss_and_grads / train_step call them).
    Returns (items, n_samples); each item is a no-argument callable."""
    import oracle
    from oracle.layers import transformer_block_bwd, mlp_layer_bwd
    descs = wl["descs"]()
    prec = wl.get("precision", 1)
    params = [p.astype(np.float64) for p in synth.gen_params(descs, prec)]
    X, T = synth.gen_batch(descs, batch, 1, prec)
    X, T = X.astype(np.float64), T.astype(np.float64)
    st = {"A": X, "caches": [None] * len(descs), "grads": [None] * len(descs)}
    state = oracle.AdamState.zeros(params)
    items = []

    def fwd(l):
        def f():
            A, caches = oracle.stack_forward([descs[l]], [params[l]], st["A"].reshape(batch, -1, descs[l].d_in))
            st["A"], st["caches"][l] = A, caches[0]
        return f

    def loss():
        st["loss"], st["A"] = oracle.mse_loss(st["A"], T, batch)

    def bwd(l):
        def f():
            p, c = st["caches"][l]
            if descs[l].kind == synth.LAYER_MLP:
                st["A"], g = mlp_layer_bwd(st["A"], c, p, descs[l].act)
            else:
                st["A"], g = transformer_block_bwd(st["A"], c, p)
            st["grads"][l] = synth.pack(descs[l], g)
            st["caches"][l] = None
        return f

    def adam(l):
        def f():
            params[l], state.m[l], state.v[l] = oracle.adam_update(params[l], st["grads"][l], state.m[l], state.v[l],
                                                                   1, 1e-4, 0.9, 0.999, 1e-8)
        return f

    L = len(descs)
    items += [fwd(l) for l in range(L)] + [loss] + [bwd(l) for l in range(L - 1, -1, -1)] + [adam(l) for l in range(L)]
    return items, batch


def cores_used():
    return len(os.sched_getaffinity(0)) if hasattr(os, "sched_getaffinity") else os.cpu_count()


def cpu_oracle_full_step(wl, batch=1):
    """The fp64 oracle (as it stands) timed on one COMPLETE training step of the full-depth workload
    at a batch of `batch` sequences: every layer's forward and backward, the loss and Adam over all
    parameters (about 40 s for cfg2 on a 16-core host).  value = batch / measured seconds."""
    items, n = oracle_step_work(wl, batch)
    t0 = time.perf_counter()
    for f in items:
        f()
    dt = time.perf_counter() - t0
    L = len(wl["descs"]())
    B = wl["per_gpu_batch"]
    desc = (f"fp64 NumPy oracle, one complete step of all {L} layers (fwd, loss, bwd, Adam on every parameter) at "
            f"batch {n} sequence(s) of the workload's shape: {dt:.1f} s measured")
    return n / dt, desc, cores_used(), dt


def run_reference(args, wl, metric, unit):
    """--impl reference: the oracle on the box's host cores.  The K timed steps together run ONE
    complete full-depth oracle training step at batch 1 (its work items — layer forwards, loss, layer
    backwards, Adam per layer — split into K consecutive slices, one per timed step), so the run stays
    within minutes and `value` = 1 sample / the measured time of that whole step (no extrapolation)."""
    items, n = oracle_step_work(wl, 1)
    warm, _ = oracle_step_work(dict(wl, descs=lambda: wl["descs"]()[:1]), 1)
    for f in warm[:max(0, min(args.warmup, len(warm)))]:
        f()
    K = max(1, args.steps)
    bounds = [round(i * len(items) / K) for i in range(K + 1)]
    times = []
    for k in range(K):
        t0 = time.perf_counter()
        for f in items[bounds[k]:bounds[k + 1]]:
            f()
        times.append(time.perf_counter() - t0)
    total = sum(times)
    value = n / total
    L = len(wl["descs"]())
    desc = (f"fp64 NumPy oracle, one complete step of all {L} layers (fwd, loss, bwd, Adam) at batch 1 sequence, "
            f"its {len(items)} work items split over the {K} timed steps: {total:.1f} s measured")
    line = {"impl": "reference", "metric": metric, "value": value, "unit": unit, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": total / K * 1e3, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": wl["name"], "global_batch": wl["per_gpu_batch"] * max(args.gpus, 1),
                       "seq_len": wl["S"], "parallelism": f"dp{args.gpus}"},
            "cpu_baseline": {"value": value, "unit": unit, "cores": cores_used(), "kind": "oracle", "sample": desc},
            "e2e": {"value": value, "unit": unit, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line))


def run_cfg5(args, wl, world, rank, local, torch, H):
    """Row a15: Y = X.W fwd + dX, dW bwd of one large GEMM, K split over the ranks (reading c19);
    each rank runs its K-slice as `chunks` row-chunk tile subtasks (reduce-scatter of the fp32
    partials over NCCL when world > 1, all-gather of dY).  Metric: whole-job TFLOP/s (3 x 2MNK
    per step), device time (CUDA events on the library's compute stream), max over ranks."""
    torch.cuda.set_device(local)
    device = torch.device("cuda", local)
    dist = None
    nccl_id = None
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("gloo", init_method="env://")
        obj = [H.harmony_get_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        nccl_id = obj[0]
    M, N, K = wl["M"], wl["N"], wl["K"]
    Kr, Mr = K // world, M // world
    g = torch.Generator(device=device)
    g.manual_seed(7 + rank)
    bf = torch.bfloat16
    X = torch.randn(M, Kr, device=device, generator=g).to(bf)
    W = (torch.randn(Kr, N, device=device, generator=g) / (K ** 0.5)).to(bf)
    dY = torch.randn(Mr, N, device=device, generator=g).to(bf)
    Y = torch.empty(Mr, N, device=device)
    dX = torch.empty(M, Kr, device=device, dtype=bf)
    dW = torch.empty(Kr, N, device=device)
    flops = 3 * 2.0 * M * N * K  # whole job per step
    with H.SplitGemm(M, N, K, chunks=wl["chunks"], rank=rank, world_size=world, device=local, precision=1,
                     nccl_id=nccl_id) as sg:
        for _ in range(args.warmup):
            sg.run(X, W, dY, Y, dX, dW)
        clocks = ClockSampler(local)
        clocks.start()
        torch.cuda.synchronize(device)
        if dist is not None:
            dist.barrier()
        dev_s = sum(sg.run(X, W, dY, Y, dX, dW) for _ in range(args.steps))
        torch.cuda.synchronize(device)
        clk = clocks.stop()
        # e2e: this rank's operand slices from pinned host memory, Y shard back, host wall clock
        Xh, Wh, dYh = X.cpu().pin_memory(), W.cpu().pin_memory(), dY.cpu().pin_memory()
        Yh = torch.empty(Mr, N).pin_memory()
        torch.cuda.synchronize(device)
        t0 = time.perf_counter()
        for _ in range(max(1, args.steps // 2)):
            X.copy_(Xh, non_blocking=True); W.copy_(Wh, non_blocking=True); dY.copy_(dYh, non_blocking=True)
            sg.run(X, W, dY, Y, dX, dW)
            Yh.copy_(Y, non_blocking=True)
            torch.cuda.synchronize(device)
        e2e_s = (time.perf_counter() - t0) / max(1, args.steps // 2)
    if dist is not None:
        t = torch.tensor([dev_s, e2e_s], dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        dev_s, e2e_s = t.tolist()
    if rank != 0:
        return
    peaks, peak_src = load_peaks()
    tflops = flops * args.steps / dev_s / 1e12
    peak = peaks.get("bf16_tflops_sustained", peaks["bf16_tflops"]) * world
    line = {"metric": "TFLOP/s of the operator-split GEMM fwd+bwd (cfg5)", "value": tflops, "unit": "TFLOP/s",
            "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "ms_per_step": dev_s / args.steps * 1e3,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "bf16",
            "data": "synthetic (torch.randn on device, seeded)",
            "config": {"workload": wl["name"], "M": M, "N": N, "K": K, "chunks": wl["chunks"], "parallelism": f"ksplit{world}",
                       "l2": "operands 4.3 GB + outputs 7 GB per step, far larger than L2; no flush"},
            "roofline": {"bound": "tensor", "kernel": "gemm_tc2_kernel (all GEMM launches of the step)",
                         "achieved": tflops, "peak": peak, "unit": "TFLOP/s", "frac": tflops / peak, "traffic": None,
                         "peak_source": f"{peak_src} bf16_tflops_sustained x {world} GPU(s)"},
            "e2e": {"value": flops / e2e_s / 1e12, "unit": "TFLOP/s",
                    "h2d_bytes_per_step": (X.numel() + W.numel() + dY.numel()) * 2, "d2h_bytes_per_step": Y.numel() * 4,
                    "timing": "host wall clock: pinned H2D of this rank's operands + run + D2H of its Y shard"},
            "gpu_launches": None, "clocks": clk}
    print(json.dumps(line))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--workload", default="cfg2", choices=sorted(WORKLOADS))
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--stash-policy", type=int, default=2)
    ap.add_argument("--schedule", default="harmony", choices=["harmony", "baseline"],
                    help="harmony: Harmony-DP; baseline: the paper's per-GPU-virtualization comparison (Fig. 5(b))")
    ap.add_argument("--tune", action="store_true",
                    help="pick microbatches, groups and stash policy by the tuner (planner feasibility, a cost model, "
                         "then 2 timed steps of the best-ranked candidates)")
    ap.add_argument("--microbatches", type=int, default=0,
                    help="m per GPU (0 = the workload's default); the microbatch size is per_gpu_batch / m")
    ap.add_argument("--groups", type=int, default=1,
                    help="G microbatch groups (direction balance: group g's backward interleaved with g+1's forward)")
    ap.add_argument("--cap-gib", type=float, default=0,
                    help="override the workload's per-GPU HBM cap (GiB; A/B runs, reported in config)")
    ap.add_argument("--fwd-pack", type=int, default=1,
                    help="forward pack size (2: each layer's forward on two microbatches at once; NEXT-4)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    wl = dict(WORKLOADS[args.workload])
    if args.cap_gib:
        wl["cap"] = int(args.cap_gib * (1 << 30))
        wl["name"] = wl["name"] + f" [cap overridden: {args.cap_gib:g} GiB]"
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        # one process per GPU: launch this script under torchrun with args.gpus ranks
        import socket
        with socket.socket() as sk:
            sk.bind(("127.0.0.1", 0))
            port = sk.getsockname()[1]
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
               "--master-addr=127.0.0.1", f"--master-port={port}", os.path.abspath(__file__)] + sys.argv[1:]
        sys.exit(subprocess.call(cmd))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        raise SystemExit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world} (launch one rank per GPU)")
    # NCCL (one process per GPU): a fixed algorithm and protocol keep the reduce-scatter's summation
    # order the same from run to run (reading c21); the caller's environment wins
    os.environ.setdefault("NCCL_ALGO", "Ring")
    os.environ.setdefault("NCCL_PROTO", "Simple")
    metric = "samples/sec/step under HBM cap"
    unit = "samples/s"

    if args.impl == "reference":
        if rank == 0 and args.workload != "cfg5":
            run_reference(args, wl, metric, unit)
        elif rank == 0:
            print(json.dumps({"impl": "reference", "unavailable": "cfg5 is a single GEMM; its oracle is sampled dot "
                                                                  "products (tests), not a throughput program"}))
        return

    import torch
    from paper_conf_hotos_lipmk21_b200 import harmony as H

    if args.workload == "cfg5":
        return run_cfg5(args, wl, world, rank, local, torch, H)
    torch.cuda.set_device(local)
    device = torch.device("cuda", local)
    dist = None
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("gloo", init_method="env://")
    precision = wl.get("precision", 1)
    descs = wl["descs"]()
    B = wl["per_gpu_batch"]
    m = args.microbatches or wl["m"]
    nccl_id = None
    if world > 1:
        obj = [H.harmony_get_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        nccl_id = obj[0]
    t_setup = time.perf_counter()
    params = synth.gen_params(descs, precision)
    tuning = None
    if args.tune and world == 1:
        from paper_conf_hotos_lipmk21_b200 import tuner
        Xt, Tt = synth.gen_batch(descs, B, 1, precision)
        Xt, Tt = torch.tensor(Xt, device=device), torch.tensor(Tt, device=device)
        tcfg = dict(hbm_cap_bytes=wl["cap"], precision=precision, lr=1e-4)
        run = tuner.measure_on_device(descs, params, Xt, Tt, tcfg, steps=3, warmup=2)
        best, cands = tuner.tune(descs, B, tcfg, lambda mm, G, pol, pk=1: run(mm, B // mm, groups=G, stash_policy=pol,
                                                                              fwd_pack=pk),
                                 incumbent=(m, args.groups, args.stash_policy if precision else 0), link_gbs=55.0)
        m, args.groups, args.stash_policy = best.microbatches, best.groups, best.stash_policy
        args.fwd_pack = best.fwd_pack
        tuning = {"best": dict(microbatches=m, groups=best.groups, stash_policy=best.stash_policy,
                               fwd_pack=best.fwd_pack),
                  "candidates": [dict(m=c.microbatches, G=c.groups, policy=c.stash_policy, fwd_pack=c.fwd_pack,
                                      feasible=c.feasible,
                                      pred_ms=None if c.pred_seconds is None else c.pred_seconds * 1e3,
                                      ms=None if c.step_seconds is None else c.step_seconds * 1e3) for c in cands]}
        del Xt, Tt
        torch.cuda.empty_cache()
    cfg = dict(rank=rank, world_size=world, device=local, hbm_cap_bytes=wl["cap"], microbatches=m,
               microbatch_size=B // m, precision=precision, stash_policy=args.stash_policy if precision else 0,
               lr=1e-4, nccl_id=nccl_id, groups=args.groups, fwd_pack=args.fwd_pack,
               schedule=H.HARMONY_SCHED_PER_GPU_VIRT if args.schedule == "baseline" else H.HARMONY_SCHED_HARMONY_DP)
    h = H.Harmony(descs, params, **cfg)
    del params
    plan = h.plan().as_dict()
    setup_s = time.perf_counter() - t_setup
    # this rank's rows of the global batch (reading c14); resident inputs for `value`
    X, T = synth.gen_batch(descs, B * world, 1, precision)
    X = X[rank * B:(rank + 1) * B]
    T = T[rank * B:(rank + 1) * B]
    Xd, Td = torch.tensor(X, device=device), torch.tensor(T, device=device)
    Xh, Th = torch.tensor(X).pin_memory(), torch.tensor(T).pin_memory()

    def barrier():
        torch.cuda.synchronize(device)
        if dist is not None:
            dist.barrier()

    # host link measured concurrently on every rank (they share the host's PCIe / memory system);
    # the slowest rank's figures bound the step
    barrier()
    bw = host_link_bandwidth(torch, device)
    nvlink = None
    if dist is not None:
        t = torch.tensor([-bw["h2d"], -bw["d2h"], -bw["duplex"]], dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        bw = {"h2d": -t[0].item(), "d2h": -t[1].item(), "duplex": -t[2].item(), "ranks": world}
        try:
            nvlink = nvlink_probe(torch, dist, device, descs[0].n_params(), world)
        except Exception as e:  # the probe is informative only
            nvlink = {"error": str(e)[:200]}
    for _ in range(args.warmup):
        h.step(Xd, Td)
    # ---- timed region: device-resident inputs, CUDA-graph replay of the step program
    clocks = ClockSampler(local)
    clocks.start()
    barrier()
    dev_s, losses, stats = 0.0, [], []
    wall0 = time.perf_counter()
    for _ in range(args.steps):
        loss, st = h.step(Xd, Td)
        dev_s += st.step_seconds
        losses.append(loss)
        stats.append(st.as_dict())
    barrier()
    wall = time.perf_counter() - wall0
    clk = clocks.stop()
    # ---- kernel roofline pass: the same steps with per-launch CUDA events (eager issue)
    H.harmony_set_profiling(h.ctx, 1)
    prof_s = 0.0
    for _ in range(args.steps):
        _, pst = h.step(Xd, Td)
        prof_s += pst.step_seconds
    prof = H.harmony_read_profile(h.ctx).as_dict()
    H.harmony_set_profiling(h.ctx, 0)
    # ---- e2e: pinned host inputs through the C ABI, host wall clock
    barrier()
    e0 = time.perf_counter()
    e2e_stats = []
    for _ in range(args.steps):
        loss, st = h.step(Xh, Th)
        e2e_stats.append(st.as_dict())
    barrier()
    e2e_wall = time.perf_counter() - e0
    # the same through the C ABI with PAGEABLE host arrays (numpy): the library stages them into
    # pinned memory itself and still replays the step's graph
    Xp, Tp = np.ascontiguousarray(X), np.ascontiguousarray(T)
    barrier()
    p0 = time.perf_counter()
    for _ in range(args.steps):
        h.step(Xp, Tp)
    barrier()
    pageable_wall = time.perf_counter() - p0
    if dist is not None:
        t = torch.tensor([dev_s, wall, e2e_wall, pageable_wall], dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        dev_s, wall, e2e_wall, pageable_wall = t.tolist()
    h.close()
    if rank != 0:
        return

    peaks, peak_src = load_peaks()
    samples = B * world * args.steps
    value = samples / dev_s
    ms = dev_s / args.steps * 1e3
    s0 = stats[-1]
    h2d = s0["h2d_bytes"]; d2h = s0["d2h_bytes"]
    # step roofline (north_star): slower of GEMM FLOPs at tensor peak and swap bytes at host-link BW
    F = plan["flops_per_step"]
    t_gemm = F / (peaks["bf16_tflops"] * 1e12)
    t_strict = max(h2d / (bw["h2d"] * 1e9), d2h / (bw["d2h"] * 1e9), (h2d + d2h) / (bw["duplex"] * 1e9))
    t_lenient = (h2d + d2h) / (max(bw["h2d"], bw["d2h"]) * 1e9)
    t_roof = max(t_gemm, t_strict)
    # the roofline GIVEN THE CAP: the cap decides how much must be stashed, swapped or recomputed, so
    # take the best stash policy's max(executed GEMM FLOPs at peak, its planned swap bytes at the link)
    cap_aware = None
    if precision == 1 and descs[0].kind == synth.LAYER_TRANSFORMER and world == 1:
        d0, S0, L0 = descs[0].d_in, descs[0].seq_len, len(descs)
        Tm = (B // m) * S0
        recomp = {2: 16.0 * Tm * d0 * d0 + 4.0 * (B // m) * S0 * S0 * d0, 3: 16.0 * Tm * d0 * d0}
        per = {}
        for pol in (0, 1, 2, 3):
            try:
                sp, _ = H.harmony_plan_dry(H.make_config(**dict(cfg, stash_policy=pol, arena=None)), descs, text_len=0)
            except H.HarmonyError:
                continue
            fx = F + recomp.get(pol, 0.0) * m * L0
            tg = fx / (peaks["bf16_tflops"] * 1e12)
            hh, dd = sp.pred_h2d_bytes, sp.pred_d2h_bytes
            ts = max(hh / (bw["h2d"] * 1e9), dd / (bw["d2h"] * 1e9), (hh + dd) / (bw["duplex"] * 1e9))
            per[pol] = {"t_ms": max(tg, ts) * 1e3, "t_gemm_ms": tg * 1e3, "t_swap_ms": ts * 1e3, "exec_flops": fx}
        if per:
            best = min(per, key=lambda k: per[k]["t_ms"])
            cap_aware = {"t_roof_ms": per[best]["t_ms"], "policy": best, "frac": per[best]["t_ms"] / ms,
                         "per_policy": per,
                         "note": "min over stash policies of max(executed GEMM FLOPs / burst peak, planned swap bytes "
                                 "at the measured host link) under this cap"}
    g = prof["gemm"]
    gemm_tflops = g["work"] / g["seconds"] / 1e12 if g["seconds"] else 0.0
    gemm_peak = peaks.get("bf16_tflops_sustained", peaks["bf16_tflops"])
    adam = prof["adam"]
    traffic = traffic_src = None
    try:
        with open(TRAFFIC_FILES[args.workload]) as f:
            tj = json.load(f)
        traffic = tj["classes"]["gemm"]["dram_bytes_per_launch"]
        traffic_src = (f"{os.path.relpath(TRAFFIC_FILES[args.workload], ROOT)}: ncu dram__bytes_read.sum + "
                       f"dram__bytes_write.sum averaged over the {tj['classes']['gemm']['launches']} tcgen05 GEMM "
                       f"launches of the profiled step (cold-cache replay)")
    except (KeyError, OSError, ValueError):
        pass
    line = {
        "metric": metric, "value": value, "unit": unit, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "bf16" if precision else "f32", "data": "synthetic (seeded, paper-shaped)",
        "config": {"workload": wl["name"], "global_batch": B * world, "seq_len": wl["S"],
                   "microbatches": m, "microbatch_size": B // m, "schedule": args.schedule, "groups": args.groups,
                   "fwd_pack": args.fwd_pack,
                   **({"tuning": tuning} if tuning else {}),
                   "parallelism": f"dp{world}", "hbm_cap_bytes_per_gpu": wl["cap"],
                   "arena_bytes": plan["arena_bytes"], "stash_policy": cfg["stash_policy"],
                   "l2": "inputs and per-step swap traffic (tens of GB) far larger than the 126 MB L2; no flush"},
        "roofline": {"bound": "tensor", "kernel": "gemm_tc2_kernel / gemm_tc_kernel (tcgen05, all GEMM launches of the step)",
                     "achieved": gemm_tflops, "peak": gemm_peak, "unit": "TFLOP/s",
                     "frac": gemm_tflops / gemm_peak if gemm_peak else None, "traffic": traffic,
                     "traffic_unit": "bytes per launch", "traffic_source": traffic_src,
                     "algorithmic_flops_per_launch": g["work"] / g["launches"] if g["launches"] else None,
                     "peak_source": f"{peak_src} bf16_tflops_sustained (kernel timed inside a long step)",
                     "launches_per_step": g["launches"] / args.steps,
                     "flops_per_step": g["work"] / args.steps,
                     # overlapping GEMM launches (compute stream + weight-gradient side stream) each count
                     # their full span above; over the union of the class's launch intervals instead:
                     "achieved_while_running": g["work"] / g["busy_seconds"] / 1e12 if g["busy_seconds"] else None,
                     "gemm_busy_ms_per_step": g["busy_seconds"] / args.steps * 1e3},
        "step_roofline": {"bound": "host_link" if t_strict > t_gemm else "tensor", "t_roof_ms": t_roof * 1e3,
                          "t_gemm_ms": t_gemm * 1e3, "t_swap_strict_ms": t_strict * 1e3,
                          "t_swap_lenient_ms": t_lenient * 1e3, "frac_strict": t_roof / (dev_s / args.steps),
                          "frac_lenient": max(t_gemm, t_lenient) / (dev_s / args.steps),
                          "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
                          "swap_gbs": (h2d + d2h) / (dev_s / args.steps) / 1e9,
                          "host_link_gbs_measured": bw, "flops_per_step": F, "cap_aware": cap_aware,
                          "nvlink_phase0": nvlink},
        "kernels": {k: dict(v, per_launch_us=(v["seconds"] / v["launches"] * 1e6 if v["launches"] else None))
                    for k, v in prof.items()},
        "attention": {"achieved_tflops": (prof["attention"]["work"] / prof["attention"]["seconds"] / 1e12
                                          if prof["attention"]["seconds"] else None),
                      "peak_tflops": gemm_peak, "kernel": "attn_fwd_kernel / attn_bwd_kernel (fused, tcgen05)"},
        "adam_hbm": {"achieved_gbs": adam["work"] / adam["seconds"] / 1e9 if adam["seconds"] else None,
                     "peak_gbs": peaks["hbm_gbs"]},
        "e2e": {"value": samples / e2e_wall, "unit": unit, "h2d_bytes_per_step": e2e_stats[-1]["h2d_input_bytes"],
                "d2h_bytes_per_step": e2e_stats[-1]["d2h_output_bytes"], "timing": "host wall clock around harmony_step",
                "ms_per_step": e2e_wall / args.steps * 1e3,
                "device_ms_per_step": sum(x["step_seconds"] for x in e2e_stats) / len(e2e_stats) * 1e3,
                "pageable_host_inputs": {"value": samples / pageable_wall, "unit": unit,
                                         "ms_per_step": pageable_wall / args.steps * 1e3,
                                         "timing": "host wall clock, numpy (pageable) X, T through harmony_step"}},
        "gpu_launches": int(sum(s["kernel_launches"] for s in stats)),
        "graph_replay": bool(stats[-1]["graph"]),
        "profiled_pass_ms_per_step": prof_s / args.steps * 1e3,
        "clocks": clk,
        "loss": losses[-1],
        "wall_s": wall, "setup_s": setup_s,
        "plan": {k: plan[k] for k in ("arena_bytes", "resident_weight_bytes", "resident_state_bytes",
                                      "resident_stash_bytes", "total_stash_bytes", "pred_h2d_bytes",
                                      "pred_d2h_bytes", "n_ops", "hazards")},
    }
    if world == 1 and not args.no_cpu_baseline:
        v, desc, cores, dt = cpu_oracle_full_step(wl, 1)
        line["cpu_baseline"] = {"value": v, "unit": unit, "cores": cores, "kind": "oracle", "sample": desc,
                                "measured_step_s": dt}
    txt = json.dumps(line)
    print(txt)
    if args.out:
        with open(args.out, "w") as f:
            f.write(txt + "\n")


if __name__ == "__main__":
    main()
