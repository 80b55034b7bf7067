"""Thin ctypes binding of libharmony.so (include/harmony.h, include/harmony_kernels.h).

Argument marshalling only: every step of the training path runs in the library's CUDA
kernels.  There is no fallback: if the library cannot be loaded, importing the binding's
functions raises.  Names follow the C ABI (harmony_init, harmony_register_layers,
harmony_step, harmony_read_state, harmony_finalize, hk_*).
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
# HARMONY_LIB: an alternative in-tree build of the same library (A/B experiments)
LIB_PATH = os.environ.get("HARMONY_LIB") or os.path.join(_PKG, "libharmony.so")

HARMONY_OK, HARMONY_E_INVALID_ARG, HARMONY_E_BAD_STATE, HARMONY_E_CAP_TOO_SMALL = 0, 1, 2, 3
HARMONY_E_HOST_OOM, HARMONY_E_CUDA, HARMONY_E_NCCL, HARMONY_E_UNSUPPORTED = 4, 5, 6, 7
HARMONY_FP32, HARMONY_BF16_FP32MASTER = 0, 1
HARMONY_LAYER_MLP, HARMONY_LAYER_TRANSFORMER = 0, 1
HARMONY_ACT_NONE, HARMONY_ACT_RELU, HARMONY_ACT_GELU_TANH = 0, 1, 2
HARMONY_PARAM, HARMONY_GRAD, HARMONY_ADAM_M, HARMONY_ADAM_V = 0, 1, 2, 3
HARMONY_SCHED_HARMONY_DP, HARMONY_SCHED_PER_GPU_VIRT, HARMONY_SCHED_HARMONY_PP = 0, 1, 2
HK_EPI_STORE_T, HK_EPI_STORE_F32, HK_EPI_RESID_F32, HK_EPI_ACC_F32 = 0, 1, 2, 3
HK_EPI_BIAS_ACT, HK_EPI_ACT_BWD, HK_EPI_BIAS_ACT_F32, HK_EPI_ACT_T = 4, 5, 6, 7


class harmony_config(C.Structure):
    _fields_ = [("struct_size", C.c_uint32), ("rank", C.c_int32), ("world_size", C.c_int32), ("device", C.c_int32),
                ("hbm_cap_bytes", C.c_uint64), ("arena", C.c_void_p), ("microbatches", C.c_int32),
                ("microbatch_size", C.c_int32), ("precision", C.c_int32), ("schedule", C.c_int32),
                ("retain_grads", C.c_int32), ("stash_policy", C.c_int32), ("lr", C.c_double), ("beta1", C.c_double),
                ("beta2", C.c_double), ("eps", C.c_double), ("weight_decay", C.c_double), ("nccl_id", C.c_uint8 * 128),
                ("groups", C.c_int32), ("fwd_pack", C.c_int32)]


class harmony_layer_desc(C.Structure):
    _fields_ = [("kind", C.c_int32), ("d_in", C.c_int32), ("d_out", C.c_int32), ("n_heads", C.c_int32),
                ("seq_len", C.c_int32), ("causal", C.c_int32), ("act", C.c_int32)]


class harmony_step_stats(C.Structure):
    _fields_ = [(n, C.c_uint64) for n in (
        "h2d_bytes", "d2h_bytes", "h2d_weight_bytes", "d2h_weight_bytes", "h2d_state_bytes", "d2h_state_bytes",
        "h2d_stash_bytes", "d2h_stash_bytes", "h2d_input_bytes", "d2h_output_bytes", "h2d_grad_bytes",
        "d2h_grad_bytes", "nvlink_bytes", "peak_arena_bytes", "kernel_launches", "n_ops")] + [
        ("step_seconds", C.c_double), ("graph", C.c_uint64)]

    def as_dict(self):
        return {n: getattr(self, n) for n, _ in self._fields_}


class harmony_plan_summary(C.Structure):
    _fields_ = [(n, C.c_uint64) for n in (
        "arena_bytes", "min_working_set_bytes", "resident_weight_bytes", "total_weight_bytes",
        "resident_state_bytes", "total_state_bytes", "resident_stash_bytes", "total_stash_bytes",
        "pred_h2d_bytes", "pred_d2h_bytes", "pred_h2d_weight_bytes", "pred_d2h_weight_bytes", "flops_per_step")] + [
        ("n_params", C.c_int64)] + [(n, C.c_int32) for n in (
        "n_ops", "n_compute_ops", "n_copy_ops", "n_comm_ops", "weight_slots", "stash_slots", "state_slots",
        "hazards")]

    def as_dict(self):
        return {n: getattr(self, n) for n, _ in self._fields_}


class harmony_kernel_profile(C.Structure):
    _fields_ = [("launches", C.c_uint64 * 6), ("seconds", C.c_double * 6), ("work", C.c_double * 6),
                ("busy_seconds", C.c_double * 6)]
    CLASSES = ("gemm", "adam", "layernorm", "softmax", "other", "attention")

    def as_dict(self):
        return {c: dict(launches=self.launches[i], seconds=self.seconds[i], work=self.work[i],
                        busy_seconds=self.busy_seconds[i])
                for i, c in enumerate(self.CLASSES)}


class harmony_timeline_rec(C.Structure):
    _fields_ = [(n, C.c_int32) for n in ("op", "kind", "stream", "cat", "layer", "micro")] + [
        ("bytes", C.c_uint64), ("t0", C.c_double), ("t1", C.c_double)]

    def as_dict(self):
        return {n: getattr(self, n) for n, _ in self._fields_}


class harmony_kernel_rec(C.Structure):
    _fields_ = [("cat", C.c_int32), ("stream", C.c_int32), ("work", C.c_double), ("t0", C.c_double), ("t1", C.c_double)]

    def as_dict(self):
        return {n: getattr(self, n) for n, _ in self._fields_}


class hk_gemm_args(C.Structure):
    _fields_ = [("dtype", C.c_int32), ("M", C.c_int32), ("N", C.c_int32), ("K", C.c_int32), ("nz0", C.c_int32),
                ("nz1", C.c_int32),
                ("A", C.c_void_p), ("a_mn_major", C.c_int32), ("lda", C.c_int64), ("a_sz0", C.c_int64),
                ("a_sz1", C.c_int64),
                ("B", C.c_void_p), ("b_mn_major", C.c_int32), ("ldb", C.c_int64), ("b_sz0", C.c_int64),
                ("b_sz1", C.c_int64),
                ("C", C.c_void_p), ("ldc", C.c_int64), ("c_sz0", C.c_int64), ("c_sz1", C.c_int64),
                ("epilogue", C.c_int32), ("act", C.c_int32), ("accumulate", C.c_int32), ("alpha", C.c_float),
                ("bias", C.c_void_p), ("aux", C.c_void_p), ("aux_out", C.c_void_p)]


_lib = None


def _nccl_path():
    try:
        import nvidia.nccl  # type: ignore
        p = os.path.join(list(nvidia.nccl.__path__)[0], "lib", "libnccl.so.2")
        return p if os.path.exists(p) else None
    except Exception:
        return None


def lib() -> C.CDLL:
    """Load libharmony.so (raises if it was not built: there is no fallback path)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise RuntimeError(f"{LIB_PATH} missing: build it with `python -m paper_conf_hotos_lipmk21_b200.build`")
    if "HARMONY_NCCL_PATH" not in os.environ:
        p = _nccl_path()
        if p:
            os.environ["HARMONY_NCCL_PATH"] = p
    L = C.CDLL(LIB_PATH)
    st = C.c_int
    P = C.c_void_p
    sig = {
        "harmony_abi_version": (C.c_int32, []),
        "harmony_last_error": (C.c_char_p, [P]),
        "harmony_get_unique_id": (st, [P]),
        "harmony_init": (st, [C.POINTER(harmony_config), C.POINTER(P)]),
        "harmony_init_group": (st, [C.POINTER(harmony_config), C.c_int32, P, C.POINTER(P)]),
        "harmony_read_rank_stats": (st, [P, C.c_int32, C.POINTER(harmony_step_stats)]),
        "harmony_plan_dry_group": (st, [C.POINTER(harmony_config), C.c_int32, C.c_int32, C.POINTER(harmony_layer_desc),
                                        C.POINTER(harmony_plan_summary), P, C.c_uint64]),
        "harmony_register_layers": (st, [P, C.c_int32, C.POINTER(harmony_layer_desc), C.POINTER(P)]),
        "harmony_step": (st, [P, P, P, C.c_int64, C.POINTER(C.c_double), C.POINTER(harmony_step_stats)]),
        "harmony_read_state": (st, [P, C.c_int32, C.c_int32, P, C.c_uint64]),
        "harmony_read_stats": (st, [P, C.POINTER(harmony_step_stats)]),
        "harmony_plan_info": (st, [P, C.POINTER(harmony_plan_summary)]),
        "harmony_plan_dry": (st, [C.POINTER(harmony_config), C.c_int32, C.POINTER(harmony_layer_desc),
                                  C.POINTER(harmony_plan_summary), P, C.c_uint64]),
        "harmony_finalize": (st, [P]),
        "harmony_read_timeline": (st, [P, P, C.c_int32, C.POINTER(C.c_int32)]),
        "harmony_read_kernel_timeline": (st, [P, P, C.c_int32, C.POINTER(C.c_int32)]),
        "hk_gemm": (st, [C.POINTER(hk_gemm_args), P]),
        "hk_layernorm_fwd": (st, [C.c_int32, C.c_int64, C.c_int32, P, P, P, P, P, P, P]),
        "hk_layernorm_bwd": (st, [C.c_int32, C.c_int64, C.c_int32, P, P, P, P, P, P, P, P, P, C.c_int32, P]),
        "hk_softmax_fwd": (st, [C.c_int32, C.c_int64, C.c_int32, C.c_int32, C.c_float, P, P, P]),
        "hk_softmax_bwd": (st, [C.c_int32, C.c_int64, C.c_int32, C.c_float, P, P, P, P]),
        "hk_colsum": (st, [C.c_int32, C.c_int64, C.c_int32, P, C.c_int64, P, C.c_int32, P]),
        "hk_adam": (st, [C.c_int32, C.c_int64, P, P, P, P, P, C.c_double, C.c_double, C.c_double, C.c_double,
                         C.c_int32, P]),
        "hk_mse": (st, [C.c_int64, P, P, C.c_float, P, P, P]),
        "hk_cast": (st, [C.c_int32, C.c_int64, P, P, P]),
        "hk_act_bwd": (st, [C.c_int32, C.c_int32, C.c_int64, P, P, P, P]),
        "hk_sync": (st, []),
        "hk_attention_fwd": (st, [C.c_int64, C.c_int32, C.c_int32, C.c_int32, C.c_int32, P, P, P, P]),
        "hk_attention_bwd": (st, [C.c_int64, C.c_int32, C.c_int32, C.c_int32, C.c_int32, P, P, P, P, P, P]),
        "harmony_abi_sizes": (None, [P]),
        "harmony_split_gemm_init": (st, [C.POINTER(harmony_config), C.c_int64, C.c_int64, C.c_int64, C.c_int32,
                                         C.POINTER(P)]),
        "harmony_split_gemm_run": (st, [P, P, P, P, P, P, P, C.POINTER(C.c_double)]),
        "harmony_split_gemm_finalize": (st, [P]),
        "harmony_split_gemm_init_group": (st, [C.c_int32, P, C.c_int64, C.c_int64, C.c_int64, C.c_int32,
                                               C.POINTER(P)]),
        "harmony_split_gemm_run_group": (st, [P, P, P, P, P, P, P, C.POINTER(C.c_double)]),
        "harmony_set_profiling": (st, [P, C.c_int32]),
        "harmony_read_profile": (st, [P, C.POINTER(harmony_kernel_profile)]),
    }
    for name, (res, args) in sig.items():
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    _lib = L
    return L


class HarmonyError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"harmony status {code}: {msg}")
        self.code = code


def _check(code, ctx=None):
    if code != HARMONY_OK:
        msg = lib().harmony_last_error(ctx)
        raise HarmonyError(code, msg.decode() if msg else "")


# ------------------------------------------------------------------------------- C-ABI wrappers
def make_config(*, rank=0, world_size=1, device=0, hbm_cap_bytes=0, arena=None, microbatches=1, microbatch_size=1,
                precision=HARMONY_FP32, schedule=HARMONY_SCHED_HARMONY_DP, retain_grads=0, stash_policy=0, lr=1e-3,
                beta1=0.9, beta2=0.999, eps=1e-8, weight_decay=0.0, nccl_id=None, groups=1,
                fwd_pack=1) -> harmony_config:
    c = harmony_config()
    c.struct_size = C.sizeof(harmony_config)
    c.rank, c.world_size, c.device = rank, world_size, device
    c.hbm_cap_bytes = int(hbm_cap_bytes)
    c.arena = arena
    c.microbatches, c.microbatch_size = microbatches, microbatch_size
    c.precision, c.schedule, c.retain_grads, c.stash_policy = precision, schedule, retain_grads, stash_policy
    c.lr, c.beta1, c.beta2, c.eps, c.weight_decay = lr, beta1, beta2, eps, weight_decay
    if nccl_id is not None:
        C.memmove(c.nccl_id, bytes(nccl_id), 128)
    c.groups = groups
    c.fwd_pack = fwd_pack
    return c


def make_descs(descs) -> C.Array:
    """descs: objects with kind, d_in, d_out, n_heads, seq_len, causal, act (e.g. synth.LayerDesc)."""
    arr = (harmony_layer_desc * len(descs))()
    for i, d in enumerate(descs):
        arr[i] = harmony_layer_desc(d.kind, d.d_in, d.d_out, d.n_heads, d.seq_len, d.causal, d.act)
    return arr


def harmony_get_unique_id() -> bytes:
    buf = (C.c_uint8 * 128)()
    _check(lib().harmony_get_unique_id(buf))
    return bytes(buf)


def harmony_init(cfg: harmony_config) -> C.c_void_p:
    ctx = C.c_void_p()
    _check(lib().harmony_init(C.byref(cfg), C.byref(ctx)))
    return ctx


def harmony_init_group(cfg: harmony_config, devices) -> C.c_void_p:
    """One context driving len(devices) data-parallel ranks (rank r on devices[r]; repeats = ranks
    sharing a GPU, the loopback)."""
    ctx = C.c_void_p()
    arr = (C.c_int32 * len(devices))(*devices)
    _check(lib().harmony_init_group(C.byref(cfg), len(devices), arr, C.byref(ctx)))
    return ctx


def harmony_read_rank_stats(ctx, rank):
    s = harmony_step_stats()
    _check(lib().harmony_read_rank_stats(ctx, int(rank), C.byref(s)), ctx)
    return s


def harmony_register_layers(ctx, descs, init_params):
    arr = make_descs(descs)
    keep = [np.ascontiguousarray(p, dtype=np.float32) for p in init_params]
    ptrs = (C.c_void_p * len(keep))(*[k.ctypes.data for k in keep])
    _check(lib().harmony_register_layers(ctx, len(keep), arr, ptrs), ctx)


def _ptr(a):
    """Host numpy array or torch tensor (host or CUDA) -> address."""
    if isinstance(a, np.ndarray):
        assert a.dtype == np.float32 and a.flags.c_contiguous
        return a.ctypes.data
    if hasattr(a, "data_ptr"):
        assert a.is_contiguous()
        return a.data_ptr()
    return int(a)


def harmony_step(ctx, x, target, batch):
    loss = C.c_double()
    stats = harmony_step_stats()
    _check(lib().harmony_step(ctx, _ptr(x), _ptr(target), int(batch), C.byref(loss), C.byref(stats)), ctx)
    return loss.value, stats


def harmony_read_state(ctx, layer, which, n):
    out = np.empty(n, dtype=np.float32)
    _check(lib().harmony_read_state(ctx, layer, which, out.ctypes.data, n), ctx)
    return out


def harmony_read_stats(ctx):
    s = harmony_step_stats()
    _check(lib().harmony_read_stats(ctx, C.byref(s)), ctx)
    return s


def harmony_plan_info(ctx):
    s = harmony_plan_summary()
    _check(lib().harmony_plan_info(ctx, C.byref(s)), ctx)
    return s


def harmony_plan_dry(cfg, descs, text_len=1 << 22):
    s = harmony_plan_summary()
    buf = C.create_string_buffer(text_len) if text_len else None
    _check(lib().harmony_plan_dry(C.byref(cfg), len(descs), make_descs(descs), C.byref(s), buf, text_len))
    return s, (buf.value.decode() if buf is not None else "")


def harmony_plan_dry_group(cfg, num_ranks, descs, text_len=1 << 22):
    s = harmony_plan_summary()
    buf = C.create_string_buffer(text_len) if text_len else None
    _check(lib().harmony_plan_dry_group(C.byref(cfg), int(num_ranks), len(descs), make_descs(descs), C.byref(s), buf,
                                        text_len))
    return s, (buf.value.decode() if buf is not None else "")


def harmony_set_profiling(ctx, on):
    _check(lib().harmony_set_profiling(ctx, int(on)), ctx)


def harmony_read_profile(ctx):
    p = harmony_kernel_profile()
    _check(lib().harmony_read_profile(ctx, C.byref(p)), ctx)
    return p


def harmony_read_timeline(ctx):
    """Per-op timeline of the last profiled step (list of dicts; see harmony.h)."""
    n = C.c_int32()
    _check(lib().harmony_read_timeline(ctx, None, 0, C.byref(n)), ctx)
    arr = (harmony_timeline_rec * max(n.value, 1))()
    _check(lib().harmony_read_timeline(ctx, arr, n.value, C.byref(n)), ctx)
    return [arr[i].as_dict() for i in range(n.value)]


def harmony_read_kernel_timeline(ctx):
    """Kernel launches of the last profiled step (list of dicts; see harmony.h)."""
    n = C.c_int32()
    _check(lib().harmony_read_kernel_timeline(ctx, None, 0, C.byref(n)), ctx)
    arr = (harmony_kernel_rec * max(n.value, 1))()
    _check(lib().harmony_read_kernel_timeline(ctx, arr, n.value, C.byref(n)), ctx)
    return [arr[i].as_dict() for i in range(n.value)]


def harmony_finalize(ctx):
    _check(lib().harmony_finalize(ctx))


class SplitGemm:
    """Operator-split GEMM fwd+bwd (harmony_split_gemm_*): this rank's K-slice of X, W."""

    def __init__(self, M, N, K, chunks=4, **cfg):
        self.cfg = make_config(**cfg)
        self.h = C.c_void_p()
        _check(lib().harmony_split_gemm_init(C.byref(self.cfg), M, N, K, chunks, C.byref(self.h)))

    def run(self, X_slice, W_slice, dY_shard, Y_shard, dX_slice, dW_slice):
        sec = C.c_double()
        _check(lib().harmony_split_gemm_run(self.h, _ptr(X_slice), _ptr(W_slice), _ptr(dY_shard), _ptr(Y_shard),
                                            _ptr(dX_slice), _ptr(dW_slice), C.byref(sec)))
        return sec.value

    def close(self):
        if self.h:
            _check(lib().harmony_split_gemm_finalize(self.h))
            self.h = None

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()


class SplitGemmGroup:
    """Operator-split GEMM fwd+bwd with every rank in this process (harmony_split_gemm_init_group):
    rank r on devices[r]; run() takes per-rank lists of tensors."""

    def __init__(self, M, N, K, devices, chunks=4):
        self.n = len(devices)
        self.h = C.c_void_p()
        arr = (C.c_int32 * self.n)(*devices)
        _check(lib().harmony_split_gemm_init_group(self.n, arr, M, N, K, chunks, C.byref(self.h)))

    def run(self, X, W, dY, Y, dX, dW):
        def arr(ts):
            assert len(ts) == self.n
            return (C.c_void_p * self.n)(*[_ptr(t) for t in ts])
        sec = C.c_double()
        _check(lib().harmony_split_gemm_run_group(self.h, arr(X), arr(W), arr(dY), arr(Y), arr(dX), arr(dW),
                                                  C.byref(sec)))
        return sec.value

    def close(self):
        if self.h:
            _check(lib().harmony_split_gemm_finalize(self.h))
            self.h = None

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()


# ------------------------------------------------------------------------------- kernel ABI
def hk(name, *args):
    """Call a kernel-level entry point, raising on error."""
    _check(getattr(lib(), name)(*args))


class Harmony:
    """Convenience owner of one context: one process = one GPU rank, or (group=[dev, ...]) one
    process driving len(group) ranks as one virtual device (harmony_init_group)."""

    def __init__(self, descs, init_params, group=None, **cfg):
        self.cfg = make_config(**cfg)
        self.ranks = len(group) if group else 1
        self.ctx = harmony_init_group(self.cfg, list(group)) if group else harmony_init(self.cfg)
        self.descs = list(descs)
        try:
            harmony_register_layers(self.ctx, self.descs, init_params)
        except Exception:
            harmony_finalize(self.ctx)
            self.ctx = None
            raise
        self.n_params = [int(np.asarray(p).size) for p in init_params]

    def step(self, x, target):
        """x, target: this rank's rows (a data-parallel group: the global batch of ranks*m*b rows; Harmony-PP:
        the one minibatch of m*b rows that flows through the ranks)."""
        mult = 1 if self.cfg.schedule == HARMONY_SCHED_HARMONY_PP else self.ranks
        return harmony_step(self.ctx, x, target, mult * self.cfg.microbatches * self.cfg.microbatch_size)

    def rank_stats(self, rank):
        return harmony_read_rank_stats(self.ctx, rank)

    def read(self, layer, which=HARMONY_PARAM):
        return harmony_read_state(self.ctx, layer, which, self.n_params[layer])

    def plan(self):
        return harmony_plan_info(self.ctx)

    def close(self):
        if self.ctx is not None:
            harmony_finalize(self.ctx)
            self.ctx = None

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
