"""Seeded synthetic inputs shared by the oracle side and the CUDA side.

This module holds NO arithmetic of the method: it only draws random numbers
(NumPy PCG64) in the shapes and distributions of the paper's workloads and lays
them out in the canonical parameter packing of include/harmony.h.  Both
`oracle/` and the CUDA path consume its output as plain data; neither is
imported here.

Recipe:
  * params: seed 0 (layer l uses SeedSequence([0, l])).
      transformer: W ~ N(0, 0.02^2); W_o, W_fc2 ~ N(0, (0.02/sqrt(2L))^2);
                   biases ~ N(0, 0.02^2); gamma ~ 1 + N(0, 0.1^2); beta ~ N(0, 0.02^2)
      mlp:         W ~ N(0, 1/d_in); b ~ N(0, 0.1^2)
  * batch for step t: seed 1000 + t; X, T ~ N(0, 1).
  * on the bf16 path (precision=1) every generated value is made bf16-exact by
    round-to-nearest-even on the fp32 bit pattern, so both sides start from
    identical numbers.
"""
from __future__ import annotations

import numpy as np

LAYER_MLP = 0
LAYER_TRANSFORMER = 1
ACT_NONE, ACT_RELU, ACT_GELU = 0, 1, 2
FP32, BF16 = 0, 1


def bf16_exact(a: np.ndarray) -> np.ndarray:
    """Round fp32 values to the nearest bf16-representable fp32 (ties to even).

    (u + 0x7FFF + ((u >> 16) & 1)) & 0xFFFF0000 on the fp32 bit pattern u.
    Used only to make generated inputs exactly representable."""
    a = np.ascontiguousarray(a, dtype=np.float32)
    u = a.view(np.uint32).astype(np.uint64)
    r = ((u + 0x7FFF + ((u >> 16) & 1)) & 0xFFFF0000).astype(np.uint32)
    return r.view(np.float32).reshape(a.shape)


class LayerDesc:
    """Mirror of harmony_layer_desc (include/harmony.h)."""

    __slots__ = ("kind", "d_in", "d_out", "n_heads", "seq_len", "causal", "act")

    def __init__(self, kind, d_in, d_out, n_heads=0, seq_len=1, causal=0, act=ACT_NONE):
        self.kind, self.d_in, self.d_out = int(kind), int(d_in), int(d_out)
        self.n_heads, self.seq_len, self.causal, self.act = int(n_heads), int(seq_len), int(causal), int(act)

    def n_params(self) -> int:
        if self.kind == LAYER_MLP:
            return self.d_in * self.d_out + self.d_out
        d = self.d_in
        return 12 * d * d + 13 * d

    def __repr__(self):
        return (f"LayerDesc(kind={self.kind}, d_in={self.d_in}, d_out={self.d_out}, h={self.n_heads}, "
                f"S={self.seq_len}, causal={self.causal}, act={self.act})")


def mlp_stack(n_layers: int, d: int, act=ACT_GELU, last_act=ACT_NONE):
    """cfg1-style MLP: Linear+act for layers 1..L-1, plain Linear last."""
    return [LayerDesc(LAYER_MLP, d, d, act=(act if i < n_layers - 1 else last_act)) for i in range(n_layers)]


def transformer_stack(n_layers: int, d: int, h: int, S: int, causal: bool):
    return [LayerDesc(LAYER_TRANSFORMER, d, d, n_heads=h, seq_len=S, causal=int(causal)) for _ in range(n_layers)]


def transformer_segments(d: int):
    """(name, shape) in canonical packing order: 12d^2 + 13d floats."""
    return [("ln1_g", (d,)), ("ln1_b", (d,)), ("w_qkv", (d, 3 * d)), ("b_qkv", (3 * d,)),
            ("w_o", (d, d)), ("b_o", (d,)), ("ln2_g", (d,)), ("ln2_b", (d,)),
            ("w_fc1", (d, 4 * d)), ("b_fc1", (4 * d,)), ("w_fc2", (4 * d, d)), ("b_fc2", (d,))]


def mlp_segments(d_in: int, d_out: int):
    return [("w", (d_in, d_out)), ("b", (d_out,))]


def segments(desc: LayerDesc):
    if desc.kind == LAYER_MLP:
        return mlp_segments(desc.d_in, desc.d_out)
    return transformer_segments(desc.d_in)


def unpack(desc: LayerDesc, flat: np.ndarray) -> dict:
    """Views of a canonical flat parameter vector, by segment name."""
    out, off = {}, 0
    for name, shape in segments(desc):
        n = int(np.prod(shape))
        out[name] = flat[off:off + n].reshape(shape)
        off += n
    assert off == flat.size, (off, flat.size)
    return out


def pack(desc: LayerDesc, parts: dict, dtype=np.float64) -> np.ndarray:
    return np.concatenate([np.asarray(parts[name], dtype=dtype).reshape(-1) for name, _ in segments(desc)])


def gen_layer_params(desc: LayerDesc, layer: int, n_layers: int, precision: int = FP32, seed: int = 0,
                     dtype=np.float32) -> np.ndarray:
    """Initial parameters of one layer in canonical packing (fp32 values)."""
    rng = np.random.Generator(np.random.PCG64(np.random.SeedSequence([seed, layer])))
    parts = {}
    if desc.kind == LAYER_MLP:
        parts["w"] = rng.standard_normal((desc.d_in, desc.d_out), dtype=np.float32) * np.float32(1.0 / np.sqrt(desc.d_in))
        parts["b"] = rng.standard_normal(desc.d_out, dtype=np.float32) * np.float32(0.1)
    else:
        d = desc.d_in
        s_out = np.float32(0.02 / np.sqrt(2.0 * n_layers))
        for name, shape in transformer_segments(d):
            z = rng.standard_normal(shape, dtype=np.float32)
            if name in ("ln1_g", "ln2_g"):
                parts[name] = np.float32(1.0) + z * np.float32(0.1)
            elif name in ("w_o", "w_fc2"):
                parts[name] = z * s_out
            else:
                parts[name] = z * np.float32(0.02)
    flat = np.concatenate([parts[name].reshape(-1) for name, _ in segments(desc)]).astype(np.float32)
    if precision == BF16:
        flat = bf16_exact(flat)
    return flat.astype(dtype, copy=False)


def gen_params(descs, precision: int = FP32, seed: int = 0):
    return [gen_layer_params(d, i, len(descs), precision, seed) for i, d in enumerate(descs)]


def sample_shape(descs):
    d0 = descs[0]
    if d0.kind == LAYER_MLP:
        return (d0.d_in,), (descs[-1].d_out,)
    return (d0.seq_len, d0.d_in), (d0.seq_len, descs[-1].d_out)


def gen_batch(descs, batch: int, step: int, precision: int = FP32, seed_base: int = 1000):
    """(X, T) for step `step` (1-based), fp32, shapes [B, *sample_shape]."""
    rng = np.random.Generator(np.random.PCG64(seed_base + step))
    xs, ts = sample_shape(descs)
    X = rng.standard_normal((batch,) + xs, dtype=np.float32)
    T = rng.standard_normal((batch,) + ts, dtype=np.float32)
    if precision == BF16:
        X, T = bf16_exact(X), bf16_exact(T)
    return X, T


def gen_gemm_operands(M: int, N: int, K: int, seed: int = 7):
    """cfg5 operands (bf16-exact fp32): X [M,K], W [K,N], dY [M,N]."""
    rng = np.random.Generator(np.random.PCG64(seed))
    X = bf16_exact(rng.standard_normal((M, K), dtype=np.float32))
    W = bf16_exact(rng.standard_normal((K, N), dtype=np.float32) * np.float32(1.0 / np.sqrt(K)))
    dY = bf16_exact(rng.standard_normal((M, N), dtype=np.float32))
    return X, W, dY


# The configurations of BASELINE.json.  Only shapes and knobs.
CONFIGS = {
    "cfg1": dict(name="mlp4_d256_b32_m4_fp32", descs=lambda: mlp_stack(4, 256), batch=32, m=4, precision=FP32,
                 cap=2 * 16 * (256 * 256 + 256)),
    "cfg2": dict(name="bert_large_L24_d1024_S512_b64_cap8GB", descs=lambda: transformer_stack(24, 1024, 16, 512, False),
                 batch=64, m=8, precision=BF16, cap=8 << 30),
    "cfg3": dict(name="gpt2xl_L48_d1600_S1024_bg8_cap16GB", descs=lambda: transformer_stack(48, 1600, 25, 1024, True),
                 batch=8, m=4, precision=BF16, cap=16 << 30),
}
