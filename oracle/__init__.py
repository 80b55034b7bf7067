"""fp64 CPU oracle for the Harmony-DP training step — TEST INFRASTRUCTURE ONLY.

Only `tests/`, `__graft_entry__.smoke()` and `bench.py`'s cpu_baseline /
`--impl reference` legs may import this package.  The product path
(`paper_conf_hotos_lipmk21_b200`, the C-ABI library) never imports, links or
executes anything here, and this package never imports the product.

What it computes: Harmony preserves the
semantics of "a single virtual accelerator device"; decomposition, grouping,
swapping, JIT updates and placement must not change the math.  So the oracle is
one plain training step of the registered layer stack on the WHOLE global batch
on one device in float64: forward, MSE loss, manual backward, Adam
(Kingma & Ba [30]).  No microbatching, swapping, sharding or
operator split.  Readings of what the paper leaves silent are
listed in DESIGN.md ("Readings") and cited per function as c1..c26.

Pins (tests/test_oracle_pins.py, `-m "not gpu"`): the hand-computed 2-layer MLP
step (tests/golden/appendix_a_mlp_step.json), central finite differences,
torch.autograd fp64 on CPU (an independent library routine), brute-force loops
on tiny inputs, closed forms (Adam steps 1-2, linear regression), invariants
(LayerNorm, softmax, Sigma dX = 0), special cases (identity block, uniform
attention), microbatch linearity and the block-matrix identity of the
operator split.  Every function below is pinned by at least one of them.
"""
from .layers import (linear_fwd, linear_bwd, gelu_tanh, gelu_tanh_grad, relu, layernorm_fwd, layernorm_bwd,
                     softmax_fwd, softmax_bwd, attention_fwd, attention_bwd, transformer_block_fwd,
                     transformer_block_bwd, mlp_layer_fwd, mlp_layer_bwd)
from .step import (stack_forward, stack_loss_and_grads, adam_update, AdamState, train_step, mse_loss)
from .split_gemm import gemm_fwd_bwd, split_gemm_fwd_bwd, sampled_gemm_entries
from .swap_model import (weight_swap_baseline_dp, weight_swap_harmony_dp, weight_swap_harmony_pp)

__all__ = [n for n in dir() if not n.startswith("_")]
