"""The paper's analytical weight-swap model (oracle; test infrastructure only).

PAPER.md P:706-735 and P:772-775 (§3 "Analytical comparison", Fig. 5(b)/(c)):
R uniform layers, |W| = sum_j |W_Lj|, m microbatches per GPU, N GPUs.
  * DP with per-GPU memory virtualization: each GPU swaps W in and out for the
    forward and the backward of each of the m microbatches, plus in and out once
    for the update: (4m + 2) N |W| per iteration.
  * Harmony-DP: W swapped in once for the forward and once for the backward
    (input-batch grouping) and out once for the update (JIT): 3 N |W|.
  * Harmony-PP: 3 |W| across all m microbatches and all N GPUs.
"""


def weight_swap_baseline_dp(W_bytes: int, m: int, N: int) -> int:
    return (4 * m + 2) * N * W_bytes


def weight_swap_harmony_dp(W_bytes: int, m: int, N: int) -> int:
    return 3 * N * W_bytes


def weight_swap_harmony_pp(W_bytes: int, m: int, N: int) -> int:
    return 3 * W_bytes
