# two-tile attention forward: kernel tests, A/B timing vs the one-tile kernel (HARMONY_ATTN_FWD=1)
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_kernels.py -m gpu -x -q -k "attention" > gpurun_out/t_attn.log 2>&1; echo "attn tests $?"; tail -3 gpurun_out/t_attn.log
for c in 0 1; do
  for k in 2 1; do
    HARMONY_ATTN_FWD=$k timeout 120 python tools/attn_bench.py --reps 20 --causal $c --b 32 2>&1 | grep attn_fwd | sed "s/^/fwd$k causal$c b32 /"
  done
done
HARMONY_ATTN_FWD=2 timeout 120 python tools/attn_bench.py --reps 20 --causal 1 --b 4 --S 1024 --h 25 2>&1 | grep attn_fwd | sed "s/^/fwd2 cfg3-shape /"
HARMONY_ATTN_FWD=1 timeout 120 python tools/attn_bench.py --reps 20 --causal 1 --b 4 --S 1024 --h 25 2>&1 | grep attn_fwd | sed "s/^/fwd1 cfg3-shape /"
