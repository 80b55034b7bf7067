# attention forward: share of exponentials on the FMA pipe (HARMONY_ATTN_POLY pairs of 32)
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
timeout 600 python -m pytest tests/test_gpu_kernels.py -m gpu -x -q -p no:cacheprovider -k "fused_attention" 2>&1 | tail -2
for k in 0 8 12 16; do
for c in 0 1; do HARMONY_ATTN_POLY=$k timeout 120 python tools/attn_bench.py --reps 20 --causal $c --b 32 2>&1 | grep attn_fwd | sed "s/^/poly$k causal$c /"; done
done
