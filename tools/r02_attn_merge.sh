# attention forward: PV(j) and S(j+2) as one UMMA burst (HARMONY_ATTN_MERGE=1) vs separate
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
HARMONY_ATTN_MERGE=1 timeout 600 python -m pytest tests/test_gpu_kernels.py -m gpu -x -q -p no:cacheprovider -k "fused_attention_forward" 2>&1 | tail -1
for v in 1 0 1 0; do for c in 0 1; do HARMONY_ATTN_MERGE=$v timeout 120 python tools/attn_bench.py --reps 20 --causal $c --b 32 2>&1 | grep attn_fwd | sed "s/^/merge$v causal$c /"; done; done
