# attention backward: UMMAs grouped per accumulator (S^T x4 then dP^T x4; dV x4 then dK x4)
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
timeout 600 python -m pytest tests/test_gpu_kernels.py -m gpu -x -q -p no:cacheprovider -k "fused_attention_backward" 2>&1 | tail -1
for c in 0 1; do
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:attn_bwd_persistent -c 3 --csv python tools/attn_bench.py --reps 3 --b 32 --causal $c 2>/dev/null | grep -E "gpu__time" | awk -F'","' -v c=$c '{print "causal" c, $(NF-2), $NF}'
done
