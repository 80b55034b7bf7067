# attention backward: alternating-sub-tile softmax split (default) vs lock-step (HARMONY_ATTN_BWD_ALT=0)
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
timeout 600 python -m pytest tests/test_gpu_kernels.py -m gpu -x -q -p no:cacheprovider -k "fused_attention" 2>&1 | tail -2
for alt in 1 0; do
  HARMONY_ATTN_BWD_ALT=$alt timeout 300 ncu --metrics gpu__time_duration.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed --clock-control none -k regex:attn_bwd_persistent -c 3 --csv python tools/attn_bench.py --reps 3 --b 32 2>/dev/null | grep -E "gpu__time|tensor" | awk -F'","' -v a=$alt '{print "alt" a, $(NF-2), $NF}'
done
