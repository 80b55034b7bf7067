# the d x d output-projection weight gradient: unsplit vs split-K 2/4/8, pair vs single-CTA tiles
for v in "" "HARMONY_GEMM_2SM=0" "HARMONY_GEMM_2SM=3"; do
  for sh in out_wgrad out_wgrad_split2 out_wgrad_split4 out_wgrad_split8; do
    env $v timeout 120 python tools/gemm_bench.py --graph --reps 20 --only $sh 2>&1 | grep '"us"' | sed "s/^/[$v] /"
  done
done
