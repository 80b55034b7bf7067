# attention forward iteration: kernel tests, timing (CUDA events, b=32 cfg2 shape, causal 0/1), trace
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
timeout 600 python -m pytest tests/test_gpu_kernels.py -m gpu -x -q -p no:cacheprovider -k "fused_attention" 2>&1 | tail -2
for k in 0 ${POLYS:-12}; do
for c in 0 1; do HARMONY_ATTN_POLY=$k timeout 120 python tools/attn_bench.py --reps 20 --causal $c --b 32 2>&1 | grep attn_fwd | sed "s/^/poly$k causal$c /"; done
done
HARMONY_NVCC_EXTRA=-DHM_ATTN_TRACE python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build_tr.log 2>&1
for k in 0 ${POLYS:-12}; do
HARMONY_ATTN_POLY=$k python tools/attn_trace.py --show 70 > gpurun_out/r02_attn_trace_p$k.txt 2>&1
for c in 0 1; do HARMONY_ATTN_POLY=$k timeout 120 python tools/attn_bench.py --reps 20 --causal $c --b 32 2>&1 | grep attn_fwd | sed "s/^/traced poly$k causal$c /"; done
done
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1
