# attention forward kernel tests, default and HARMONY_ATTN_FWD=1
timeout 200 python -m pytest tests/test_gpu_kernels.py -m gpu -x -q -k "fused_attention_forward" 2>&1 | grep -E "^E  |FAILED|passed" | head -6
HARMONY_ATTN_FWD=1 timeout 200 python -m pytest tests/test_gpu_kernels.py -m gpu -x -q -k "fused_attention_forward" 2>&1 | tail -1
