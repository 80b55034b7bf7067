timeout 900 python -m pytest tests/test_gpu_kernels.py -x -q 2>&1 | tail -2
bash tools/gpu_attn.sh 2>&1 | tail -7
GEMM_BENCH_TOKENS=16384 python tools/gemm_bench.py --graph 2>&1 | tail -13
