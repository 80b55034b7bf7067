# GEMM A/B: normal epilogue vs TMEM-drain-only (mainloop-bound), cuBLAS on the same shapes
set -x
timeout 300 python tools/gemm_bench.py --cublas --graph > gpurun_out/gb_normal.log 2>&1
HARMONY_GEMM_TMA_EPI=2 timeout 300 python tools/gemm_bench.py --graph > gpurun_out/gb_drain.log 2>&1
HARMONY_GEMM_2SM=3 timeout 300 python tools/gemm_bench.py --graph > gpurun_out/gb_bn128.log 2>&1
timeout 300 python tools/gemm_bench.py --graph --sweep > gpurun_out/gb_sweep.log 2>&1
timeout 900 python -m pytest tests/test_gpu_fullsize.py -x -q -s -k full_stack 2>&1 | tail -5 > gpurun_out/fullstack.log
for f in gb_normal gb_drain gb_bn128 gb_sweep fullstack; do echo "== $f"; cat gpurun_out/$f.log; done
