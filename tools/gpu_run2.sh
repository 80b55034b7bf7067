set -x
timeout 900 python -m pytest tests/test_gpu_fullsize.py -x -q -s 2>&1 | tail -30 > gpurun_out/fullsize.log
timeout 300 python tools/gemm_bench.py > gpurun_out/gemm_bench.log 2>&1
timeout 900 python bench.py --workload cfg3 --no-cpu-baseline > gpurun_out/bench_cfg3.json 2> gpurun_out/bench_cfg3.err
tail -30 gpurun_out/fullsize.log; cat gpurun_out/gemm_bench.log; cat gpurun_out/bench_cfg3.json; tail -5 gpurun_out/bench_cfg3.err
