set -x
timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_step.py tests/test_gpu_fullsize.py -x -q -k "not full_stack" 2>&1 | tail -4 > gpurun_out/pytest_gpu.log
cat gpurun_out/pytest_gpu.log
timeout 600 python bench.py > gpurun_out/bench_cfg2.json 2> gpurun_out/bench_cfg2.err
timeout 600 python bench.py --workload cfg5 --steps 3 --warmup 3 > gpurun_out/bench_cfg5.json 2> gpurun_out/bench_cfg5.err
timeout 900 python bench.py --workload cfg3 --no-cpu-baseline > gpurun_out/bench_cfg3.json 2> gpurun_out/bench_cfg3.err
for w in cfg2 cfg5 cfg3; do python -c "import json;d=json.load(open('gpurun_out/bench_$w.json'));print('$w', d['value'], d['unit'], d['roofline']['frac'])" || tail -5 gpurun_out/bench_$w.err; done
