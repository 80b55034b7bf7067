set -x
timeout 900 python -m pytest tests/test_gpu_step.py tests/test_gpu_kernels.py -x -q 2>&1 | tail -4 > gpurun_out/pytest_gpu.log
cat gpurun_out/pytest_gpu.log
for pol in 2 3 2 3; do
  timeout 600 python bench.py --no-cpu-baseline --stash-policy $pol > gpurun_out/bench_p$pol.json 2> gpurun_out/bench_p$pol.err
  python -c "import json;d=json.load(open('gpurun_out/bench_p$pol.json'));print('policy $pol', round(d['value'],1), d['step_roofline']['h2d_bytes_per_step'], d['step_roofline']['d2h_bytes_per_step'], {k: round(v['per_launch_us'] or 0,2) for k,v in d['kernels'].items()})"
done
