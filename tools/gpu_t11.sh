timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo "tests exit $?"
tail -2 gpurun_out/gpu_tests.log
timeout 900 python bench.py --workload cfg3 --no-cpu-baseline > gpurun_out/bench_cfg3.json 2> gpurun_out/bench_cfg3.err
python -c "import json;d=json.load(open('gpurun_out/bench_cfg3.json'));print('cfg3', round(d['value'],2), d['ms_per_step'], d['step_roofline']['frac_strict'], d['e2e']['value'])"
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/bench.json 2> gpurun_out/bench.err
python -c "import json;d=json.load(open('gpurun_out/bench.json'));print('cfg2', round(d['value'],1), d['ms_per_step'], d['step_roofline']['frac_strict'], d['e2e']['value'], d['plan'])"
