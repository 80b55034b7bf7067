timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo "tests exit $?"
tail -2 gpurun_out/gpu_tests.log
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench exit $?"
python -c "import json;d=json.load(open('gpurun_out/bench.json'));print('cfg2', d['value'], d['roofline']['frac'], d['step_roofline']['frac_strict'], d['attention'], {k:round(v['seconds']/d['steps']*1e3,2) for k,v in d['kernels'].items()})"
timeout 900 python bench.py --workload cfg3 --no-cpu-baseline > gpurun_out/bench_cfg3.json 2> gpurun_out/bench_cfg3.err; echo "bench cfg3 exit $?"
python -c "import json;d=json.load(open('gpurun_out/bench_cfg3.json'));print('cfg3', d['value'], d['roofline']['frac'], d['step_roofline']['frac_strict'], {k:round(v['seconds']/d['steps']*1e3,2) for k,v in d['kernels'].items()})"
