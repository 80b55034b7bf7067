timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo "tests exit $?"
tail -3 gpurun_out/gpu_tests.log
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench exit $?"
python -c "import json;d=json.load(open('gpurun_out/bench.json'));print(d['value'], d['roofline']['frac'], d['step_roofline']['frac_strict'], d['e2e']['value'], {k:round(v['seconds']/d['steps']*1e3,2) for k,v in d['kernels'].items()})"
