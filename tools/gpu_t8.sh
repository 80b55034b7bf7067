timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo "tests exit $?"
tail -2 gpurun_out/gpu_tests.log
for i in 1 2; do
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/bench_$i.json 2> gpurun_out/bench.err
python -c "import json;d=json.load(open('gpurun_out/bench_$i.json'));print('cfg2', round(d['value'],1), d['e2e']['value'], d['roofline']['frac'], {k:round(v['seconds']/d['steps']*1e3,2) for k,v in d['kernels'].items()})"
done
