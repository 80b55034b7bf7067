for i in 1 2 3; do
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/bench_$i.json 2> gpurun_out/bench.err
python -c "import json;d=json.load(open('gpurun_out/bench_$i.json'));print('cfg2', round(d['value'],1), d['clocks']['sm_mhz'], {k:round(v['seconds']/d['steps']*1e3,2) for k,v in d['kernels'].items()})"
done
