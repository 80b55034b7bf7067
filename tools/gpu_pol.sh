for pol in 3; do for m in 4 8; do
timeout 600 python bench.py --no-cpu-baseline --stash-policy $pol --microbatches $m > gpurun_out/bench_p${pol}_m$m.json 2>gpurun_out/bench_p${pol}_m$m.err
python -c "import json;d=json.load(open('gpurun_out/bench_p${pol}_m$m.json'));print('pol $pol m $m', round(d['value'],1), d['plan']['pred_h2d_bytes'], d['plan']['pred_d2h_bytes'], {k:round(v['seconds']/d['steps']*1e3,2) for k,v in d['kernels'].items()})" || tail -2 gpurun_out/bench_p${pol}_m$m.err
done; done
