for m in 4 2 1; do
timeout 900 python bench.py --workload cfg3 --no-cpu-baseline --microbatches $m --steps 3 > gpurun_out/bench_cfg3_m$m.json 2>gpurun_out/bench_cfg3_m$m.err
python -c "import json;d=json.load(open('gpurun_out/bench_cfg3_m$m.json'));print('m $m', round(d['value'],2), d['ms_per_step'], d['step_roofline']['frac_strict'], d['plan']['pred_h2d_bytes'], d['plan']['pred_d2h_bytes'], {k:round(v['seconds']/d['steps']*1e3,2) for k,v in d['kernels'].items()})" || tail -2 gpurun_out/bench_cfg3_m$m.err
done
