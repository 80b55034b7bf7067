for m in 4 2 1; do
  timeout 600 python bench.py --no-cpu-baseline --steps 5 --warmup 3 --microbatches $m > gpurun_out/bench_m$m.json 2> gpurun_out/bench_m$m.err
  python -c "import json;d=json.load(open('gpurun_out/bench_m$m.json'));print('cfg2 m=$m', round(d['value'],1), d['ms_per_step'], d['step_roofline']['frac_strict'], d['plan']['pred_h2d_bytes'], {k:round(v['seconds']/5*1e3,2) for k,v in d['kernels'].items()})" || tail -3 gpurun_out/bench_m$m.err
done
for m in 2 1; do
  timeout 900 python bench.py --workload cfg3 --no-cpu-baseline --steps 3 --microbatches $m > gpurun_out/bench_cfg3_m$m.json 2> gpurun_out/bench_cfg3_m$m.err
  python -c "import json;d=json.load(open('gpurun_out/bench_cfg3_m$m.json'));print('cfg3 m=$m', round(d['value'],2), d['ms_per_step'], d['step_roofline']['frac_strict'])" || tail -3 gpurun_out/bench_cfg3_m$m.err
done
