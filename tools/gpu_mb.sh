for m in 8 4 2 1; do
  timeout 600 python bench.py --no-cpu-baseline --steps 5 --warmup 3 --microbatches $m > gpurun_out/bench_m$m.json 2> gpurun_out/bench_m$m.err
  python -c "import json;d=json.load(open('gpurun_out/bench_m$m.json'));print('m=$m', round(d['value'],1), d['ms_per_step'], d['plan'], {k:round(v['seconds']/5*1e3,2) for k,v in d['kernels'].items()})" || tail -3 gpurun_out/bench_m$m.err
done
