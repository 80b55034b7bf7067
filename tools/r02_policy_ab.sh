# stash policy A/B at the cfg2 default geometry (m=2)
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
for v in "--stash-policy 2" "--stash-policy 3" "--stash-policy 3 --groups 2"; do
  timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline $v > gpurun_out/ab.json 2>gpurun_out/ab.err
  python -c "
import json
d=json.loads(open('gpurun_out/ab.json').read().strip().splitlines()[-1])
sr=d['step_roofline']
print('$v', 'samples/s', round(d['value'],1), 'ms', round(d['ms_per_step'],2), 'clk', d['clocks']['sm_mhz'], 'h2d GB', round(sr['h2d_bytes_per_step']/1e9,2), 'd2h GB', round(sr['d2h_bytes_per_step']/1e9,2), 'attn', round(d['kernels']['attention']['seconds']/d['steps']*1e3 if 'kernels' in d else 0,2))" || tail -3 gpurun_out/ab.err
done
