# per-layer stash policy mix (last k layers policy 3): bitwise tests, bench k = 0/4/8/12 same box
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
timeout 900 python -m pytest tests/test_gpu_step.py -m gpu -x -q -p no:cacheprovider -k "per_layer_attention or recompute_policies" 2>&1 | tail -1
for k in 0 4 8 0 4; do
  timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --attn-stash-layers $k > gpurun_out/ab.json 2>gpurun_out/ab.err
  python -c "
import json
d=json.loads(open('gpurun_out/ab.json').read().strip().splitlines()[-1])
k=d['kernels']
print('k=$k', round(d['value'],1), round(d['ms_per_step'],2), d['clocks']['sm_mhz'], 'h2d', round(d['step_roofline']['h2d_bytes_per_step']/1e9,2), {c: round(x['seconds']/d['steps']*1e3,2) for c,x in k.items() if x['seconds']})" || tail -5 gpurun_out/ab.err
done
