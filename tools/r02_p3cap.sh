# upper bound of skipping the attention recompute: policy 3 with room for its whole stash (16 GiB) vs policy 2
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
for v in "2 8" "3 16" "2 16" "3 8"; do
  set -- $v
  timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --stash-policy $1 --cap-gib $2 > gpurun_out/ab.json 2>gpurun_out/ab.err
  python -c "
import json
d=json.loads(open('gpurun_out/ab.json').read().strip().splitlines()[-1])
k=d['kernels']
print('policy $1 cap $2', round(d['value'],1), round(d['ms_per_step'],2), d['clocks']['sm_mhz'], 'h2d', round(d['step_roofline']['h2d_bytes_per_step']/1e9,2), {c: round(x['seconds']/d['steps']*1e3,2) for c,x in k.items() if x['seconds']})" || tail -5 gpurun_out/ab.err
done
