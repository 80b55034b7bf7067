# forward pack (NEXT-4): bitwise tests, bench A/B (fwd_pack 1 / 2)
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
timeout 900 python -m pytest tests/test_gpu_step.py -m gpu -x -q -p no:cacheprovider -k "forward_pack" 2>&1 | tail -3
for pk in 2 1 2 1; do
  timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --fwd-pack $pk > gpurun_out/ab.json 2>gpurun_out/ab.err
  python -c "
import json
d=json.loads(open('gpurun_out/ab.json').read().strip().splitlines()[-1])
k=d['kernels']
print('bench fwd_pack=$pk', round(d['value'],1), round(d['ms_per_step'],2), d['clocks']['sm_mhz'], {c: round(x['seconds']/d['steps']*1e3,2) for c,x in k.items() if x['seconds']})" || tail -5 gpurun_out/ab.err
done
