# QKV weight gradient forked before the QKV dgrad (no idle join): step tests, bench x2, kernel timeline
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
timeout 900 python -m pytest tests/test_gpu_step.py -m gpu -x -q -p no:cacheprovider 2>&1 | tail -1
for i in 1 2; do
  timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/ab.json 2>gpurun_out/ab.err
  python -c "
import json
d=json.loads(open('gpurun_out/ab.json').read().strip().splitlines()[-1])
k=d['kernels']
print('bench', round(d['value'],1), round(d['ms_per_step'],2), d['clocks']['sm_mhz'], {c: round(x['seconds']/d['steps']*1e3,2) for c,x in k.items() if x['seconds']})" || tail -5 gpurun_out/ab.err
done
cd tools && timeout 600 python ktimeline.py --out ../gpurun_out/ktl_join.json > ../gpurun_out/ktl_join.txt 2>&1; echo "ktl $?"
