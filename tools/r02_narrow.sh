# half-width tail tiles in the CTA-pair GEMM: kernel tests, GEMM set on/off, cfg2 bench on/off
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
timeout 900 python -m pytest tests/test_gpu_kernels.py -m gpu -x -q -p no:cacheprovider -k "gemm" 2>&1 | tail -2
for nar in 1 0; do
  HARMONY_GEMM_NARROW=$nar timeout 300 python tools/gemm_bench.py --reps 20 > gpurun_out/r02_narrow_gemm_$nar.jsonl 2>&1
  python -c "
import json
d={}
for l in open('gpurun_out/r02_narrow_gemm_$nar.jsonl'):
  try: j=json.loads(l)
  except Exception: continue
  if 'us' in j: d[j['gemm']]=j['us']
print('narrow=$nar', {k: round(v,1) for k,v in d.items()}, 'total', round(sum(d.values()),1))"
done
for nar in 1 0; do
  HARMONY_GEMM_NARROW=$nar timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/ab.json 2>gpurun_out/ab.err
  python -c "
import json
d=json.loads(open('gpurun_out/ab.json').read().strip().splitlines()[-1])
print('bench narrow=$nar', round(d['value'],1), round(d['ms_per_step'],2), d['clocks']['sm_mhz'], round(d['kernels']['gemm']['seconds']/d['steps']*1e3,2))"
done
timeout 900 python -m pytest tests/test_gpu_step.py -m gpu -x -q -p no:cacheprovider 2>&1 | tail -2
