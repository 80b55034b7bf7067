# quick check after a kernel change: kernel + step tests, GEMM set, cfg2 bench
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_step.py -q -x -p no:cacheprovider 2>&1 | tail -2
timeout 300 python tools/gemm_bench.py --reps 20 > gpurun_out/r02_quick_gemm.jsonl 2>&1
python -c "
import json
d={}
for l in open('gpurun_out/r02_quick_gemm.jsonl'):
  try: j=json.loads(l)
  except Exception: continue
  if 'us' in j: d[j['gemm']]=j['us']
print({k: round(v,1) for k,v in d.items()}, 'total', round(sum(d.values()),1))"
timeout 900 python bench.py --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/r02_quick_bench.json 2>/dev/null
python -c "
import json
d=json.loads(open('gpurun_out/r02_quick_bench.json').read().strip().splitlines()[-1])
print('bench', d['value'], d['ms_per_step'], d['roofline']['frac'], d['clocks']['sm_mhz'])"
