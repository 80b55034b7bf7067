# A/B: epilogue input (residual / pre-activation) by ld.global vs TMA through the staging box
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
HARMONY_GEMM_AUX_LDG=1 timeout 900 python -m pytest tests/test_gpu_kernels.py -q -x -p no:cacheprovider 2>&1 | tail -2
for v in 1 0 1 0; do
HARMONY_GEMM_AUX_LDG=$v timeout 300 python tools/gemm_bench.py --reps 20 > gpurun_out/r02_auxldg$v.jsonl 2>&1
python -c "
import json
d={}
for l in open('gpurun_out/r02_auxldg$v.jsonl'):
  try: j=json.loads(l)
  except Exception: continue
  d[j['gemm']]=j['us']
print('ldg=$v', {k: round(d[k],1) for k in ('out_fwd','fc2_fwd','fc2_dgrad')}, 'total', round(sum(v for k,v in d.items() if k!='ALL' and 'us' ),1))"
done
for v in 1 0; do
HARMONY_GEMM_AUX_LDG=$v timeout 900 python bench.py --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/r02_bench_auxldg$v.json 2>/dev/null
python -c "
import json
d=json.loads(open('gpurun_out/r02_bench_auxldg$v.json').read().strip().splitlines()[-1])
print('bench ldg=$v', d['value'], d['ms_per_step'], d['clocks']['sm_mhz'])"
done
