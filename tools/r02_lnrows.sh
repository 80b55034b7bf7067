# LayerNorm backward rows per block (HARMONY_LN_ROWS 16 = default, 32, 64): fewer column partials to reduce
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
HARMONY_LN_ROWS=64 timeout 600 python -m pytest tests/test_gpu_kernels.py -m gpu -x -q -p no:cacheprovider -k "layernorm" 2>&1 | tail -1
for v in 16 64 32 16 64 32; do
  HARMONY_LN_ROWS=$v timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/ab.json 2>gpurun_out/ab.err
  python -c "
import json
d=json.loads(open('gpurun_out/ab.json').read().strip().splitlines()[-1])
k=d['kernels']
print('rows=$v', round(d['value'],1), round(d['ms_per_step'],2), d['clocks']['sm_mhz'], {c: round(x['seconds']/d['steps']*1e3,2) for c,x in k.items() if x['seconds']})"
done
