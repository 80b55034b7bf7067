# programmatic dependent launch: full gpu suite, smoke, bench A/B (HARMONY_PDL=0/1)
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
for v in 1 0; do
  HARMONY_PDL=$v timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/ab.json 2>gpurun_out/ab.err
  python -c "
import json
d=json.loads(open('gpurun_out/ab.json').read().strip().splitlines()[-1])
k=d['kernels']
print('bench pdl=$v', round(d['value'],1), round(d['ms_per_step'],2), d['clocks']['sm_mhz'], 'e2e', round(d['e2e']['value'],1), {c: round(x['seconds']/d['steps']*1e3,2) for c,x in k.items() if x['seconds']})" || tail -5 gpurun_out/ab.err
done
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 1500 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/r02_gpu_tests_pdl.txt 2>&1; echo "tests $?"; tail -2 gpurun_out/r02_gpu_tests_pdl.txt
