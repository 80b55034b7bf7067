# Every bench workload on one B200 (run under gpurun): writes gpurun_out/final_<workload>.json
timeout 900 python bench.py > gpurun_out/final_cfg2.json 2> gpurun_out/final_cfg2.err; echo "cfg2 exit $?"
timeout 900 python bench.py --workload cfg3 --no-cpu-baseline > gpurun_out/final_cfg3.json 2> gpurun_out/final_cfg3.err; echo "cfg3 exit $?"
timeout 1200 python bench.py --workload cfg4s --no-cpu-baseline --steps 3 > gpurun_out/final_cfg4s.json 2> gpurun_out/final_cfg4s.err; echo "cfg4s exit $?"
timeout 600 python bench.py --workload cfg1 --no-cpu-baseline > gpurun_out/final_cfg1.json 2> gpurun_out/final_cfg1.err; echo "cfg1 exit $?"
timeout 900 python bench.py --workload cfg5 --steps 3 > gpurun_out/final_cfg5.json 2> gpurun_out/final_cfg5.err; echo "cfg5 exit $?"
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/final_ref.json 2> gpurun_out/final_ref.err; echo "ref exit $?"
for f in cfg2 cfg3 cfg4s cfg1 cfg5 ref; do python -c "import json;d=json.loads(open('gpurun_out/final_$f.json').read().strip().splitlines()[-1]);print('$f', d.get('value'), d.get('unit'), (d.get('roofline') or {}).get('frac'), (d.get('step_roofline') or {}).get('frac_strict'), (d.get('e2e') or {}).get('value'))"; done
