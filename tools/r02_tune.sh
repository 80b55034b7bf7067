# the tuner over (m, G, stash policy, forward pack) on cfg2
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
timeout 1500 python bench.py --tune --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/r02_final_cfg2_tuned.json 2> gpurun_out/r02_final_cfg2_tuned.err; echo "tune $?"
python -c "
import json
d=json.loads(open('gpurun_out/r02_final_cfg2_tuned.json').read().strip().splitlines()[-1])
t=d['config']['tuning']; print('best', t['best'], 'value', round(d['value'],1))
for c in t['candidates']:
    if c['ms'] is not None: print(c)"
