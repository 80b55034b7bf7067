# e2e with pageable host inputs (X and T staged to pinned memory on the host's cores), default cfg2 bench
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
timeout 600 python -m pytest tests/test_gpu_step.py -m gpu -x -q -p no:cacheprovider -k "pageable or host_inputs or graph" 2>&1 | tail -1
for i in 1 2; do
  timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/ab.json 2>gpurun_out/ab.err
  python -c "
import json
d=json.loads(open('gpurun_out/ab.json').read().strip().splitlines()[-1])
e=d['e2e']
print('value', round(d['value'],1), 'e2e pinned', round(e['value'],1), 'e2e pageable', round(e['pageable_host_inputs']['value'],1), d['clocks']['sm_mhz'])"
done
