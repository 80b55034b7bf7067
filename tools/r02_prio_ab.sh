# same-box A/B: compute-stream priority on (default) / off (HARMONY_PRIO=0)
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
for v in 1 0 1 0 1 0; do
  HARMONY_PRIO=$v timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/ab.json 2>gpurun_out/ab.err
  python -c "
import json
d=json.loads(open('gpurun_out/ab.json').read().strip().splitlines()[-1])
print('prio=$v', round(d['value'],1), round(d['ms_per_step'],2), d['clocks']['sm_mhz'])"
done
