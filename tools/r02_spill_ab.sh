# does the stash spill traffic pace the step?  staging slots 2 / 4, and the same step uncapped-ish (16 GiB: no spills)
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
for v in "X=0" "HARMONY_STAGE_SLOTS=4" "HARMONY_STAGE_SLOTS=6" "X=1 --cap-gib 16" "X=0"; do
  set -- $v; env $1 timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline $2 $3 > gpurun_out/ab.json 2>gpurun_out/ab.err
  python -c "
import json
d=json.loads(open('gpurun_out/ab.json').read().strip().splitlines()[-1])
print('$v', round(d['value'],1), round(d['ms_per_step'],2), d['clocks']['sm_mhz'], 'h2d', d['step_roofline']['h2d_bytes_per_step'])" || tail -5 gpurun_out/ab.err
done
