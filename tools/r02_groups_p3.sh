# stash policy 3 with microbatch groups (direction balance) at the 8 GiB cap, vs the default
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
for v in "2 2 1" "3 4 2" "3 4 4" "3 8 4" "2 4 2" "2 2 1"; do
  set -- $v
  timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --stash-policy $1 --microbatches $2 --groups $3 > gpurun_out/ab.json 2>gpurun_out/ab.err
  python -c "
import json
d=json.loads(open('gpurun_out/ab.json').read().strip().splitlines()[-1])
print('policy $1 m $2 G $3', round(d['value'],1), round(d['ms_per_step'],2), d['clocks']['sm_mhz'], 'h2d', round(d['step_roofline']['h2d_bytes_per_step']/1e9,2))" || tail -3 gpurun_out/ab.err
done
