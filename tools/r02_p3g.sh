# stash policy 2 vs 3 x microbatches x groups at cfg2 (direction balancing of the stash traffic)
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
for cfg in "2 2 1" "3 2 1" "3 2 2" "2 4 1" "3 4 1" "3 4 2" "3 4 4" "2 2 2"; do
set -- $cfg
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --stash-policy $1 --microbatches $2 --groups $3 > gpurun_out/r02_p3g_$1_$2_$3.json 2>/dev/null
python -c "
import json
d=json.loads(open('gpurun_out/r02_p3g_$1_$2_$3.json').read().strip().splitlines()[-1])
p=d['plan']
print('policy $1 m $2 G $3', round(d['value'],1), round(d['ms_per_step'],1), 'h2d', p['pred_h2d_bytes']/1e9, 'd2h', p['pred_d2h_bytes']/1e9, 'clk', d['clocks']['sm_mhz'])" 2>&1 | tail -1
done
