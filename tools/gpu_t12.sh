python tools/timeline.py --workload cfg2 --microbatches 2 --out gpurun_out/timeline_cfg2_m2.json > /dev/null 2>&1
python -c "
import json; d=json.load(open('gpurun_out/timeline_cfg2_m2.json'))['summary']
print('g2', round(d['plain_step_ms'],1), round(d['compute_idle_ms'],1), round(d['h2d']['busy_ms'],1), round(d['d2h']['busy_ms'],1), d['compute_idle_top'][:4])"
for g in 3 4; do
HARMONY_STAGE_SLOTS=$g timeout 900 python bench.py --no-cpu-baseline > gpurun_out/bench_g$g.json 2>/dev/null
python -c "import json;d=json.load(open('gpurun_out/bench_g$g.json'));print('cfg2 g$g', round(d['value'],1), d['clocks']['sm_mhz'], d['plan']['pred_h2d_bytes'])"
done
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/bench_g2.json 2>/dev/null
python -c "import json;d=json.load(open('gpurun_out/bench_g2.json'));print('cfg2 g2', round(d['value'],1), d['clocks']['sm_mhz'], d['plan']['pred_h2d_bytes'])"
