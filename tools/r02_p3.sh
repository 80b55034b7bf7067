# why is stash policy 3 (C + LSE stashed: no attention recompute) slower than policy 2 at cfg2?
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
for pol in 2 3; do
timeout 600 python tools/timeline.py --workload cfg2 --stash-policy $pol > gpurun_out/r02_timeline_cfg2_p$pol.json 2>&1; echo "timeline $pol $?"
timeout 600 python tools/ktimeline.py --workload cfg2 --stash-policy $pol > gpurun_out/r02_ktl_cfg2_p$pol.json 2>&1; echo "ktl $pol $?"
done
for pol in 2 3; do
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --stash-policy $pol > gpurun_out/r02_bench_p$pol.json 2>/dev/null
python -c "
import json
d=json.loads(open('gpurun_out/r02_bench_p$pol.json').read().strip().splitlines()[-1])
print($pol, d['value'], d['ms_per_step'], d['plan'], d['clocks']['sm_mhz'])"
done
