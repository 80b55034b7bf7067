# cfg3s: full cfg3 under a 6 GiB cap (4.1x), plus the default cfg2 line at HEAD
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
SECONDS=0; timeout 1500 python bench.py --workload cfg3s --no-cpu-baseline --steps 3 --warmup 3 > gpurun_out/r02_bench_cfg3s.json 2> gpurun_out/r02_bench_cfg3s.err; echo "cfg3s $? ${SECONDS}s"
tail -3 gpurun_out/r02_bench_cfg3s.err
timeout 900 python bench.py --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/r02_bench_cfg2_s2.json 2> gpurun_out/r02_bench_cfg2_s2.err; echo "cfg2 $?"
for f in cfg3s cfg2_s2; do python -c "
import json
d=json.loads(open('gpurun_out/r02_bench_$f.json').read().strip().splitlines()[-1])
sr=d['step_roofline']
print('$f', round(d['value'],2), d['unit'], 'ms', round(d['ms_per_step'],1), 'frac_strict', round(sr['frac_strict'],3), 'bound', sr['bound'], 'h2d GB', round(sr['h2d_bytes_per_step']/1e9,2), 'clk', d['clocks'])"; done
