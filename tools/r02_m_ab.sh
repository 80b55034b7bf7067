# microbatch count A/B at cfg2 (64 sequences per GPU): m = 1 (T = 32768 tokens per GEMM) vs m = 2
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1; echo "build $?"
for v in "--microbatches 1" "--microbatches 2" "--microbatches 1 --groups 1 --stash-policy 3"; do
  timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline $v > gpurun_out/ab.json 2>gpurun_out/ab.err
  python -c "
import json
d=json.loads(open('gpurun_out/ab.json').read().strip().splitlines()[-1])
sr=d['step_roofline']; k=d['kernels']
print('$v', 'samples/s', round(d['value'],1), 'ms', round(d['ms_per_step'],2), 'clk', d['clocks']['sm_mhz'], 'h2d GB', round(sr['h2d_bytes_per_step']/1e9,2), {c: round(v['seconds']/d['steps']*1e3,2) for c,v in k.items() if v['seconds']})" || tail -3 gpurun_out/ab.err
done
