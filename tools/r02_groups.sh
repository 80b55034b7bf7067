# microbatch groups: bitwise tests, then the op-input stash policy (host-link bound) under the 8 GiB cap at G = 1, 2, 4
mkdir -p gpurun_out
python -m paper_conf_hotos_lipmk21_b200.build > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_step.py -m gpu -x -q -k "groups or operator_split" > gpurun_out/t_groups.log 2>&1; echo "groups tests $?"; tail -2 gpurun_out/t_groups.log
for G in 1 2 4; do
  timeout 900 python bench.py --steps 4 --warmup 2 --no-cpu-baseline --stash-policy 0 --microbatches 4 --groups $G > gpurun_out/bench_p0_g$G.json 2> gpurun_out/bench_p0_g$G.err
  python -c "import json;d=json.loads(open('gpurun_out/bench_p0_g$G.json').read().strip().splitlines()[-1]);sr=d['step_roofline'];print('p0 G=$G', round(d['value'],2), round(d['ms_per_step'],1), 'strict', round(sr['frac_strict'],3), 'swap_strict_ms', round(sr['t_swap_strict_ms'],1), 'h2d/d2h GB', sr['h2d_bytes_per_step']/1e9, sr['d2h_bytes_per_step']/1e9, d['clocks']['reasons'])"
done
timeout 900 python bench.py --workload cfg3 --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_cfg3_g1.json 2>&1
timeout 900 python bench.py --workload cfg3 --steps 5 --warmup 3 --no-cpu-baseline --groups 2 > gpurun_out/bench_cfg3_g2.json 2>&1
for G in 1 2; do python -c "import json;d=json.loads(open('gpurun_out/bench_cfg3_g$G.json').read().strip().splitlines()[-1]);sr=d['step_roofline'];print('cfg3 G=$G', round(d['value'],2), round(d['ms_per_step'],1), 'strict', round(sr['frac_strict'],3), sr['h2d_bytes_per_step']/1e9, sr['d2h_bytes_per_step']/1e9)"; done
